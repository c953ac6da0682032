// sshopm_instance.cu — instantiates the kernels for one (m, n), selected with
// -DSSHOPM_M / -DSSHOPM_N by build.py (one object per line of shapes.def).
#include "launchers.h"

#ifndef SSHOPM_M
#error "define SSHOPM_M and SSHOPM_N"
#endif

namespace sshopm {
namespace {
constexpr int M = SSHOPM_M;
constexpr int N = SSHOPM_N;
using Sh = Shape<M, N>;

void class_index(int32_t* out) {
  constexpr Tables<M, N> T{};
  for (int c = 0; c < T.U; ++c)
    for (int t = 0; t < M; ++t) out[c * M + t] = T.cls_idx[c][t];
}

template <int SH, int MODE>
const void* wt_fn() { return reinterpret_cast<const void*>(sshopm_solve_wt_kernel<M, N, SH, MODE>); }

template <int SH, bool W, int F>
cudaError_t occ2(int schedule, int smem, int* bps) {
  if (schedule == 7) {   // warp-tensor pipeline: F = MODE (0 raw, 1 records only, 2 both); smem = staging bytes
    if constexpr (F <= 2) {
      const void* fn = wt_fn<SH, F>();
      if (smem > 48 * 1024) {
        cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
        if (e != cudaSuccess) return e;
      }
      return cudaOccupancyMaxActiveBlocksPerMultiprocessor(bps, fn, 256, smem);
    }
    return cudaErrorInvalidValue;
  }
  if constexpr (SH == 3) {
    if (schedule == 2) return cudaErrorInvalidValue;         // per-tensor alpha: schedule 1 only
  } else {
    if (schedule == 2) return cudaOccupancyMaxActiveBlocksPerMultiprocessor(bps, sshopm_solve_tpl_kernel<M, N, SH, W>, 256, 0);
  }
  if (schedule == 6 && F == 0)
    return cudaOccupancyMaxActiveBlocksPerMultiprocessor(bps, sshopm_solve_lean_kernel<M, N, SH, W>, 256, 0);
  return cudaOccupancyMaxActiveBlocksPerMultiprocessor(bps, sshopm_solve_kernel<M, N, SH, W, F>,
                                                       (F == 0 || F == 4) ? Sh::TPB : 256, smem);
}
template <int SH, bool W>
cudaError_t occ1(int schedule, int fused, int smem, int* bps) {
  if (fused == 4) return occ2<SH, W, 4>(schedule, smem, bps);   // schedule 1 with item chunks (small N)
  if (fused == 3) return occ2<SH, W, 3>(schedule, smem, bps);
  return fused == 2 ? occ2<SH, W, 2>(schedule, smem, bps) : fused == 1 ? occ2<SH, W, 1>(schedule, smem, bps)
                    : occ2<SH, W, 0>(schedule, smem, bps);
}
template <bool W>
cudaError_t occw(int shift, int schedule, int fused, int smem, int* bps) {
  switch (shift) {
    case 0: return occ1<0, W>(schedule, fused, smem, bps);
    case 1: return occ1<1, W>(schedule, fused, smem, bps);
    case 2: return occ1<2, W>(schedule, fused, smem, bps);
    default: return occ1<3, W>(schedule, fused, smem, bps);
  }
}
cudaError_t occupancy(int shift, bool wide, int schedule, int fused, int smem, int* bps) {
  return wide ? occw<true>(shift, schedule, fused, smem, bps) : occw<false>(shift, schedule, fused, smem, bps);
}

template <int SH, bool W, int F>
cudaError_t solve2(const SolveParams& p, int schedule, int grid, int smem, cudaStream_t st) {
  if (schedule == 7) {
    if constexpr (!W && F <= 2) {
      if (smem > 48 * 1024) {
        cudaError_t e = cudaFuncSetAttribute(sshopm_solve_wt_kernel<M, N, SH, F>,
                                             cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
        if (e != cudaSuccess) return e;
      }
      sshopm_solve_wt_kernel<M, N, SH, F><<<grid, 256, smem, st>>>(p);
      return cudaGetLastError();
    }
    return cudaErrorInvalidValue;                            // the api launches schedule 7 with W = false
  }
  if (schedule == 2) {
    if constexpr (SH == 3) return cudaErrorInvalidValue;     // per-tensor alpha: schedule 1 only
    else sshopm_solve_tpl_kernel<M, N, SH, W><<<grid, 256, 0, st>>>(p);
  } else if (schedule == 6 && F == 0) {                      // lean predicated refill (measured slower, kept)
    sshopm_solve_lean_kernel<M, N, SH, W><<<grid, 256, 0, st>>>(p);
  } else {                                                   // schedule 1 (default) or the fused dedup
    if (smem > 48 * 1024) {
      cudaError_t e = cudaFuncSetAttribute(sshopm_solve_kernel<M, N, SH, W, F>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
      if (e != cudaSuccess) return e;
    }
#ifndef SSHOPM_SOLVE_THREADS
#define SSHOPM_SOLVE_THREADS 256
#endif
    sshopm_solve_kernel<M, N, SH, W, F><<<grid, (F == 0 || F == 4) ? Sh::TPB : SSHOPM_SOLVE_THREADS, smem, st>>>(p);
  }
  return cudaGetLastError();
}
template <int SH, bool W>
cudaError_t solve1(const SolveParams& p, int schedule, int fused, int grid, int smem, cudaStream_t st) {
  if (fused == 4) return solve2<SH, W, 4>(p, schedule, grid, smem, st);   // schedule 1 with item chunks (small N)
  if (fused == 3) return solve2<SH, W, 3>(p, schedule, grid, smem, st);
  return fused == 2 ? solve2<SH, W, 2>(p, schedule, grid, smem, st) : fused == 1 ? solve2<SH, W, 1>(p, schedule, grid, smem, st)
                    : solve2<SH, W, 0>(p, schedule, grid, smem, st);
}
template <bool W>
cudaError_t solvew(const SolveParams& p, int shift, int schedule, int fused, int grid, int smem, cudaStream_t st) {
  switch (shift) {
    case 0: return solve1<0, W>(p, schedule, fused, grid, smem, st);
    case 1: return solve1<1, W>(p, schedule, fused, grid, smem, st);
    case 2: return solve1<2, W>(p, schedule, fused, grid, smem, st);
    default: return solve1<3, W>(p, schedule, fused, grid, smem, st);
  }
}
cudaError_t solve(const SolveParams& p, int shift, bool wide, int schedule, int fused, int grid, int smem, cudaStream_t st) {
  return wide ? solvew<true>(p, shift, schedule, fused, grid, smem, st) : solvew<false>(p, shift, schedule, fused, grid, smem, st);
}

cudaError_t pack(long long n, const float* e, float4* packed, unsigned int* counter, int n_starts, const float* starts,
                 float* starts_n, int alpha_mode, const float* alpha_in, float* alpha_t, int grid, cudaStream_t st) {
  sshopm_pack_kernel<M, N><<<grid, 256, 0, st>>>(n, e, packed, counter, n_starts, starts, starts_n, alpha_mode, alpha_in,
                                                 alpha_t);
  return cudaGetLastError();
}

cudaError_t classify(long long n, int kmax, const float* e, const int32_t* count, const float* lam, const float* x,
                     float ctol, int8_t* out, int grid, cudaStream_t st) {
  sshopm_classify_kernel<M, N><<<grid, 128, 0, st>>>(n, kmax, e, count, lam, x, ctol, out);
  return cudaGetLastError();
}

cudaError_t apply(long long n_items, const float4* packed, const float* x, float* g, float* lam, int grid, cudaStream_t st) {
  sshopm_apply_kernel<M, N><<<grid, 256, 0, st>>>(n_items, packed, x, g, lam);
  return cudaGetLastError();
}

int wt_smem(int S) { return wt_smem_per_warp<N>(S); }

cudaError_t occupancy_rec(int shift, int* bps) {
  switch (shift) {
    case 0: return cudaOccupancyMaxActiveBlocksPerMultiprocessor(bps, sshopm_solve_rec_kernel<M, N, 0>, 256, 0);
    case 1: return cudaOccupancyMaxActiveBlocksPerMultiprocessor(bps, sshopm_solve_rec_kernel<M, N, 1>, 256, 0);
    case 2: return cudaOccupancyMaxActiveBlocksPerMultiprocessor(bps, sshopm_solve_rec_kernel<M, N, 2>, 256, 0);
    default: return cudaOccupancyMaxActiveBlocksPerMultiprocessor(bps, sshopm_solve_rec_kernel<M, N, 3>, 256, 0);
  }
}
cudaError_t solve_rec(const RecParams& p, int shift, int grid, cudaStream_t st) {
  switch (shift) {
    case 0: sshopm_solve_rec_kernel<M, N, 0><<<grid, 256, 0, st>>>(p); break;
    case 1: sshopm_solve_rec_kernel<M, N, 1><<<grid, 256, 0, st>>>(p); break;
    case 2: sshopm_solve_rec_kernel<M, N, 2><<<grid, 256, 0, st>>>(p); break;
    default: sshopm_solve_rec_kernel<M, N, 3><<<grid, 256, 0, st>>>(p); break;
  }
  return cudaGetLastError();
}

const Launchers kL = {M, N, Tables<M, N>::U, Tables<M, N>::Q, Sh::PW,
                      paper_flops_per_iter<M, N>(), executed_flops_per_iter<M, N>(),
                      Sh::BFORM ? 1 : 0,
                      steps_per_trip<M, N>() == 4 ? 10 : (steps_per_trip<M, N>() == 3 && !(N == 3 && M >= 6) ? 8
                                                          : (N == 3 && M >= 8 ? 4 : 6)), 1,   // refill threshold K
                      // ((8,3) with the Horner step: K = 4, C4a 5.27 -> 5.23 ms; (6,3) keeps 6: profiles/r2/horner3.md)
                      // (swept on B200: profiles/r1/solve_variants.txt, profiles/r2/solve_variants_s6.jsonl)
                      wt_smem, class_index, occupancy, pack, solve, classify, apply, occupancy_rec, solve_rec, Sh::TPB};
}  // namespace

#define SSHOPM_CAT2(a, b, c) get_launchers_##a##_##b
#define SSHOPM_NAME(a, b) SSHOPM_CAT2(a, b, x)
const Launchers* SSHOPM_NAME(SSHOPM_M, SSHOPM_N)() { return &kL; }

}  // namespace sshopm
