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

template <int SH, bool W, int F>
cudaError_t occ2(int schedule, int smem, int* bps) {
  return schedule == 2 ? cudaOccupancyMaxActiveBlocksPerMultiprocessor(bps, sshopm_solve_tpl_kernel<M, N, SH, W>, 256, 0)
                       : cudaOccupancyMaxActiveBlocksPerMultiprocessor(bps, sshopm_solve_kernel<M, N, SH, W, F>, 256, smem);
}
template <int SH, bool W>
cudaError_t occ1(int schedule, int fused, int smem, int* bps) {
  return fused == 2 ? occ2<SH, W, 2>(schedule, smem, bps) : fused == 1 ? occ2<SH, W, 1>(schedule, smem, bps)
                    : occ2<SH, W, 0>(schedule, smem, bps);
}
cudaError_t occupancy(int shift, bool wide, int schedule, int fused, int smem, int* bps) {
  if (wide) return shift == 0 ? occ1<0, true>(schedule, fused, smem, bps) : shift == 1 ? occ1<1, true>(schedule, fused, smem, bps) : occ1<2, true>(schedule, fused, smem, bps);
  return shift == 0 ? occ1<0, false>(schedule, fused, smem, bps) : shift == 1 ? occ1<1, false>(schedule, fused, smem, bps) : occ1<2, false>(schedule, fused, smem, bps);
}

template <int SH, bool W, int F>
cudaError_t solve2(const SolveParams& p, int schedule, int grid, int smem, cudaStream_t st) {
  if (schedule == 2) {
    sshopm_solve_tpl_kernel<M, N, SH, W><<<grid, 256, 0, st>>>(p);
  } else {
    if (smem > 48 * 1024) {
      cudaError_t e = cudaFuncSetAttribute(sshopm_solve_kernel<M, N, SH, W, F>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
      if (e != cudaSuccess) return e;
    }
    sshopm_solve_kernel<M, N, SH, W, F><<<grid, 256, smem, st>>>(p);
  }
  return cudaGetLastError();
}
template <int SH, bool W>
cudaError_t solve1(const SolveParams& p, int schedule, int fused, int grid, int smem, cudaStream_t st) {
  return fused == 2 ? solve2<SH, W, 2>(p, schedule, grid, smem, st) : fused == 1 ? solve2<SH, W, 1>(p, schedule, grid, smem, st)
                    : solve2<SH, W, 0>(p, schedule, grid, smem, st);
}
cudaError_t solve(const SolveParams& p, int shift, bool wide, int schedule, int fused, int grid, int smem, cudaStream_t st) {
  if (wide) return shift == 0 ? solve1<0, true>(p, schedule, fused, grid, smem, st) : shift == 1 ? solve1<1, true>(p, schedule, fused, grid, smem, st) : solve1<2, true>(p, schedule, fused, grid, smem, st);
  return shift == 0 ? solve1<0, false>(p, schedule, fused, grid, smem, st) : shift == 1 ? solve1<1, false>(p, schedule, fused, grid, smem, st) : solve1<2, false>(p, schedule, fused, grid, smem, st);
}

cudaError_t pack(long long n, const float* e, float4* packed, unsigned int* counter, int n_starts, const float* starts,
                 float* starts_n, int grid, cudaStream_t st) {
  sshopm_pack_kernel<M, N><<<grid, 256, 0, st>>>(n, e, packed, counter, n_starts, starts, starts_n);
  return cudaGetLastError();
}

cudaError_t apply(long long n_items, const float4* packed, const float* x, float* g, float* lam, int grid, cudaStream_t st) {
  sshopm_apply_kernel<M, N><<<grid, 256, 0, st>>>(n_items, packed, x, g, lam);
  return cudaGetLastError();
}

const Launchers kL = {M, N, Tables<M, N>::U, Tables<M, N>::Q, Sh::PW,
                      paper_flops_per_iter<M, N>(), executed_flops_per_iter<M, N>(),
                      Sh::BFORM ? 1 : 0, 10, 1,
                      class_index, occupancy, pack, solve, apply};
}  // namespace

#define SSHOPM_CAT2(a, b, c) get_launchers_##a##_##b
#define SSHOPM_NAME(a, b) SSHOPM_CAT2(a, b, x)
const Launchers* SSHOPM_NAME(SSHOPM_M, SSHOPM_N)() { return &kL; }

}  // namespace sshopm
