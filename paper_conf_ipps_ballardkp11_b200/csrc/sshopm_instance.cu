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

template <int SH>
cudaError_t occ1(int smem, int* bps) {
  return cudaOccupancyMaxActiveBlocksPerMultiprocessor(bps, sshopm_solve_kernel<M, N, SH>, 256, smem);
}
cudaError_t occupancy(int shift, int smem, int* bps) {
  return shift == 0 ? occ1<0>(smem, bps) : shift == 1 ? occ1<1>(smem, bps) : occ1<2>(smem, bps);
}

template <int SH>
cudaError_t solve1(const SolveParams& p, int grid, int smem, cudaStream_t st) {
  if (smem > 48 * 1024) {
    cudaError_t e = cudaFuncSetAttribute(sshopm_solve_kernel<M, N, SH>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e != cudaSuccess) return e;
  }
  sshopm_solve_kernel<M, N, SH><<<grid, 256, smem, st>>>(p);
  return cudaGetLastError();
}
cudaError_t solve(const SolveParams& p, int shift, int grid, int smem, cudaStream_t st) {
  return shift == 0 ? solve1<0>(p, grid, smem, st) : shift == 1 ? solve1<1>(p, grid, smem, st) : solve1<2>(p, grid, smem, st);
}

cudaError_t pack(long long n, const float* e, float4* packed, unsigned int* counter, int grid, cudaStream_t st) {
  sshopm_pack_kernel<M, N><<<grid, 256, 0, st>>>(n, e, packed, counter);
  return cudaGetLastError();
}

cudaError_t apply(long long n_items, const float4* packed, const float* x, float* g, float* lam, int grid, cudaStream_t st) {
  sshopm_apply_kernel<M, N><<<grid, 256, 0, st>>>(n_items, packed, x, g, lam);
  return cudaGetLastError();
}

const Launchers kL = {M, N, Tables<M, N>::U, Tables<M, N>::Q, Sh::PW,
                      paper_flops_per_iter<M, N>(), executed_flops_per_iter<M, N>(),
                      Sh::BFORM ? 1 : 0, 8,
                      class_index, occupancy, pack, solve, apply};
}  // namespace

#define SSHOPM_CAT2(a, b, c) get_launchers_##a##_##b
#define SSHOPM_NAME(a, b) SSHOPM_CAT2(a, b, x)
const Launchers* SSHOPM_NAME(SSHOPM_M, SSHOPM_N)() { return &kL; }

}  // namespace sshopm
