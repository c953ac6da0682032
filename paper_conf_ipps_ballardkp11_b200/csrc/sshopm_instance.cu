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

cudaError_t occupancy(bool neg, int smem, int* bps) {
  return neg ? cudaOccupancyMaxActiveBlocksPerMultiprocessor(bps, sshopm_solve_kernel<M, N, true>, 256, smem)
             : cudaOccupancyMaxActiveBlocksPerMultiprocessor(bps, sshopm_solve_kernel<M, N, false>, 256, smem);
}

cudaError_t solve(const SolveParams& p, bool neg, int grid, int smem, cudaStream_t st) {
  if (smem > 48 * 1024) {
    cudaError_t e = neg ? cudaFuncSetAttribute(sshopm_solve_kernel<M, N, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem)
                        : cudaFuncSetAttribute(sshopm_solve_kernel<M, N, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e != cudaSuccess) return e;
  }
  if (neg) sshopm_solve_kernel<M, N, true><<<grid, 256, smem, st>>>(p);
  else sshopm_solve_kernel<M, N, false><<<grid, 256, smem, st>>>(p);
  return cudaGetLastError();
}

cudaError_t apply(long long n_items, const float* e, const float* x, float* g, float* lam, int grid, cudaStream_t st) {
  sshopm_apply_kernel<M, N><<<grid, 256, 0, st>>>(n_items, e, x, g, lam);
  return cudaGetLastError();
}

const Launchers kL = {M, N, Tables<M, N>::U, Tables<M, N>::Q,
                      paper_flops_per_iter<M, N>(), executed_flops_per_iter<M, N>(),
                      Sh::BFORM ? 1 : 0, 8,
                      class_index, occupancy, solve, apply};
}  // namespace

#define SSHOPM_CAT2(a, b, c) get_launchers_##a##_##b
#define SSHOPM_NAME(a, b) SSHOPM_CAT2(a, b, x)
const Launchers* SSHOPM_NAME(SSHOPM_M, SSHOPM_N)() { return &kL; }

}  // namespace sshopm
