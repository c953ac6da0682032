// launchers.h — per-(m, n) entry points exported by each compiled instance.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>
#include "sshopm_kernels.cuh"

namespace sshopm {

struct Launchers {
  int m, n, U, Q, PW;        // PW = packed 4-byte words per tensor (multiple of 4)
  long long paper_flops, exec_flops;
  int bform;                 // 1 if the B-form (coefficient-folded) registers are used
  int default_refill;
  int default_schedule;
  int (*wt_smem_per_warp)(int S);       // schedule 7 staging bytes per warp
  void (*class_index)(int32_t* out);   // [U][m], 0-based
  cudaError_t (*occupancy)(int shift, bool wide, int schedule, int fused, int smem_bytes, int* blocks_per_sm);
  cudaError_t (*pack)(long long n_tensors, const float* entries, float4* packed, unsigned int* counter, int n_starts,
                      const float* starts, float* starts_n, int alpha_mode, const float* alpha_in, float* alpha_t,
                      int grid, cudaStream_t st);
  cudaError_t (*solve)(const SolveParams& p, int shift, bool wide, int schedule, int fused, int grid, int smem_bytes,
                       cudaStream_t st);
  cudaError_t (*classify)(long long n_tensors, int kmax, const float* entries, const int32_t* count, const float* lam,
                          const float* x, float ctol, int8_t* out, int grid, cudaStream_t st);
  cudaError_t (*apply)(long long n_items, const float4* packed, const float* x, float* g, float* lam, int grid,
                       cudaStream_t st);
  // records path (schedule 8, sshopm_solve_dedup with fuse_dedup = 4)
  cudaError_t (*occupancy_rec)(int shift, int* blocks_per_sm);
  cudaError_t (*solve_rec)(const RecParams& p, int shift, int grid, cudaStream_t st);
  int solve_tpb;             // threads per CTA of the non-fused schedule-1 solve kernel (256, or 128 for (6,3))
};

}  // namespace sshopm
