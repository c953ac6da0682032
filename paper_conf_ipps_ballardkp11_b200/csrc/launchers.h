// launchers.h — per-(m, n) entry points exported by each compiled instance.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>
#include "sshopm_kernels.cuh"

namespace sshopm {

struct Launchers {
  int m, n, U, Q;
  long long paper_flops, exec_flops;
  int bform;                 // 1 if the B-form (coefficient-folded) registers are used
  int default_refill;
  void (*class_index)(int32_t* out);   // [U][m], 0-based
  cudaError_t (*occupancy)(bool neg, int smem_bytes, int* blocks_per_sm);
  cudaError_t (*solve)(const SolveParams& p, bool neg, int grid, int smem_bytes, cudaStream_t st);
  cudaError_t (*apply)(long long n_items, const float* e, const float* x, float* g, float* lam, int grid, cudaStream_t st);
};

}  // namespace sshopm
