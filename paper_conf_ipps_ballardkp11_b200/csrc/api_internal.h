// api_internal.h — helpers shared by the C-ABI translation units.
#pragma once
#include <atomic>
#include <cuda_runtime.h>
#include <stdint.h>
#include "launchers.h"

struct sshopm_ctx {
  const sshopm::Launchers* L;
  std::atomic<long long> launches;
};

namespace sshopm {
int cuda_fail(cudaError_t e, const char* where);
FastDiv make_fastdiv(uint32_t d);
int device_sms();
int dedup_impl(const Launchers* L, int64_t N, int S, const float* d_lambda, const float* d_x, const uint8_t* d_conv,
               float lam_tol, float ang_tol, int kmax, int32_t* d_count, float* d_olam, float* d_ox, int32_t* d_mult,
               int32_t* d_rep, cudaStream_t st);
}  // namespace sshopm
