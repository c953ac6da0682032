// api_internal.h — helpers shared by the C-ABI translation units.
#pragma once
#include <atomic>
#include <cuda_runtime.h>
#include <stdint.h>
#include "launchers.h"

namespace sshopm { struct HostCache; struct GeneralTables; }

struct sshopm_ctx {
  const sshopm::Launchers* L;      // compiled (m, n) kernels, or null
  // host-side launch-shape cache (occupancy per non-fused kernel variant, per device); 0 = not computed
  std::atomic<int> occ_dev;
  std::atomic<int> occ[4][2][6];   // [shift][wide][schedule - 1]
  sshopm::GeneralTables* gen;      // table-driven kernel tables (any (m, n))
  int m, n, U;
  std::atomic<long long> launches;
  sshopm::HostCache* hc;     // run_host device buffers / streams (created lazily, guarded by its mutex)
};

namespace sshopm {
int cuda_fail(cudaError_t e, const char* where);
FastDiv make_fastdiv(uint32_t d);
int device_sms();

struct Workspace {
  void* base = nullptr;
  unsigned int* counter = nullptr;   // 256-byte header: chunk counter of the solve kernel
  float* starts_n = nullptr;         // [S][round4(n)] normalised starts (256-byte aligned region)
  float4* packed = nullptr;          // [N][PW/4] packed coefficient rows
  unsigned int* ovf_count = nullptr; // fused dedup: untracked chunk count (header word 1)
  unsigned int* ovf_list = nullptr;  // fused dedup: untracked chunk indices [n_chunks]
  float* alpha_t = nullptr;          // per-tensor shift [N] (alpha modes 1-3)
  bool owned = false;
};
size_t workspace_bytes(const Launchers* L, int64_t N, int S);
size_t handle_workspace_bytes(const sshopm_ctx* h, int64_t N, int S);
int acquire_workspace(const Launchers* L, int64_t N, int S, void* user, size_t user_bytes, cudaStream_t st, Workspace* ws);
int release_workspace(Workspace* ws, cudaStream_t st);
int dedup_impl(int m, int n, int64_t N, int S, const float* d_lambda, const float* d_x, const uint8_t* d_conv,
               float lam_tol, float ang_tol, int kmax, int32_t* d_count, float* d_olam, float* d_ox, int32_t* d_mult,
               int32_t* d_rep, cudaStream_t st);
void free_host_cache(sshopm_ctx* h);
int chunk_tensors_for(int S);
int make_dedup_params(int n, int64_t N, int S, float lam_tol, float ang_tol, int kmax, int32_t* d_count,
                      float* d_olam, float* d_ox, int32_t* d_mult, int32_t* d_rep, DedupParams* p);
int launch_dedup(int m, int n, const DedupParams& p, cudaStream_t st);
int launch_dedup_list(int m, int n, const DedupParams& p, const unsigned int* count, const unsigned int* list,
                      int chunk_tensors, cudaStream_t st);
}  // namespace sshopm
