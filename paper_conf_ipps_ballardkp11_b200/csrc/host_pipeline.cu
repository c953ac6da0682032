// host_pipeline.cu — sshopm_run_host: end-to-end solve + dedup on HOST buffers.
//
// Tensors are processed in chunks of `chunk_tensors`; chunk c runs on stream
// c % kSlots with its own device buffers, so the host->device copy of one
// chunk, the solve/dedup kernels of another and the device->host copy of a
// third overlap (copy engines and SMs work concurrently).  Only the per-tensor
// dedup records (and optionally the raw per-start outputs) come back.
#include <cstring>
#include <vector>

#include "api_internal.h"
#include "sshopm.h"

using namespace sshopm;

namespace {
constexpr int kSlots = 3;

struct Slot {
  cudaStream_t st = nullptr;
  float *ent = nullptr, *lam = nullptr, *x = nullptr, *olam = nullptr, *ox = nullptr;
  int32_t *it = nullptr, *cnt = nullptr, *mult = nullptr, *rep = nullptr;
  uint8_t* cv = nullptr;
};

void free_slot(Slot& s) {
  if (s.st) cudaStreamSynchronize(s.st);
  cudaFree(s.ent); cudaFree(s.lam); cudaFree(s.x); cudaFree(s.olam); cudaFree(s.ox);
  cudaFree(s.it); cudaFree(s.cnt); cudaFree(s.mult); cudaFree(s.rep); cudaFree(s.cv);
  if (s.st) cudaStreamDestroy(s.st);
  s = Slot();
}
}  // namespace

extern "C" int sshopm_run_host(sshopm_t h, int64_t N, const float* h_entries, int S, const float* h_starts,
                               float alpha, float tol, int maxit, float lam_tol, float ang_tol, int kmax,
                               int32_t* h_out_count, float* h_out_lambda, float* h_out_x, int32_t* h_out_mult,
                               int32_t* h_out_rep, float* h_raw_lambda, float* h_raw_x, int32_t* h_raw_iters,
                               uint8_t* h_raw_converged, int64_t chunk_tensors, unsigned long long* h_total_iters) {
  if (!h || N < 0 || S < 1 || maxit < 0 || kmax < 1) return SSHOPM_EINVAL;
  if (h_total_iters) *h_total_iters = 0;
  if (N == 0) return SSHOPM_OK;
  if (!h_entries || !h_starts || !h_out_count || !h_out_lambda || !h_out_x || !h_out_mult) return SSHOPM_EINVAL;
  const bool raw = h_raw_lambda || h_raw_x || h_raw_iters || h_raw_converged;
  if (raw && !(h_raw_lambda && h_raw_x && h_raw_iters && h_raw_converged)) return SSHOPM_EINVAL;
  const int n = h->L->n, U = h->L->U;
  long long chunk = chunk_tensors > 0 ? chunk_tensors : 65536;
  if (chunk > N) chunk = N;

  int rc = SSHOPM_OK;
  Slot slots[kSlots];
  float* d_starts = nullptr;
  unsigned long long* d_total = nullptr;
  cudaError_t e = cudaSuccess;
#define CK(call, where) do { e = (call); if (e != cudaSuccess) { rc = (e == cudaErrorMemoryAllocation) ? SSHOPM_ENOMEM : cuda_fail(e, where); goto done; } } while (0)
  CK(cudaMalloc(&d_starts, sizeof(float) * S * n), "run_host: malloc");
  CK(cudaMalloc(&d_total, sizeof(unsigned long long)), "run_host: malloc");
  for (int i = 0; i < kSlots && i * chunk < N; ++i) {
    Slot& s = slots[i];
    CK(cudaStreamCreateWithFlags(&s.st, cudaStreamNonBlocking), "run_host: stream");
    CK(cudaMalloc(&s.ent, sizeof(float) * chunk * U), "run_host: malloc");
    CK(cudaMalloc(&s.lam, sizeof(float) * chunk * S), "run_host: malloc");
    CK(cudaMalloc(&s.x, sizeof(float) * chunk * S * n), "run_host: malloc");
    CK(cudaMalloc(&s.it, sizeof(int32_t) * chunk * S), "run_host: malloc");
    CK(cudaMalloc(&s.cv, chunk * S), "run_host: malloc");
    CK(cudaMalloc(&s.cnt, sizeof(int32_t) * chunk), "run_host: malloc");
    CK(cudaMalloc(&s.olam, sizeof(float) * chunk * kmax), "run_host: malloc");
    CK(cudaMalloc(&s.ox, sizeof(float) * chunk * kmax * n), "run_host: malloc");
    CK(cudaMalloc(&s.mult, sizeof(int32_t) * chunk * kmax), "run_host: malloc");
    CK(cudaMalloc(&s.rep, sizeof(int32_t) * chunk * kmax), "run_host: malloc");
  }
  CK(cudaMemcpyAsync(d_starts, h_starts, sizeof(float) * S * n, cudaMemcpyHostToDevice, slots[0].st), "run_host: H2D");
  CK(cudaMemsetAsync(d_total, 0, sizeof(unsigned long long), slots[0].st), "run_host: memset");
  CK(cudaStreamSynchronize(slots[0].st), "run_host: sync");
  for (long long c0 = 0, ci = 0; c0 < N; c0 += chunk, ++ci) {
    Slot& s = slots[ci % kSlots];
    const long long cn = (N - c0 < chunk) ? (N - c0) : chunk;
    CK(cudaMemcpyAsync(s.ent, h_entries + c0 * U, sizeof(float) * cn * U, cudaMemcpyHostToDevice, s.st), "run_host: H2D");
    sshopm_solve_opts o;
    memset(&o, 0, sizeof(o));
    o.d_total_iters = d_total;
    rc = sshopm_solve_ex(h, cn, s.ent, S, d_starts, alpha, tol, maxit, s.lam, s.x, s.it, s.cv, &o, s.st);
    if (rc != SSHOPM_OK) goto done;
    rc = dedup_impl(h->L, cn, S, s.lam, s.x, s.cv, lam_tol, ang_tol, kmax, s.cnt, s.olam, s.ox, s.mult, s.rep, s.st);
    if (rc != SSHOPM_OK) goto done;
    h->launches.fetch_add(1);
    CK(cudaMemcpyAsync(h_out_count + c0, s.cnt, sizeof(int32_t) * cn, cudaMemcpyDeviceToHost, s.st), "run_host: D2H");
    CK(cudaMemcpyAsync(h_out_lambda + c0 * kmax, s.olam, sizeof(float) * cn * kmax, cudaMemcpyDeviceToHost, s.st), "run_host: D2H");
    CK(cudaMemcpyAsync(h_out_x + c0 * kmax * n, s.ox, sizeof(float) * cn * kmax * n, cudaMemcpyDeviceToHost, s.st), "run_host: D2H");
    CK(cudaMemcpyAsync(h_out_mult + c0 * kmax, s.mult, sizeof(int32_t) * cn * kmax, cudaMemcpyDeviceToHost, s.st), "run_host: D2H");
    if (h_out_rep)
      CK(cudaMemcpyAsync(h_out_rep + c0 * kmax, s.rep, sizeof(int32_t) * cn * kmax, cudaMemcpyDeviceToHost, s.st), "run_host: D2H");
    if (raw) {
      CK(cudaMemcpyAsync(h_raw_lambda + c0 * S, s.lam, sizeof(float) * cn * S, cudaMemcpyDeviceToHost, s.st), "run_host: D2H");
      CK(cudaMemcpyAsync(h_raw_x + c0 * S * n, s.x, sizeof(float) * cn * S * n, cudaMemcpyDeviceToHost, s.st), "run_host: D2H");
      CK(cudaMemcpyAsync(h_raw_iters + c0 * S, s.it, sizeof(int32_t) * cn * S, cudaMemcpyDeviceToHost, s.st), "run_host: D2H");
      CK(cudaMemcpyAsync(h_raw_converged + c0 * S, s.cv, cn * S, cudaMemcpyDeviceToHost, s.st), "run_host: D2H");
    }
  }
  for (int i = 0; i < kSlots; ++i)
    if (slots[i].st) CK(cudaStreamSynchronize(slots[i].st), "run_host: sync");
  if (h_total_iters) CK(cudaMemcpy(h_total_iters, d_total, sizeof(unsigned long long), cudaMemcpyDeviceToHost), "run_host: D2H");
#undef CK
done:
  for (int i = 0; i < kSlots; ++i) free_slot(slots[i]);
  cudaFree(d_starts);
  cudaFree(d_total);
  return rc;
}
