// host_pipeline.cu — sshopm_run_host: end-to-end solve + dedup on HOST buffers.
//
// Tensors are processed in chunks of `chunk_tensors`; chunk c uses slot c % kSlots with its own device
// buffers and two streams: the host->device copy and the solve on a lowest-priority stream, the dedup and
// the device->host copies on a highest-priority stream (so a finished chunk's dedup CTAs are scheduled
// before the next chunk's pending solve CTAs; with one stream per slot the order varied from call to call:
// C2 e2e 5.12-6.17 ms, now 5.20-5.25), so copies and kernels of different chunks overlap.  Only the
// per-tensor dedup records (and optionally the raw per-start outputs) come back.
//
// Device buffers and streams are cached in the handle (HostCache) and reused
// across calls — allocation, not transfer, would otherwise dominate; calls on
// one handle serialise on the cache mutex.  sshopm_destroy frees the cache.
#include <cstdlib>
#include <cstring>
#include <chrono>
#include <mutex>
#include <vector>
#include <cstdio>

#include "api_internal.h"
#include "sshopm.h"

using namespace sshopm;

namespace sshopm {
constexpr int kSlots = 3;

struct Slot {
  cudaStream_t st = nullptr;       // H2D, pack + solve (lowest priority)
  cudaStream_t hi = nullptr;       // dedup + D2H (highest priority: their CTAs go before pending solve CTAs)
  cudaEvent_t solved = nullptr, done = nullptr;
  float *ent = nullptr, *lam = nullptr, *x = nullptr, *olam = nullptr, *ox = nullptr;
  int32_t *it = nullptr, *cnt = nullptr, *mult = nullptr, *rep = nullptr;
  uint8_t* cv = nullptr;
  void* ws = nullptr;
  size_t ws_bytes = 0;
};

struct HostCache {
  std::mutex mu;
  int device = -1;
  long long chunk = 0;
  int S = 0, kmax = 0;
  Slot slots[kSlots];
  float* d_starts = nullptr;
  unsigned long long* d_total = nullptr;
};

static void free_slots(HostCache* c) {
  for (int i = 0; i < kSlots; ++i) {
    Slot& s = c->slots[i];
    if (s.st) cudaStreamSynchronize(s.st);
    if (s.hi) cudaStreamSynchronize(s.hi);
    cudaFree(s.ent); cudaFree(s.lam); cudaFree(s.x); cudaFree(s.olam); cudaFree(s.ox);
    cudaFree(s.it); cudaFree(s.cnt); cudaFree(s.mult); cudaFree(s.rep); cudaFree(s.cv); cudaFree(s.ws);
    if (s.st) cudaStreamDestroy(s.st);
    if (s.hi) cudaStreamDestroy(s.hi);
    if (s.solved) cudaEventDestroy(s.solved);
    if (s.done) cudaEventDestroy(s.done);
    s = Slot();
  }
  cudaFree(c->d_starts);
  cudaFree(c->d_total);
  c->d_starts = nullptr;
  c->d_total = nullptr;
  c->chunk = 0;
}

void free_host_cache(sshopm_ctx* h) {
  if (!h->hc) return;
  int cur = -1;
  cudaGetDevice(&cur);
  if (h->hc->device >= 0) cudaSetDevice(h->hc->device);
  free_slots(h->hc);
  if (cur >= 0) cudaSetDevice(cur);
  delete h->hc;
  h->hc = nullptr;
}
}  // namespace sshopm

extern "C" int sshopm_run_host(sshopm_t h, int64_t N, const float* h_entries, int S, const float* h_starts,
                               float alpha, float tol, int maxit, float lam_tol, float ang_tol, int kmax,
                               int32_t* h_out_count, float* h_out_lambda, float* h_out_x, int32_t* h_out_mult,
                               int32_t* h_out_rep, float* h_raw_lambda, float* h_raw_x, int32_t* h_raw_iters,
                               uint8_t* h_raw_converged, int64_t chunk_tensors, unsigned long long* h_total_iters) {
  const auto t_enter = std::chrono::steady_clock::now();
  if (!h || N < 0 || S < 1 || maxit < 0 || kmax < 1) return SSHOPM_EINVAL;
  if (h_total_iters) *h_total_iters = 0;
  if (N == 0) return SSHOPM_OK;
  if (!h_entries || !h_starts || !h_out_count || !h_out_lambda || !h_out_x || !h_out_mult) return SSHOPM_EINVAL;
  const bool raw = h_raw_lambda || h_raw_x || h_raw_iters || h_raw_converged;
  if (raw && !(h_raw_lambda && h_raw_x && h_raw_iters && h_raw_converged)) return SSHOPM_EINVAL;
  const int n = h->n, U = h->U;
  // default: N / 8 tensors per chunk, clamped to 64K..256K (round 2 sweep with the dedup / D2H on a high-priority
  // stream, profiles/r2/e2e_chunks.txt: C2 128K 5.15 / 64K 5.26 ms, C3 128K 11.84, C4a 64K 6.02 / 32K 6.18,
  // C5 256K 37.6 / 128K 38.3; round 1: profiles/r1/e2e_sweep.txt)
  long long chunk = chunk_tensors > 0 ? chunk_tensors : N / 8;
  if (chunk_tensors <= 0) chunk = chunk < 65536 ? 65536 : (chunk > 262144 ? 262144 : chunk);
  if (chunk > N) chunk = N;

  HostCache* c;
  {
    // lazy creation under a process-wide lock, so concurrent first calls on one handle create one cache
    static std::mutex create_mu;
    std::lock_guard<std::mutex> g(create_mu);
    if (!h->hc) h->hc = new (std::nothrow) HostCache;
    c = h->hc;
  }
  if (!c) return SSHOPM_ENOMEM;
  std::lock_guard<std::mutex> lock(c->mu);
  int dev = 0;
  cudaGetDevice(&dev);
  // SSHOPM_E2E_TRACE=file: append a per-chunk timeline (H2D start/end, kernels end, D2H end; ms from the
  // first event) to `file` — a diagnostic for the pipeline's exposed fill / drain, off by default
  static const char* trace_path = getenv("SSHOPM_E2E_TRACE");
  std::vector<cudaEvent_t> tev;
  std::vector<long long> tcn;
  int rc = SSHOPM_OK;
  cudaError_t e = cudaSuccess;
#define CK(call, where) do { e = (call); if (e != cudaSuccess) { rc = (e == cudaErrorMemoryAllocation) ? SSHOPM_ENOMEM : cuda_fail(e, where); goto done; } } while (0)
  if (c->device != dev || c->chunk < chunk || c->S != S || c->kmax < kmax) {
    if (c->device >= 0) {
      int cur = dev;
      cudaSetDevice(c->device);
      free_slots(c);
      cudaSetDevice(cur);
    }
    c->device = dev;
    c->S = S;
    c->kmax = kmax;
    CK(cudaMalloc(&c->d_starts, sizeof(float) * S * n), "run_host: malloc");
    CK(cudaMalloc(&c->d_total, sizeof(unsigned long long)), "run_host: malloc");
    for (int i = 0; i < kSlots; ++i) {
      Slot& s = c->slots[i];
      int plo = 0, phi = 0;
      CK(cudaDeviceGetStreamPriorityRange(&plo, &phi), "run_host: priorities");
      CK(cudaStreamCreateWithPriority(&s.st, cudaStreamNonBlocking, plo), "run_host: stream");
      CK(cudaStreamCreateWithPriority(&s.hi, cudaStreamNonBlocking, phi), "run_host: stream");
      CK(cudaEventCreateWithFlags(&s.solved, cudaEventDisableTiming), "run_host: event");
      CK(cudaEventCreateWithFlags(&s.done, cudaEventDisableTiming), "run_host: event");
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
      s.ws_bytes = handle_workspace_bytes(h, chunk, S);
      CK(cudaMalloc(&s.ws, s.ws_bytes), "run_host: malloc");
    }
    c->chunk = chunk;
  }
  static const bool ramp = [] { const char* v = getenv("SSHOPM_RAMP"); return !(v && v[0] == '0'); }();
  CK(cudaMemcpyAsync(c->d_starts, h_starts, sizeof(float) * S * n, cudaMemcpyHostToDevice, c->slots[0].st), "run_host: H2D");
  CK(cudaMemsetAsync(c->d_total, 0, sizeof(unsigned long long), c->slots[0].st), "run_host: memset");
  CK(cudaStreamSynchronize(c->slots[0].st), "run_host: sync");
  {
  const auto t_setup = std::chrono::steady_clock::now();
  for (long long c0 = 0, ci = 0, cn = 0; c0 < N; c0 += cn, ++ci) {
    Slot& s = c->slots[ci % kSlots];
    // ramped chunk sizes: chunk/4, chunk/2 first and last, so the exposed pipeline fill (first H2D) and
    // drain (last dedup + D2H) are short; full chunks in between (SSHOPM_RAMP=0 disables)
    const long long left = N - c0;
    cn = chunk;
    if (ramp && N > 4 * chunk) {
      const long long q = chunk / 4;
      if (ci == 0) cn = q;                                   // ramp up: chunk/4, chunk/2, chunk, ...
      else if (ci == 1) cn = 2 * q;
      else if (left > chunk + 2 * q) cn = chunk < left - 3 * q ? chunk : left - 3 * q;   // leave >= 3/4 chunk
      else if (left > 2 * q) cn = left - q;                 // ... and end on a quarter chunk
    }
    if (cn > chunk) cn = chunk;                              // the buffers hold `chunk` tensors (q = chunk / 4 rounds down)
    if (cn < 1) cn = 1;
    if (cn > left) cn = left;
    auto mark = [&]() {
      if (!trace_path) return;
      cudaEvent_t ev;
      cudaEventCreate(&ev);
      cudaEventRecord(ev, s.st);
      tev.push_back(ev);
    };
    if (trace_path) tcn.push_back(cn);
    CK(cudaStreamWaitEvent(s.st, s.done, 0), "run_host: wait");      // the slot's previous dedup / D2H
    mark();
    CK(cudaMemcpyAsync(s.ent, h_entries + c0 * U, sizeof(float) * cn * U, cudaMemcpyHostToDevice, s.st), "run_host: H2D");
    mark();
    sshopm_solve_opts o;
    memset(&o, 0, sizeof(o));
    o.d_total_iters = c->d_total;
    o.d_workspace = s.ws;
    o.workspace_bytes = s.ws_bytes;
    rc = sshopm_solve_ex(h, cn, s.ent, S, c->d_starts, alpha, tol, maxit, s.lam, s.x, s.it, s.cv, &o, s.st);
    if (rc != SSHOPM_OK) goto done;
    CK(cudaEventRecord(s.solved, s.st), "run_host: event");
    CK(cudaStreamWaitEvent(s.hi, s.solved, 0), "run_host: wait");
    rc = sshopm_dedup(h, cn, S, s.lam, s.x, s.cv, lam_tol, ang_tol, kmax, s.cnt, s.olam, s.ox, s.mult, s.rep, s.hi);
    if (rc != SSHOPM_OK) goto done;
    {
      cudaStream_t st_solve = s.st;   // the D2H copies and the trace marks follow on the dedup stream
      s.st = s.hi;
      s.hi = st_solve;
    }
    mark();
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
    mark();
    CK(cudaEventRecord(s.done, s.st), "run_host: event");
    {
      cudaStream_t st_dd = s.st;      // swap back: s.st = solve stream, s.hi = dedup stream
      s.st = s.hi;
      s.hi = st_dd;
    }
  }
  const auto t_enq = std::chrono::steady_clock::now();
  for (int i = 0; i < kSlots; ++i) {
    if (c->slots[i].st) CK(cudaStreamSynchronize(c->slots[i].st), "run_host: sync");
    if (c->slots[i].hi) CK(cudaStreamSynchronize(c->slots[i].hi), "run_host: sync");
  }
  if (trace_path && !tev.empty()) {
    const auto t_sync = std::chrono::steady_clock::now();
    auto ms = [](std::chrono::steady_clock::duration d) { return std::chrono::duration<double, std::milli>(d).count(); };
    if (FILE* f = fopen(trace_path, "a")) {
      fprintf(f, "# run_host N=%lld chunk=%lld: host ms setup %.4f, enqueue %.4f, sync %.4f\n", (long long)N, chunk,
              ms(t_setup - t_enter), ms(t_enq - t_setup), ms(t_sync - t_enq));
      fprintf(f, "# chunk tensors h2d_start h2d_end kernels_end d2h_end (ms)\n");
      for (size_t i = 0; i + 3 < tev.size(); i += 4) {
        float t[4];
        for (int j = 0; j < 4; ++j) cudaEventElapsedTime(&t[j], tev[0], tev[i + j]);
        fprintf(f, "%zu %lld %.4f %.4f %.4f %.4f\n", i / 4, tcn[i / 4], t[0], t[1], t[2], t[3]);
      }
      fclose(f);
    }
    for (cudaEvent_t ev : tev) cudaEventDestroy(ev);
  }
  }
  if (h_total_iters) CK(cudaMemcpy(h_total_iters, c->d_total, sizeof(unsigned long long), cudaMemcpyDeviceToHost), "run_host: D2H");
#undef CK
done:
  if (rc != SSHOPM_OK) {
    for (int i = 0; i < kSlots; ++i) {
      if (c->slots[i].st) cudaStreamSynchronize(c->slots[i].st);
      if (c->slots[i].hi) cudaStreamSynchronize(c->slots[i].hi);
    }
    free_slots(c);
    c->device = -1;
  }
  return rc;
}
