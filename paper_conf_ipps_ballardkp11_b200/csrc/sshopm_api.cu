// sshopm_api.cu — the C ABI of libsshopm.so (declared in include/sshopm.h).
//
// Argument validation, dispatch over the compiled (m, n) instances
// (shapes.def), launch sizing from the device's SM count and the kernel's
// occupancy, and the dedup kernels.  No device memory is allocated here
// except inside sshopm_run_host (host_pipeline.cu).
#include <atomic>
#include <cmath>
#include <cstdlib>
#include <cstdio>
#include <cstring>
#include <new>

#include "launchers.h"
#include "sshopm.h"
#include "sshopm_dedup.cuh"
#include "api_internal.h"
#include "general.h"

namespace sshopm {
#define SHAPE(mm, nn) const Launchers* get_launchers_##mm##_##nn();
#include "shapes.def"
#undef SHAPE

static const Launchers* find_launchers(int m, int n) {
#define SHAPE(mm, nn) if (m == mm && n == nn) return get_launchers_##mm##_##nn();
#include "shapes.def"
#undef SHAPE
  return nullptr;
}

static thread_local char g_last_cuda_error[512] = "";

int cuda_fail(cudaError_t e, const char* where) {
  snprintf(g_last_cuda_error, sizeof(g_last_cuda_error), "%s: %s (%s)", where, cudaGetErrorName(e), cudaGetErrorString(e));
  return SSHOPM_ECUDA;
}

FastDiv make_fastdiv(uint32_t d) {
  FastDiv f;
  f.d = d;
  uint32_t s = 0;
  while ((1ull << s) < d) ++s;
  f.shift = s;
  f.magic = (uint32_t)((((1ull << 32) * ((1ull << s) - d)) / d) + 1);
  return f;
}

static size_t starts_region(const Launchers* L, int S) {
  const size_t b = (size_t)S * (size_t)((L->n + 3) / 4 * 4) * 4;
  return (b + 255) / 256 * 256;
}

size_t handle_workspace_bytes(const sshopm_ctx* h, int64_t N, int S) {
  return h->L ? workspace_bytes(h->L, N, S) : 256;          // the general kernel needs no workspace
}

#ifndef SSHOPM_CHUNK_ITEMS
#define SSHOPM_CHUNK_ITEMS 256   // schedule 1: items per claimed chunk (whole tensors, at least one)
#endif
int chunk_tensors_for(int S) { return (S >= SSHOPM_CHUNK_ITEMS) ? 1 : (SSHOPM_CHUNK_ITEMS + S - 1) / S; }

static size_t packed_region(const Launchers* L, int64_t N) { return ((size_t)N * (size_t)L->PW * 4 + 255) / 256 * 256; }

static size_t chunk_list_region(int64_t N, int S) {
  (void)S;   // one entry per tensor: chunk indices (schedule 1 fused ring) or tensor indices (schedule 7)
  return ((size_t)N * 4 + 255) / 256 * 256;
}

size_t workspace_bytes(const Launchers* L, int64_t N, int S) {
  return 256 + starts_region(L, S) + packed_region(L, N) + chunk_list_region(N, S) + (size_t)N * 4;
}

int acquire_workspace(const Launchers* L, int64_t N, int S, void* user, size_t user_bytes, cudaStream_t st, Workspace* ws) {
  const size_t need = workspace_bytes(L, N, S);
  ws->owned = false;
  void* base = user;
  if (!user || user_bytes < need || ((uintptr_t)user & 255)) {
    if (user && user_bytes < need) return SSHOPM_EINVAL;
    if (user && ((uintptr_t)user & 255)) return SSHOPM_EINVAL;
    cudaError_t e = cudaMallocAsync(&base, need, st);
    if (e == cudaErrorMemoryAllocation) return SSHOPM_ENOMEM;
    if (e != cudaSuccess) return cuda_fail(e, "workspace: cudaMallocAsync");
    ws->owned = true;
  }
  ws->base = base;
  ws->counter = reinterpret_cast<unsigned int*>(base);
  ws->ovf_count = ws->counter + 1;
  ws->starts_n = reinterpret_cast<float*>(reinterpret_cast<char*>(base) + 256);
  ws->packed = reinterpret_cast<float4*>(reinterpret_cast<char*>(base) + 256 + starts_region(L, S));
  ws->ovf_list = reinterpret_cast<unsigned int*>(reinterpret_cast<char*>(base) + 256 + starts_region(L, S) +
                                                 packed_region(L, N));
  ws->alpha_t = reinterpret_cast<float*>(reinterpret_cast<char*>(base) + 256 + starts_region(L, S) + packed_region(L, N) +
                                         chunk_list_region(N, S));
  return SSHOPM_OK;
}

int release_workspace(Workspace* ws, cudaStream_t st) {
  if (ws->owned && ws->base) {
    cudaError_t e = cudaFreeAsync(ws->base, st);
    ws->base = nullptr;
    if (e != cudaSuccess) return cuda_fail(e, "workspace: cudaFreeAsync");
  }
  return SSHOPM_OK;
}

static std::atomic<int> g_sms_cache[64];

int device_sms() {
  int dev = 0, sms = 0;
  if (cudaGetDevice(&dev) != cudaSuccess) return -1;
  if (dev >= 0 && dev < 64 && (sms = g_sms_cache[dev].load(std::memory_order_relaxed)) > 0) return sms;
  if (cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess) return -1;
  if (dev >= 0 && dev < 64) g_sms_cache[dev].store(sms, std::memory_order_relaxed);
  return sms;
}

// occupancy of a non-fused solve variant, cached in the handle for the current device
static cudaError_t cached_occupancy(sshopm_ctx* h, int shift, bool wide, int schedule, int* bps) {
  int dev = 0;
  const cudaError_t ge = cudaGetDevice(&dev);
  if (ge != cudaSuccess) return ge;
  if (h->occ_dev.load(std::memory_order_acquire) != dev + 1) {
    for (auto& a : h->occ)
      for (auto& b : a)
        for (auto& c : b) c.store(0, std::memory_order_relaxed);
    h->occ_dev.store(dev + 1, std::memory_order_release);
  }
  std::atomic<int>& slot = h->occ[shift][wide ? 1 : 0][schedule - 1];
  int v = slot.load(std::memory_order_relaxed);
  if (v > 0) { *bps = v; return cudaSuccess; }
  cudaError_t e = h->L->occupancy(shift, wide, schedule, 0, 0, &v);
  if (e == cudaSuccess && v > 0) slot.store(v, std::memory_order_relaxed);
  *bps = v;
  return e;
}
}  // namespace sshopm

using namespace sshopm;

extern "C" {

const char* sshopm_status_string(int code) {
  switch (code) {
    case SSHOPM_OK: return "ok";
    case SSHOPM_EINVAL: return "invalid argument";
    case SSHOPM_EUNSUPPORTED: return "unsupported shape or size";
    case SSHOPM_ECUDA: return "CUDA error (see sshopm_last_cuda_error)";
    case SSHOPM_ENOMEM: return "out of memory";
    default: return "unknown status";
  }
}

const char* sshopm_last_cuda_error(void) { return g_last_cuda_error; }

int sshopm_ipc_alloc(size_t bytes, void** d_ptr, void* h_handle) {
  static_assert(sizeof(cudaIpcMemHandle_t) == SSHOPM_IPC_HANDLE_BYTES, "IPC handle size");
  if (!d_ptr || !h_handle || bytes == 0) return SSHOPM_EINVAL;
  *d_ptr = nullptr;
  cudaError_t e = cudaMalloc(d_ptr, bytes);
  if (e == cudaErrorMemoryAllocation) { cudaGetLastError(); return SSHOPM_ENOMEM; }
  if (e != cudaSuccess) return cuda_fail(e, "sshopm_ipc_alloc");
  cudaIpcMemHandle_t hd;
  e = cudaIpcGetMemHandle(&hd, *d_ptr);
  if (e != cudaSuccess) { cudaFree(*d_ptr); *d_ptr = nullptr; return cuda_fail(e, "sshopm_ipc_alloc: handle"); }
  memcpy(h_handle, &hd, sizeof(hd));
  return SSHOPM_OK;
}

int sshopm_ipc_free(void* d_ptr) {
  if (!d_ptr) return SSHOPM_EINVAL;
  cudaError_t e = cudaFree(d_ptr);
  if (e != cudaSuccess) return cuda_fail(e, "sshopm_ipc_free");
  return SSHOPM_OK;
}

int sshopm_ipc_import(const void* h_handle, void** d_ptr) {
  if (!h_handle || !d_ptr) return SSHOPM_EINVAL;
  cudaIpcMemHandle_t hd;
  memcpy(&hd, h_handle, sizeof(hd));
  cudaError_t e = cudaIpcOpenMemHandle(d_ptr, hd, cudaIpcMemLazyEnablePeerAccess);
  if (e != cudaSuccess) return cuda_fail(e, "sshopm_ipc_import");
  return SSHOPM_OK;
}

int sshopm_ipc_release(void* d_ptr) {
  if (!d_ptr) return SSHOPM_EINVAL;
  cudaError_t e = cudaIpcCloseMemHandle(d_ptr);
  if (e != cudaSuccess) return cuda_fail(e, "sshopm_ipc_release");
  return SSHOPM_OK;
}

const char* sshopm_supported_shapes(void) {
  static const char* s =
#define SHAPE(mm, nn) #mm "x" #nn ","
#include "shapes.def"
#undef SHAPE
      "";   // compiled (unrolled) shapes; any other m <= 16, n <= 16 uses the table-driven general kernel
  return s;
}

int sshopm_create(int m, int n, sshopm_t* out) {
  if (!out || m < 2 || n < 1) return SSHOPM_EINVAL;
  *out = nullptr;
  const Launchers* L = find_launchers(m, n);
  GeneralTables* gen = general_create(m, n);                 // also backs opts.schedule = 3 on compiled shapes
  if (!L && !gen) return SSHOPM_EUNSUPPORTED;
  sshopm_ctx* h = new (std::nothrow) sshopm_ctx;
  if (!h) { general_destroy(gen); return SSHOPM_ENOMEM; }
  h->L = L;
  h->gen = gen;
  h->m = m;
  h->n = n;
  h->U = L ? L->U : gen->U;
  h->launches.store(0);
  h->hc = nullptr;
  h->occ_dev.store(0);
  for (auto& a : h->occ)
    for (auto& b : a)
      for (auto& c : b) c.store(0);
  *out = h;
  return SSHOPM_OK;
}

int sshopm_destroy(sshopm_t h) {
  if (h) free_host_cache(h);
  if (h) general_destroy(h->gen);
  delete h;
  return SSHOPM_OK;
}

int sshopm_num_unique(sshopm_t h, int* U) {
  if (!h || !U) return SSHOPM_EINVAL;
  *U = h->U;
  return SSHOPM_OK;
}

int sshopm_class_index(sshopm_t h, int32_t* h_idx) {
  if (!h || !h_idx) return SSHOPM_EINVAL;
  if (h->L) h->L->class_index(h_idx);
  else for (int i = 0; i < h->U * h->m; ++i) h_idx[i] = h->gen->idx[i];
  return SSHOPM_OK;
}

int sshopm_flops_per_iter(sshopm_t h, int64_t* paper, int64_t* executed) {
  if (!h) return SSHOPM_EINVAL;
  if (paper) *paper = h->L ? h->L->paper_flops : h->gen->paper_flops;
  if (executed) *executed = h->L ? h->L->exec_flops : h->gen->exec_flops;
  return SSHOPM_OK;
}

int sshopm_launch_count(sshopm_t h, int64_t* count) {
  if (!h || !count) return SSHOPM_EINVAL;
  *count = h->launches.load();
  return SSHOPM_OK;
}

int sshopm_workspace_size(sshopm_t h, int64_t N, int S, size_t* bytes) {
  if (!h || N < 0 || S < 0 || !bytes) return SSHOPM_EINVAL;
  *bytes = handle_workspace_bytes(h, N, S);
  return SSHOPM_OK;
}

int sshopm_records_size(sshopm_t h, int64_t N, int S, size_t* bytes) {
  if (!h || N < 0 || S < 0 || !bytes) return SSHOPM_EINVAL;
  *bytes = (size_t)N * (size_t)S * 16u * (size_t)sshopm::dd_rec4(h->n);
  return SSHOPM_OK;
}

}  // extern "C"

namespace sshopm {
// The solve (pack + solve kernels) and, if dd != null, the fused dedup (ring
// in the solve kernel + sshopm_dedup_list_kernel for untracked chunks), or the
// standalone dedup after the solve when the fused form does not apply.
// Records path (fuse_dedup = 4, schedule 8): pack, sshopm_solve_rec_kernel into the per-start record scratch,
// dedup of the records.  The raw per-start outputs are not written.
static int solve_records(sshopm_t h, int64_t N, const float* d_entries, int S, const float* d_starts, float alpha,
                         float tol, int maxit, const sshopm_solve_opts* opts, const DedupParams* dd, cudaStream_t st) {
  const Launchers* L = h->L;
  const int sms = device_sms();
  if (sms <= 0) return cuda_fail(cudaGetLastError(), "sshopm_solve_dedup: no device");
  const int alpha_mode = opts->alpha_mode;
  if (alpha_mode < 0 || alpha_mode > 3) return SSHOPM_EINVAL;
  if (alpha_mode == 1 && !opts->d_alpha) return SSHOPM_EINVAL;
  const int shift = alpha_mode ? 3 : (alpha == 0.f ? 0 : (alpha > 0.f ? 1 : 2));
  if (opts->unit_starts < 0) return SSHOPM_EINVAL;
  int unit = opts->unit_starts > 0 ? opts->unit_starts : 32;
  if (unit > S) unit = S;
  const long long upt = (S + unit - 1) / unit;
  const long long n_units = (long long)N * upt;
  if (n_units >= (1LL << 32) - (1LL << 20) || (long long)N * S >= (1LL << 32) - 1) return SSHOPM_EUNSUPPORTED;
  const size_t rbytes = (size_t)N * (size_t)S * 16u * (size_t)dd_rec4(h->n);
  float4* rec = reinterpret_cast<float4*>(opts->d_records);
  bool own = false;
  if (rec) {
    if (opts->records_bytes < rbytes || ((uintptr_t)rec & 15)) return SSHOPM_EINVAL;
  } else {
    cudaError_t e = cudaMallocAsync(reinterpret_cast<void**>(&rec), rbytes, st);
    if (e == cudaErrorMemoryAllocation) return SSHOPM_ENOMEM;
    if (e != cudaSuccess) return cuda_fail(e, "records: cudaMallocAsync");
    own = true;
  }
  auto done = [&](int rc) {
    if (own) {
      cudaError_t e = cudaFreeAsync(rec, st);
      if (rc == SSHOPM_OK && e != cudaSuccess) rc = cuda_fail(e, "records: cudaFreeAsync");
    }
    return rc;
  };
  int bps = 0;
  cudaError_t e = L->occupancy_rec(shift, &bps);
  if (e != cudaSuccess) return done(cuda_fail(e, "sshopm_solve_dedup: occupancy"));
  if (bps < 1) bps = 1;
  if (opts->ctas_per_sm > 0 && opts->ctas_per_sm < bps) bps = opts->ctas_per_sm;
  long long grid = (long long)sms * bps;
  if (grid * 256 > n_units) grid = (n_units + 255) / 256;          // a lane per unit at most
  if (grid < 1) grid = 1;
  Workspace ws;
  int rc = acquire_workspace(L, N, S, opts->d_workspace, opts->workspace_bytes, st, &ws);
  if (rc != SSHOPM_OK) return done(rc);
  long long pgrid = ((N > S ? N : S) + 255) / 256;
  if (pgrid > (long long)sms * 8) pgrid = (long long)sms * 8;
  e = L->pack(N, d_entries, ws.packed, ws.counter, S, d_starts, ws.starts_n, alpha_mode,
              alpha_mode == 1 ? opts->d_alpha : nullptr, ws.alpha_t, (int)pgrid, st);
  if (e != cudaSuccess) { release_workspace(&ws, st); return done(cuda_fail(e, "sshopm_solve_dedup: pack launch")); }
  RecParams p;   // counter: word 0 of the workspace header, zeroed by the pack kernel
  p.packed = ws.packed;
  p.starts_n = reinterpret_cast<const float4*>(ws.starts_n);
  p.rec = rec;
  p.total_iters = opts->d_total_iters;
  p.counter = ws.counter;
  p.n_units = (uint32_t)n_units;
  p.units_per_tensor = (uint32_t)upt;
  p.unit = (uint32_t)unit;
  p.S = (uint32_t)S;
  p.div_upt = make_fastdiv((uint32_t)upt);
  p.alpha = alpha;
  p.tol = tol;
  p.alpha_t = ws.alpha_t;
  p.maxit = maxit;
  int k = opts->refill_threshold > 0 ? opts->refill_threshold : 4;
  p.refill_k = k < 1 ? 1 : (k > 32 ? 32 : k);
  e = L->solve_rec(p, shift, (int)grid, st);
  if (e != cudaSuccess) { release_workspace(&ws, st); return done(cuda_fail(e, "sshopm_solve_dedup: launch")); }
  h->launches.fetch_add(2);
  DedupParams q = *dd;
  q.rec = rec;
  rc = launch_dedup(h->m, h->n, q, st);
  if (rc == SSHOPM_OK) h->launches.fetch_add(1);
  int r2 = release_workspace(&ws, st);
  return done(rc != SSHOPM_OK ? rc : r2);
}

static int solve_impl(sshopm_t h, int64_t N, const float* d_entries, int S, const float* d_starts, float alpha,
                      float tol, int maxit, float* d_out_lambda, float* d_out_x, int32_t* d_out_iters,
                      uint8_t* d_out_converged, const sshopm_solve_opts* opts, const DedupParams* dd, cudaStream_t st) {
  if (!h || N < 0 || S < 1 || maxit < 0 || std::isnan(alpha) || std::isnan(tol)) return SSHOPM_EINVAL;
  if (N == 0) return SSHOPM_OK;
  if (opts && opts->fuse_dedup == 4) {                             // records path: no raw outputs
    if (!dd || !d_entries || !d_starts) return SSHOPM_EINVAL;
    if (!h->L || (opts->schedule != 0 && opts->schedule != 8)) return SSHOPM_EUNSUPPORTED;
    return solve_records(h, N, d_entries, S, d_starts, alpha, tol, maxit, opts, dd, st);
  }
  if (!d_entries || !d_starts || !d_out_lambda || !d_out_x || !d_out_iters || !d_out_converged) return SSHOPM_EINVAL;
  if (N > (1LL << 40) / S) return SSHOPM_EUNSUPPORTED;
  const Launchers* L = h->L;
  const int sms = device_sms();
  if (sms <= 0) return cuda_fail(cudaGetLastError(), "sshopm_solve: no device");
  if (opts && (opts->schedule < 0 || opts->schedule > 7)) return SSHOPM_EINVAL;
  if (!L || (opts && opts->schedule >= 3 && opts->schedule <= 5)) {   // table-driven general kernel (any (m, n))
    if (!h->gen) return SSHOPM_EUNSUPPORTED;
    int rc = general_solve(h->gen, N, d_entries, S, d_starts, alpha, tol, maxit, d_out_lambda, d_out_x, d_out_iters,
                           d_out_converged, opts, st);
    if (rc != SSHOPM_OK) return rc;
    h->launches.fetch_add(1);
    if (dd) {
      DedupParams q = *dd;
      q.lambda = d_out_lambda;
      q.x = d_out_x;
      q.conv = d_out_converged;
      rc = launch_dedup(h->m, h->n, q, st);
      if (rc == SSHOPM_OK) h->launches.fetch_add(1);
    }
    return rc;
  }

  // shift: scalar alpha (R4), or per tensor (alpha_mode 1: caller's array; 2 / 3: +- convexity bound, R17)
  const int alpha_mode = opts ? opts->alpha_mode : 0;
  if (alpha_mode < 0 || alpha_mode > 3) return SSHOPM_EINVAL;
  if (alpha_mode == 1 && !opts->d_alpha) return SSHOPM_EINVAL;
  const int shift = alpha_mode ? 3 : (alpha == 0.f ? 0 : (alpha > 0.f ? 1 : 2));
  const bool wide = (long long)N * S >= (1LL << 31) - (1LL << 20);
  // schedule: 1 = item per lane (two-chunk refill, default), 2 = tensor per lane, 6 = item per lane with the
  // lean predicated refill (C2: 4.33 vs 4.26 ms for schedule 1, profiles/r2/solve_variants.md)
  int schedule = (opts && opts->schedule > 0) ? opts->schedule : L->default_schedule;
  if (schedule != 1 && schedule != 2 && schedule != 6 && schedule != 7) return SSHOPM_EINVAL;   // 3-5: general
  if (shift == 3 && schedule == 2) schedule = 1;                 // per-tensor alpha: not on schedule 2
  // records-only request (opts->fuse_dedup = 2): the warp-tensor pipeline clusters in the solve kernel and
  // writes per-start outputs only for tensors it cannot cluster in registers (> 32 clusters)
  if (dd && opts && opts->fuse_dedup == 2) schedule = 7;
  int wt_mode = 0, wt_smem = 0;
  if (schedule == 7) {
    const int per_warp = L->wt_smem_per_warp(S);
    wt_mode = dd && opts && opts->fuse_dedup == 2 ? 1 : (dd && opts && opts->fuse_dedup == 1 ? 2 : 0);
    if (wt_mode && S != 128) wt_mode = 0;                        // in-kernel clustering: S = 128 register form
    wt_smem = 8 * per_warp;
    if (wt_smem > 200 * 1024) { schedule = 1; wt_mode = 0; }     // staging does not fit: schedule 1
  }
  int bps = 0;
  cudaError_t e = schedule == 7 ? L->occupancy(shift, false, 7, wt_mode, wt_smem, &bps)
                                : cached_occupancy(h, shift, wide, schedule, &bps);
  if (e != cudaSuccess) return cuda_fail(e, "sshopm_solve: occupancy");
  if (bps < 1) bps = 1;
  // fused dedup (opt-in, opts->fuse_dedup = 1): schedule 1, S <= 1024, and only if its shared memory
  // costs no occupancy.  Measured slower than the two-pass form on B200 at C2 (6.2 vs 5.4 ms): the
  // ring + in-kernel clustering push the register-capped solve into spills.
  int fused = 0;                                         // 0 none, 1 shared-memory dedup, 2 register dedup
  int smem = 0;
#ifndef SSHOPM_FUSED_REGS
#define SSHOPM_FUSED_REGS 1
#endif
  const bool fregs = SSHOPM_FUSED_REGS && dd && S == 128 && ((uintptr_t)d_out_lambda % 16 == 0) && ((uintptr_t)d_out_x % 16 == 0) &&
                     ((uintptr_t)d_out_converged % 4 == 0);
  if (dd && (schedule == 1 || schedule == 6) && S <= 1024 && opts && opts->fuse_dedup == 1) {
    const int fs = 8 * fused_smem_words(S, L->n, fregs) * 4;
    int fb = 0;
    if (fs <= 200 * 1024 && L->occupancy(shift, wide, 1, fregs ? 2 : 1, fs, &fb) == cudaSuccess && fb >= bps) {
      fused = fregs ? 2 : 1;
      smem = fs;
    }
  }
  // warp-specialised fused dedup (opts->fuse_dedup = 3): 7 solve warps + 1 dedup warp per CTA
  if (dd && (schedule == 1 || schedule == 6) && S <= 1024 && opts && opts->fuse_dedup == 3) {
    const int fs = ws_smem_words(S, L->n) * 4;
    int fb = 0;
    if (fs <= 200 * 1024 && L->occupancy(shift, wide, 1, 3, fs, &fb) == cudaSuccess && fb >= 1) {
      fused = 3;
      smem = fs;
      bps = fb;
    }
  }
  if (fused) schedule = 1;                                       // the fused ring lives in the schedule-1 kernel
  if (opts && opts->ctas_per_sm > 0 && opts->ctas_per_sm < bps) bps = opts->ctas_per_sm;
  if (opts && opts->chunk_tensors < 0) return SSHOPM_EINVAL;
  int chunk_tensors = chunk_tensors_for(S);                        // schedule 1: >= 256 items per chunk
  if (schedule == 6) {
    // lean schedule: chunks of up to 1024 items, at least 8 per resident warp
    const long long warps = (long long)sms * bps * 8;
    long long c = N / (warps * 8);
    const long long cmax = S >= 1024 ? 1 : 1024 / S;
    if (c > cmax) c = cmax;
    if (c < 1) c = 1;
    chunk_tensors = (int)c;
    if (opts && opts->chunk_tensors > 0) chunk_tensors = opts->chunk_tensors;
  }
  long long n_chunks = (N + chunk_tensors - 1) / chunk_tensors;
  if (n_chunks >= (1LL << 32) - (1LL << 20) || N >= (1LL << 32) - (1LL << 20)) return SSHOPM_EUNSUPPORTED;
  // schedule 1 claims chunks of items: whole tensors normally; for small problems (fewer chunks than
  // twice the resident warps) chunks of a part of a tensor, so every resident warp gets work (C1, the
  // paper's 1024 tensors: 512 two-tensor chunks would occupy 512 of 4736 warps)
  long long chunk_items = (long long)chunk_tensors * S;
  bool itemch = false;                                           // launches the FUSED_MODE 4 instance
  const int wpc = (schedule == 1 && !fused) ? L->solve_tpb / 32 : 8;   // warps per solve CTA
  if (schedule == 1 && !fused) {
    const long long warps = (long long)sms * bps * wpc;
    if (n_chunks < 2 * warps) {
      long long ci = ((long long)N * S + 2 * warps - 1) / (2 * warps);
      if (ci < 32) ci = 32;
      if (ci < chunk_items) {
        chunk_items = ci;
        n_chunks = ((long long)N * S + ci - 1) / ci;
        itemch = true;
      }
    }
  }
  long long grid = (long long)sms * bps;
  if (schedule == 7) {
    if (grid * 8 > N) grid = (N + 7) / 8;                          // warps claim whole tensors
  } else if (schedule != 2) {
    if (grid * wpc > n_chunks) grid = (n_chunks + wpc - 1) / wpc;
  } else {
    if (grid * 256 > N) grid = (N + 255) / 256;
  }
  if (grid < 1) grid = 1;

  Workspace ws;
  int rc = acquire_workspace(L, N, S, opts ? opts->d_workspace : nullptr, opts ? opts->workspace_bytes : 0, st, &ws);
  if (rc != SSHOPM_OK) return rc;
  long long pgrid = ((N > S ? N : S) + 255) / 256;
  if (pgrid > (long long)sms * 8) pgrid = (long long)sms * 8;
  e = L->pack(N, d_entries, ws.packed, ws.counter, S, d_starts, ws.starts_n, alpha_mode,
              alpha_mode == 1 ? opts->d_alpha : nullptr, ws.alpha_t, (int)pgrid, st);
  if (e != cudaSuccess) { release_workspace(&ws, st); return cuda_fail(e, "sshopm_solve: pack launch"); }

  SolveParams p;
  p.packed = ws.packed;
  p.starts_n = reinterpret_cast<const float4*>(ws.starts_n);
  p.out_lambda = d_out_lambda;
  p.out_x = d_out_x;
  p.out_iters = d_out_iters;
  p.out_conv = d_out_converged;
  p.total_iters = opts ? opts->d_total_iters : nullptr;
  p.counter = ws.counter;
  p.n_tensors = N;
  p.n_chunks = n_chunks;
  p.chunk_tensors = chunk_tensors;
  p.chunk_items = chunk_items;
  p.n_items = (long long)N * S;
  p.S = S;
  p.divS = make_fastdiv((uint32_t)S);
  p.s_log2 = -1;
  p.s_mask = (uint32_t)S - 1u;
  if ((S & (S - 1)) == 0)
    for (int b = 0; b < 31; ++b)
      if ((1 << b) == S) p.s_log2 = b;
  p.alpha = alpha;
  p.alpha_t = ws.alpha_t;
  p.tol = tol;
  p.maxit = maxit;
  int k = (opts && opts->refill_threshold > 0) ? opts->refill_threshold : L->default_refill;
  p.refill_k = k < 1 ? 1 : (k > 32 ? 32 : k);
  if (dd) p.dd = *dd;
  p.dd.lambda = d_out_lambda;
  p.dd.x = d_out_x;
  p.dd.conv = d_out_converged;
  p.ovf_count = ws.ovf_count;
  p.ovf_list = ws.ovf_list;
  p.fused_regs = fregs ? 1 : 0;
  if (schedule == 7) { fused = wt_mode; smem = wt_smem; }
  e = L->solve(p, shift, schedule == 7 ? false : wide, schedule, itemch ? 4 : fused, (int)grid, smem, st);
  if (e != cudaSuccess) { release_workspace(&ws, st); return cuda_fail(e, "sshopm_solve: launch"); }
  h->launches.fetch_add(2);
  if (dd) {
    if (schedule == 7 && wt_mode) rc = launch_dedup_list(h->m, h->n, p.dd, ws.ovf_count, ws.ovf_list, 1, st);
    else if (fused) rc = launch_dedup_list(h->m, h->n, p.dd, ws.ovf_count, ws.ovf_list, chunk_tensors, st);
    else rc = launch_dedup(h->m, h->n, p.dd, st);
    if (rc != SSHOPM_OK) { release_workspace(&ws, st); return rc; }
    h->launches.fetch_add(1);
  }
  return release_workspace(&ws, st);
}
}  // namespace sshopm

extern "C" {

int sshopm_solve_ex(sshopm_t h, int64_t N, const float* d_entries, int S, const float* d_starts,
                    float alpha, float tol, int maxit,
                    float* d_out_lambda, float* d_out_x, int32_t* d_out_iters, uint8_t* d_out_converged,
                    const sshopm_solve_opts* opts, void* stream) {
  return solve_impl(h, N, d_entries, S, d_starts, alpha, tol, maxit, d_out_lambda, d_out_x, d_out_iters,
                    d_out_converged, opts, nullptr, (cudaStream_t)stream);
}

int sshopm_solve_dedup(sshopm_t h, int64_t N, const float* d_entries, int S, const float* d_starts,
                       float alpha, float tol, int maxit,
                       float* d_out_lambda, float* d_out_x, int32_t* d_out_iters, uint8_t* d_out_converged,
                       float lam_tol, float ang_tol, int kmax,
                       int32_t* d_out_count, float* d_out_clambda, float* d_out_cx, int32_t* d_out_mult,
                       int32_t* d_out_rep, const sshopm_solve_opts* opts, void* stream) {
  if (!h) return SSHOPM_EINVAL;
  DedupParams dd;
  int rc = make_dedup_params(h->n, N, S, lam_tol, ang_tol, kmax, d_out_count, d_out_clambda, d_out_cx, d_out_mult,
                             d_out_rep, &dd);
  if (rc != SSHOPM_OK) return rc;
  return solve_impl(h, N, d_entries, S, d_starts, alpha, tol, maxit, d_out_lambda, d_out_x, d_out_iters,
                    d_out_converged, opts, N > 0 ? &dd : nullptr, (cudaStream_t)stream);
}

int sshopm_solve(sshopm_t h, int64_t N, const float* d_entries, int S, const float* d_starts,
                 float alpha, float tol, int maxit,
                 float* d_out_lambda, float* d_out_x, int32_t* d_out_iters, uint8_t* d_out_converged,
                 void* stream) {
  return sshopm_solve_ex(h, N, d_entries, S, d_starts, alpha, tol, maxit, d_out_lambda, d_out_x, d_out_iters,
                         d_out_converged, nullptr, stream);
}

int sshopm_classify(sshopm_t h, int64_t N, const float* d_entries, int kmax, const int32_t* d_count,
                    const float* d_lambda, const float* d_x, float ctol, int8_t* d_out_type, void* stream) {
  if (!h || N < 0 || kmax < 1 || !(ctol >= 0.f)) return SSHOPM_EINVAL;
  if (N == 0) return SSHOPM_OK;
  if (!d_entries || !d_count || !d_lambda || !d_x || !d_out_type) return SSHOPM_EINVAL;
  if (!h->L) return SSHOPM_EUNSUPPORTED;                          // compiled shapes only
  const int sms = device_sms();
  if (sms <= 0) return cuda_fail(cudaGetLastError(), "sshopm_classify: no device");
  long long grid = (N * kmax + 127) / 128;
  if (grid > (long long)sms * 32) grid = (long long)sms * 32;
  cudaError_t e = h->L->classify(N, kmax, d_entries, d_count, d_lambda, d_x, ctol, d_out_type, (int)grid,
                                 (cudaStream_t)stream);
  if (e != cudaSuccess) return cuda_fail(e, "sshopm_classify: launch");
  h->launches.fetch_add(1);
  return SSHOPM_OK;
}

int sshopm_apply(sshopm_t h, int64_t N, const float* d_entries, const float* d_x,
                 float* d_out_g, float* d_out_lam, void* stream) {
  if (!h || N < 0) return SSHOPM_EINVAL;
  if (N == 0) return SSHOPM_OK;
  if (!d_entries || !d_x || !d_out_g || !d_out_lam) return SSHOPM_EINVAL;
  cudaStream_t st = (cudaStream_t)stream;
  const int sms = device_sms();
  if (sms <= 0) return cuda_fail(cudaGetLastError(), "sshopm_apply: no device");
  if (!h->L) {
    int rc = general_apply(h->gen, N, d_entries, d_x, d_out_g, d_out_lam, st);
    if (rc == SSHOPM_OK) h->launches.fetch_add(1);
    return rc;
  }
  long long grid = (N + 255) / 256;
  if (grid > (long long)sms * 16) grid = (long long)sms * 16;
  Workspace ws;
  int rc = acquire_workspace(h->L, N, 0, nullptr, 0, st, &ws);
  if (rc != SSHOPM_OK) return rc;
  cudaError_t e = h->L->pack(N, d_entries, ws.packed, nullptr, 0, nullptr, nullptr, 0, nullptr, nullptr, (int)grid, st);
  if (e == cudaSuccess) e = h->L->apply(N, ws.packed, d_x, d_out_g, d_out_lam, (int)grid, st);
  if (e != cudaSuccess) { release_workspace(&ws, st); return cuda_fail(e, "sshopm_apply: launch"); }
  h->launches.fetch_add(2);
  return release_workspace(&ws, st);
}

}  // extern "C"

namespace sshopm {
template <int NN, bool EVEN, bool REC>
static cudaError_t launch_dedup_t2(const DedupParams& p, int grid, int block, int smem, cudaStream_t st) {
  if (smem > 48 * 1024) {
    cudaError_t e = cudaFuncSetAttribute(sshopm_dedup_kernel<NN, EVEN, REC>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e != cudaSuccess) return e;
  }
  sshopm_dedup_kernel<NN, EVEN, REC><<<grid, block, smem, st>>>(p);
  return cudaGetLastError();
}
template <int NN, bool EVEN>
static cudaError_t launch_dedup_t(const DedupParams& p, int grid, int block, int smem, cudaStream_t st) {
  return p.rec ? launch_dedup_t2<NN, EVEN, true>(p, grid, block, smem, st)
               : launch_dedup_t2<NN, EVEN, false>(p, grid, block, smem, st);
}

template <int NN, bool EVEN, bool REC>
static cudaError_t launch_dedup128_2(const DedupParams& p, int grid, int block, int smem, cudaStream_t st) {
  if (smem > 48 * 1024) {
    cudaError_t e = cudaFuncSetAttribute(sshopm_dedup128_kernel<NN, EVEN, REC>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e != cudaSuccess) return e;
  }
  sshopm_dedup128_kernel<NN, EVEN, REC><<<grid, block, smem, st>>>(p);
  return cudaGetLastError();
}
template <int NN, bool EVEN>
static cudaError_t launch_dedup128(const DedupParams& p, int grid, int block, int smem, cudaStream_t st) {
  return p.rec ? launch_dedup128_2<NN, EVEN, true>(p, grid, block, smem, st)
               : launch_dedup128_2<NN, EVEN, false>(p, grid, block, smem, st);
}

int make_dedup_params(int n, int64_t N, int S, float lam_tol, float ang_tol, int kmax, int32_t* d_count,
                      float* d_olam, float* d_ox, int32_t* d_mult, int32_t* d_rep, DedupParams* p) {
  if (S < 1 || kmax < 1 || !(lam_tol >= 0.f) || !(ang_tol >= 0.f) || N < 0) return SSHOPM_EINVAL;
  if (N > 0 && (!d_count || !d_olam || !d_ox || !d_mult)) return SSHOPM_EINVAL;
  if (S > 1024) return SSHOPM_EUNSUPPORTED;
  if (n > 16) return SSHOPM_EUNSUPPORTED;                    // the blocked kernel's largest n
  p->lambda = nullptr;
  p->x = nullptr;
  p->conv = nullptr;
  p->rec = nullptr;
  p->out_count = d_count;
  p->out_lambda = d_olam;
  p->out_x = d_ox;
  p->out_mult = d_mult;
  p->out_rep = d_rep;
  p->n_tensors = N;
  p->S = S;
  p->kmax = kmax;
  p->lam_tol = lam_tol;
  p->cos_tol = ang_tol >= 3.14159265358979f ? -1.0f : cosf(ang_tol);
  return SSHOPM_OK;
}

static int dedup_launch_shape(int n, int64_t N, int S, bool fast, int* grid, int* block, int* smem) {
  const int sms = device_sms();
  if (sms <= 0) return cuda_fail(cudaGetLastError(), "sshopm_dedup: no device");
  const int per_warp = fast ? dedup128_smem_per_warp(n) : dedup_smem_words(S, n) * 4;
  int wpb = (96 * 1024) / per_warp;
  static const int wmax = [] { const char* v = getenv("SSHOPM_DEDUP_WARPS"); int w = v ? atoi(v) : 8;
                               return w < 1 ? 1 : (w > 8 ? 8 : w); }();   // warps per dedup CTA (default 8)
  if (wpb > wmax) wpb = wmax;
  if (wpb < 1) wpb = 1;
  *smem = wpb * per_warp;
  *block = 32 * wpb;
  long long g = (N + wpb - 1) / wpb;
  if (g > (long long)sms * 16) g = (long long)sms * 16;
  if (g < 1) g = 1;
  *grid = (int)g;
  return SSHOPM_OK;
}

int launch_dedup(int m, int n, const DedupParams& p, cudaStream_t st) {
  if (p.n_tensors == 0) return SSHOPM_OK;
  if (!p.rec && (!p.lambda || !p.x || !p.conv)) return SSHOPM_EINVAL;
  const int S = p.S;
  const bool fast = (S == 128) && n <= 8 &&
                    (p.rec ? ((uintptr_t)p.rec % 16 == 0)
                           : (((uintptr_t)p.lambda % 16 == 0) && ((uintptr_t)p.x % 16 == 0) && ((uintptr_t)p.conv % 4 == 0)));
  int grid, block, smem;
  int rc = dedup_launch_shape(n, p.n_tensors, S, fast, &grid, &block, &smem);
  if (rc != SSHOPM_OK) return rc;
  const bool even = (m % 2) == 0;
  cudaError_t e = cudaErrorInvalidValue;
  switch (n) {
#define DD(NN) case NN: e = fast ? (even ? launch_dedup128<NN, true>(p, grid, block, smem, st) : launch_dedup128<NN, false>(p, grid, block, smem, st)) \
                             : (even ? launch_dedup_t<NN, true>(p, grid, block, smem, st) : launch_dedup_t<NN, false>(p, grid, block, smem, st)); break;
    DD(1) DD(2) DD(3) DD(4) DD(5) DD(6) DD(7) DD(8)
#undef DD
#define DG(NN) case NN: e = even ? launch_dedup_t<NN, true>(p, grid, block, smem, st) \
                             : launch_dedup_t<NN, false>(p, grid, block, smem, st); break;
    DG(9) DG(10) DG(11) DG(12) DG(13) DG(14) DG(15) DG(16)
#undef DG
    default: return SSHOPM_EUNSUPPORTED;
  }
  if (e != cudaSuccess) return cuda_fail(e, "sshopm_dedup: launch");
  return SSHOPM_OK;
}

template <int NN, bool EVEN>
static cudaError_t launch_list_t(const DedupParams& p, const unsigned int* count, const unsigned int* list, int ct,
                                 int grid, int block, int smem, cudaStream_t st) {
  if (smem > 48 * 1024) {
    cudaError_t e = cudaFuncSetAttribute(sshopm_dedup_list_kernel<NN, EVEN>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e != cudaSuccess) return e;
  }
  sshopm_dedup_list_kernel<NN, EVEN><<<grid, block, smem, st>>>(p, count, list, ct);
  return cudaGetLastError();
}

int launch_dedup_list(int m, int n, const DedupParams& p, const unsigned int* count, const unsigned int* list,
                      int chunk_tensors, cudaStream_t st) {
  int grid, block, smem;
  int rc = dedup_launch_shape(n, p.n_tensors, p.S, false, &grid, &block, &smem);
  if (rc != SSHOPM_OK) return rc;
  const int sms = device_sms();
  if (grid > sms * 2) grid = sms * 2;                     // untracked chunks are rare
  const bool even = (m % 2) == 0;
  cudaError_t e = cudaErrorInvalidValue;
  switch (n) {
#define DD(NN) case NN: e = even ? launch_list_t<NN, true>(p, count, list, chunk_tensors, grid, block, smem, st) \
                             : launch_list_t<NN, false>(p, count, list, chunk_tensors, grid, block, smem, st); break;
    DD(1) DD(2) DD(3) DD(4) DD(5) DD(6) DD(7) DD(8) DD(9) DD(10) DD(11) DD(12) DD(13) DD(14) DD(15) DD(16)
#undef DD
    default: return SSHOPM_EUNSUPPORTED;
  }
  if (e != cudaSuccess) return cuda_fail(e, "sshopm_dedup_list: launch");
  return SSHOPM_OK;
}

int dedup_impl(int m, int n, int64_t N, int S, const float* d_lambda, const float* d_x, const uint8_t* d_conv,
               float lam_tol, float ang_tol, int kmax, int32_t* d_count, float* d_olam, float* d_ox, int32_t* d_mult,
               int32_t* d_rep, cudaStream_t st) {
  DedupParams p;
  int rc = make_dedup_params(n, N, S, lam_tol, ang_tol, kmax, d_count, d_olam, d_ox, d_mult, d_rep, &p);
  if (rc != SSHOPM_OK) return rc;
  if (N == 0) return SSHOPM_OK;
  if (!d_lambda || !d_x || !d_conv) return SSHOPM_EINVAL;
  p.lambda = d_lambda;
  p.x = d_x;
  p.conv = d_conv;
  return launch_dedup(m, n, p, st);
}
}  // namespace sshopm

extern "C" int sshopm_dedup(sshopm_t h, int64_t N, int S,
                            const float* d_lambda, const float* d_x, const uint8_t* d_converged,
                            float lam_tol, float ang_tol, int kmax,
                            int32_t* d_out_count, float* d_out_lambda, float* d_out_x, int32_t* d_out_mult,
                            int32_t* d_out_rep, void* stream) {
  if (!h) return SSHOPM_EINVAL;
  int r = dedup_impl(h->m, h->n, N, S, d_lambda, d_x, d_converged, lam_tol, ang_tol, kmax, d_out_count, d_out_lambda,
                     d_out_x, d_out_mult, d_out_rep, (cudaStream_t)stream);
  if (r == SSHOPM_OK && N > 0) h->launches.fetch_add(1);
  return r;
}
