/*
 * sshopm.h — C ABI of libsshopm.so: batched SS-HOPM (shifted symmetric
 * higher-order power method) over many small symmetric tensors on B200.
 *
 * Paper: Ballard, Kolda, Plantenga, "Efficiently Computing Tensor Eigenvalues
 * on a GPU", IPDPS-W 2011.  Citations "P:L<n>" are lines of that paper's text
 * (reference/PAPER.md); "R<k>" are the readings listed in DESIGN.md.
 *
 * Conventions shared by every entry point
 * ---------------------------------------
 * - Every call returns an int status (SSHOPM_OK = 0 or an error code below)
 *   and never aborts the process.  Argument checks are synchronous.
 * - Pointers named d_* are DEVICE pointers owned by the caller; pointers named
 *   h_* are HOST pointers owned by the caller.  The library never frees or
 *   retains caller memory beyond the call (asynchronous kernels read/write it
 *   until the stream reaches that point).
 * - Floating point data are IEEE float32, integer data int32 / uint8, all
 *   row-major and contiguous, no padding.
 * - Device work is enqueued asynchronously on `stream` (a cudaStream_t passed
 *   as void*; NULL = legacy default stream).  Launch errors are returned as
 *   SSHOPM_ECUDA; errors raised while kernels run surface at the caller's
 *   next synchronisation (documented CUDA behaviour).
 * - A handle is immutable after sshopm_create, so concurrent calls on
 *   different streams are safe.  N = 0 is a no-op returning SSHOPM_OK.
 *
 * Storage format of one tensor (Table I)
 * ---------------------------------------------------------------------
 * A symmetric A in R^[m,n] (Definition 1) is stored as its
 * U = C(m+n-1, m) unique values (Property 1), one per index class,
 * classes in the paper's lexicographic order of index representations
 * (nondecreasing tensor indices).  entries[t][c] = a_{i_1..i_m} for
 * class c of tensor t (reading R8: entry values, not polynomial coefficients).
 */
#ifndef SSHOPM_H
#define SSHOPM_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct sshopm_ctx* sshopm_t;

enum {
  SSHOPM_OK = 0,
  SSHOPM_EINVAL = 1,       /* bad argument (null pointer with N > 0, m < 2, n < 1, S < 1, maxit < 0, NaN alpha/tol, ...) */
  SSHOPM_EUNSUPPORTED = 2, /* (m, n) or S outside what this build was compiled for */
  SSHOPM_ECUDA = 3,        /* CUDA runtime error at launch / copy (see sshopm_last_cuda_error) */
  SSHOPM_ENOMEM = 4        /* host or device allocation failed */
};

/* Create a solver for tensors of order m and dimension n.
 * Enumerates the index classes and coefficients (Sec. III) and selects the
 * kernel specialised for (m, n) at compile time (Sec. V-D loop unrolling,
 * P:L327-331).  Holds host state only; allocates no device memory.
 * Errors: EINVAL (m < 2, n < 1, out == NULL), EUNSUPPORTED ((m, n) not built). */
int sshopm_create(int m, int n, sshopm_t* out);

/* Destroy a handle.  NULL is accepted (no-op). */
int sshopm_destroy(sshopm_t h);

/* U = C(m+n-1, m), the number of unique entries per tensor (Property 1). */
int sshopm_num_unique(sshopm_t h, int* U);

/* Write the U index representations, 0-based, lexicographic order,
 * into host array h_idx[U][m].  For tests and documentation. */
int sshopm_class_index(sshopm_t h, int32_t* h_idx);

/* Flop counts per SS-HOPM iteration of one (tensor, start) lane:
 *   *paper    = (m+2) U + (m+1) T1 + 5 n   (reading R12 of the paper's counting,
 *               Eq. 4 + Eq. 6 + shift/normalise; T1 = n C(m+n-2, m-1); parity unpinned)
 *   *executed = FP32 flops of this library's evaluation (FMA = 2 flops) —
 *               the algorithmic count used for the ALU roofline.
 * Either pointer may be NULL. */
int sshopm_flops_per_iter(sshopm_t h, int64_t* paper, int64_t* executed);

/* Batched SS-HOPM (Fig. 1; problem statement P:L305-307).
 * For every tensor t < N and start s < S, runs SS-HOPM from x_0 = starts[s] /
 * ||starts[s]|| (normalised on the device in FP32, reading R7):
 *     lam_0 = A x_0^m; repeat  xhat = +-(A x_k^{m-1} + alpha x_k)  ("+" iff alpha >= 0, R5),
 *                              x_{k+1} = xhat / ||xhat||, lam_{k+1} = A x_{k+1}^m
 *     until |lam_{k+1} - lam_k| <= tol * max(1, |lam_{k+1}|) (converged, R2) or maxit updates.
 * Outputs for lane (t, s) at index t*S + s:
 *     d_out_lambda[N][S]   lam at the stopping update
 *     d_out_x[N][S][n]     x at the stopping update (unit norm)
 *     d_out_iters[N][S]    number of x-updates performed (Fig. 1 loop trips)
 *     d_out_converged[N][S] 1 if the tolerance test fired, else 0
 * Special cases: tol < 0 -> fixed-K mode (exactly maxit updates, converged = 0);
 * maxit = 0 -> (lam_0, x_0), iters 0; a zero start or ||xhat|| = 0 stops the
 * lane with converged = 0 and the last (lam, x) (R6).
 * Inputs: d_entries[N][U], d_starts[S][n] (shared by all tensors).
 * Errors: EINVAL (null pointers with N > 0, S < 1, maxit < 0, NaN alpha or tol),
 *         ECUDA. */
int sshopm_solve(sshopm_t h, int64_t N, const float* d_entries, int S, const float* d_starts,
                 float alpha, float tol, int maxit,
                 float* d_out_lambda, float* d_out_x, int32_t* d_out_iters, uint8_t* d_out_converged,
                 void* stream);

/* Device workspace needed by sshopm_solve_ex for N tensors and S starts
 * (bytes): a 256-byte header (work counter), the S normalised starts and one
 * 16-byte aligned packed coefficient row per tensor (precomputed
 * coefficients).  sshopm_solve and sshopm_apply allocate it
 * themselves (cudaMallocAsync / cudaFreeAsync on the stream). */
int sshopm_workspace_size(sshopm_t h, int64_t N, int S, size_t* bytes);

/* Scratch bytes of the records path (fuse_dedup = 4): N * S * 16 * ceil((n + 1) / 4). */
int sshopm_records_size(sshopm_t h, int64_t N, int S, size_t* bytes);

/* Tuning / instrumentation knobs for sshopm_solve_ex (0 / NULL = library default).  Zero-initialise the
 * whole struct (memset) and set only the fields you need: fields are appended as the library grows
 * (d_records, records_bytes and unit_starts were added in round 2), so a caller must be compiled against
 * this header. */
typedef struct {
  int refill_threshold;            /* lanes that must be idle before a warp refills (1..32); default per (m, n) */
  int ctas_per_sm;                 /* persistent CTAs per SM; default = max occupancy */
  unsigned long long* d_total_iters; /* optional device counter: += sum of iters over all lanes (atomicAdd) */
  void* d_workspace;               /* optional caller-owned device workspace, 256-byte aligned, >= sshopm_workspace_size */
  size_t workspace_bytes;          /* its size; a too-small or misaligned workspace returns EINVAL */
  int schedule;                    /* 0 default, 1 = item per lane (warps claim chunks of whole tensors),
                                      2 = tensor per lane (a lane walks one tensor's starts), 6 = item per lane
                                      with a branch-free predicated refill and one chunk in flight, 7 = warp-
                                      tensor pipeline (shared-memory staging, coalesced flushes); 6 and 7 are
                                      measured slower on B200 and kept for comparison; results identical.
                                      Table-driven general kernel (the only path for (m, n) without a compiled
                                      kernel): 5 = blocked (default): warp per tensor, the
                                      tensor's coefficient-folded rows once per warp in shared memory, blocks of
                                      Eq. 6 per degree-(m-2) prefix ("blocked approach"); 3 = item per
                                      lane, the tensor row per lane in shared memory; 4 = block per tensor,
                                      thread per start (the paper's mapping); 3-5 also force the
                                      table-driven path on compiled shapes (5 returns EUNSUPPORTED if its
                                      shared memory does not fit; the default then falls back to 3, then 4). */
  int fuse_dedup;                  /* sshopm_solve_dedup only: 0 = default (two passes),
                                      1 = solve warps cluster their chunks, 3 = one dedup warp per CTA,
                                      2 = records only (schedule 7 pipeline), 4 = records path (schedule 8):
                                      lanes own units of consecutive starts of one tensor (no coefficient
                                      reload per item), each start leaves one 16-byte (lambda | NaN, x)
                                      record in scratch that the dedup reads; the raw per-start outputs are
                                      not written (their pointers may be NULL) and out_iters is not
                                      produced (d_total_iters still counts).  Dedup outputs identical in
                                      every mode. */
  int alpha_mode;                  /* shift: 0 = the scalar alpha argument (default);
                                      1 = per tensor, d_alpha[N] (device); 2 = per tensor automatic convex shift
                                      alpha_t = +(m-1) sum_{all indices} |a| (>= beta(A): lambda_k nondecreasing,
                                      converges to local maxima, Kolda-Mayo [1]); 3 = automatic concave shift -(...)
                                      (minima).  Modes 1-3 use schedule 1. */
  const float* d_alpha;            /* alpha_mode 1: per-tensor shifts [N] */
  int chunk_tensors;               /* schedule 6: tensors per work chunk a warp claims (0 = default:
                                      up to 1024 items, at least 8 chunks per resident warp) */
  void* d_records;                 /* fuse_dedup = 4: optional caller-owned scratch for the per-start records,
                                      16-byte aligned, >= sshopm_records_size bytes (else allocated on the stream) */
  size_t records_bytes;            /* its size */
  int unit_starts;                 /* fuse_dedup = 4: starts per work unit a lane claims (0 = default 32) */
} sshopm_solve_opts;

/* sshopm_solve with options (opts may be NULL).  Launches two kernels on
 * `stream`: the pack kernel (coefficient rows) and the solve kernel. */
int sshopm_solve_ex(sshopm_t h, int64_t N, const float* d_entries, int S, const float* d_starts,
                    float alpha, float tol, int maxit,
                    float* d_out_lambda, float* d_out_x, int32_t* d_out_iters, uint8_t* d_out_converged,
                    const sshopm_solve_opts* opts, void* stream);

/* Per-tensor eigenpair dedup (reading R16).
 * For each tensor t: visit converged starts in start order; a start joins the
 * first existing cluster whose representative r has
 *     |lam_s - lam_r| <= lam_tol * max(1, |lam_r|)  and  angle(x_s, x_r) <= ang_tol
 * (sign-free for even m, R15; for odd m (lam, x) ~ (-lam, -x)), else it
 * founds a new cluster.  Clusters are ordered by representative lam
 * descending, ties by representative start ascending.
 * Outputs: d_out_count[N] total clusters (may exceed kmax), and for the first
 * kmax clusters d_out_lambda[N][kmax], d_out_x[N][kmax][n], d_out_mult[N][kmax]
 * (members), d_out_rep[N][kmax] (representative start, -1 in empty slots;
 * d_out_rep may be NULL).  Empty slots: lambda 0, x 0, mult 0.
 * Inputs are sshopm_solve's outputs.  Errors: EINVAL (kmax < 1, negative
 * tolerances, null pointers), EUNSUPPORTED (S > 1024 or n > 16), ECUDA. */
int sshopm_dedup(sshopm_t h, int64_t N, int S,
                 const float* d_lambda, const float* d_x, const uint8_t* d_converged,
                 float lam_tol, float ang_tol, int kmax,
                 int32_t* d_out_count, float* d_out_lambda, float* d_out_x, int32_t* d_out_mult,
                 int32_t* d_out_rep, void* stream);

/* Solve + dedup in one pass (the whole per-tensor hot path, DESIGN.md "Fused
 * dedup"): same arguments and outputs as sshopm_solve_ex followed by
 * sshopm_dedup with the same tolerances, and bitwise the same results.  Each
 * warp of the solve kernel clusters a chunk of tensors as soon as it has
 * written the chunk's last start (reading the raw outputs back from L2); the
 * few chunks it cannot track are clustered by a small follow-up kernel.
 * Raw outputs are required (they are also the dedup's input).  The fused forms
 * are opt-in: opts->fuse_dedup = 1, the solve warps cluster their own chunks;
 * 3, one warp per CTA clusters the chunks the other seven complete (a CTA
 * queue in shared memory); 2, records only: the warp-tensor pipeline
 * (schedule 7) clusters each tensor from its shared-memory staging and writes
 * raw outputs only for tensors with more than 32 clusters (S = 128; the raw
 * output arrays are then scratch).  All are measured slower than the two
 * passes on B200.  By default, and whenever a fused
 * form does not apply, the two passes run back to back on the stream.
 * Errors: as sshopm_solve_ex and sshopm_dedup. */
int sshopm_solve_dedup(sshopm_t h, int64_t N, const float* d_entries, int S, const float* d_starts,
                       float alpha, float tol, int maxit,
                       float* d_out_lambda, float* d_out_x, int32_t* d_out_iters, uint8_t* d_out_converged,
                       float lam_tol, float ang_tol, int kmax,
                       int32_t* d_out_count, float* d_out_clambda, float* d_out_cx, int32_t* d_out_mult,
                       int32_t* d_out_rep, const sshopm_solve_opts* opts, void* stream);

/* Eigenpair type of each dedup record (reading R18; fibre directions are the
 * local maxima of A g^m on the sphere).  For record
 * k of tensor t (k < count[t]) with (lam, x) = (d_lambda[t][k], d_x[t][k]):
 * C = U^T [(m-1) A x^{m-2} - lam I] U on x-perp (Definition 2 with p = 2);
 * d_out_type[t][k] = +1 local maximum (C negative definite), -1 local minimum,
 * 0 saddle, 2 degenerate (an eigenvalue of C within ctol * max(1, |lam|) of 0),
 * 3 empty slot (k >= count[t]).  Inputs are sshopm_dedup's outputs and the
 * tensors' entries.  Compiled (m, n) only (else EUNSUPPORTED). */
int sshopm_classify(sshopm_t h, int64_t N, const float* d_entries, int kmax, const int32_t* d_count,
                    const float* d_lambda, const float* d_x, float ctol, int8_t* d_out_type, void* stream);

/* Test hook: d_out_g[N][n] = A x^{m-1} (Eq. 6) and d_out_lam[N] = A x^m
 * (Eq. 4 via Euler's identity x.(A x^{m-1})) for N (tensor, x) pairs, using
 * exactly the solver's compiled evaluation.  d_x[N][n] is NOT normalised. */
int sshopm_apply(sshopm_t h, int64_t N, const float* d_entries, const float* d_x,
                 float* d_out_g, float* d_out_lam, void* stream);

/* End-to-end call on HOST buffers: copies h_entries to the device in chunks,
 * runs solve + dedup on each chunk, and copies the dedup records back, with
 * copies and compute overlapped on internal streams.  Raw per-start outputs
 * are returned only if the h_out_* raw pointers are non-NULL.  Blocks until
 * done.  Host buffers should be pinned (cudaHostAlloc / registered) for full
 * bandwidth.  Device memory is allocated and freed inside the call.
 * Errors: as sshopm_solve and sshopm_dedup, plus ENOMEM. */
int sshopm_run_host(sshopm_t h, int64_t N, const float* h_entries, int S, const float* h_starts,
                    float alpha, float tol, int maxit,
                    float lam_tol, float ang_tol, int kmax,
                    int32_t* h_out_count, float* h_out_lambda, float* h_out_x, int32_t* h_out_mult,
                    int32_t* h_out_rep,
                    float* h_raw_lambda, float* h_raw_x, int32_t* h_raw_iters, uint8_t* h_raw_converged,
                    int64_t chunk_tensors, unsigned long long* h_total_iters);

/* Number of kernels this handle has launched since creation (instrumentation). */
int sshopm_launch_count(sshopm_t h, int64_t* count);

/* Human-readable status string; also the text of the last CUDA error. */
const char* sshopm_status_string(int code);
const char* sshopm_last_cuda_error(void);

/* Peer memory for the multi-GPU record gather.  Rank 0 allocates
 * the gather buffer here and exports it; every other rank maps it and passes pointers into it as
 * sshopm_dedup's outputs, so the dedup kernel's record stores travel over NVLink straight into rank 0's
 * memory: the gather is fused into the kernel that produces the records (no separate collective).
 *   sshopm_ipc_alloc: cudaMalloc of `bytes` on the current device (the one allocation this library
 *     hands out; free it with sshopm_ipc_free); *d_ptr receives it and h_handle (host, caller-owned,
 *     SSHOPM_IPC_HANDLE_BYTES) the opaque handle other processes of this node pass to sshopm_ipc_import.
 *   sshopm_ipc_import: maps such a handle into this process (peer access enabled lazily); *d_ptr is
 *     the buffer's device address here.  Map once, reuse; sshopm_ipc_release unmaps it.
 * Errors: EINVAL (null arguments, bytes == 0), ENOMEM, ECUDA (the runtime refused: e.g. no P2P path). */
#define SSHOPM_IPC_HANDLE_BYTES 64
int sshopm_ipc_alloc(size_t bytes, void** d_ptr, void* h_handle);
int sshopm_ipc_free(void* d_ptr);
int sshopm_ipc_import(const void* h_handle, void** d_ptr);
int sshopm_ipc_release(void* d_ptr);

/* Comma-separated list of (m,n) pairs compiled into this build, e.g. "2x3,4x3". */
const char* sshopm_supported_shapes(void);

#ifdef __cplusplus
}
#endif
#endif /* SSHOPM_H */
