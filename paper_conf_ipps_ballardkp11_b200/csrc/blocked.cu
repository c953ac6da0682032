// blocked.cu — warp-per-tensor blocked SS-HOPM for larger (m, n).
//
// The paper unrolls (4,3) fully into registers and notes that "to scale to
// larger problems we need a blocked approach" (Sec. V-D; future work,
// "register blocking ... classify the various shapes of register
// blocks").  Here the blocks are those of Eq. 6 regrouped by monomial
// (DESIGN.md "Evaluation"):
//
//   (A x^{m-1})_j = sum_{|p| = m-2} x^p sum_{i >= last(p)} x_i B[p + e_i][j],
//   B[q][j] = ((m-1)!/q!) a_{class(q + e_j)},
//
// i.e. for every degree-(m-2) prefix p (in lexicographic order) one block of
// rows q = p + e_i, i = last(p) .. n-1, which are consecutive in the
// lexicographic order of q.  Mapping on sm_100a:
//   * a warp owns one tensor at a time; its B-form rows (Q x round4(n) words,
//     coefficient-folded when the tensor is staged) live ONCE in the warp's
//     shared memory and are read by all 32 lanes as broadcast LDS.128 — the
//     general item-per-lane kernel keeps 32 private copies instead, which
//     limits it to a few warps per SM once U grows;
//   * lanes are starts of the warp's tensor (refilled in batches from the
//     tensor's start counter, as in the unrolled kernel); two B buffers per
//     warp let idle lanes begin the next tensor while stragglers finish the
//     previous one (no per-tensor tail);
//   * the dimension n is a template parameter, so x, g and the inner i / j
//     loops of a block are registers and unrolled code; the prefix monomials
//     x^p (degree m-2, any m) are x^{p - e_l} x_l with x_l a register (l is
//     compile-time in the grouped loop), so only degrees 1..m-3 are built per
//     step, in lane-interleaved shared memory (bank-conflict free).
// Stopping rule, shift, degenerate cases and outputs are those of every other
// kernel (readings R1-R7); results match the oracle under the same contract.
#include <cstdio>
#include <cstring>

#include "api_internal.h"
#include "general.h"
#include "sshopm.h"

namespace sshopm {

struct BlkParams {
  const float* entries;      // [N][U]
  const float* starts;       // [S][n] raw
  const uint32_t* recipe;    // [L] parent | var << 16 (degree >= 2; degree-1 entries unused)
  const float* coef;         // [Q] (m-1)!/q!
  const uint32_t* cls;       // [Q][n] class(q + e_j)
  const int* cls_mult;       // [U] m!/k! (automatic shift)
  const uint32_t* pidx;      // [P] per degree-(m-2) prefix p (grouped by last index l, stable): the
                             //     index of p - e_l among the stored monomials (m >= 4)
  const uint32_t* gcnt;      // [n] prefixes per last index
  const uint32_t* qperm;     // [Q] B-row order (per grouped prefix p: q = p + e_i, i = last(p)..n-1)
  float* out_lambda;
  float* out_x;
  int32_t* out_iters;
  uint8_t* out_conv;
  unsigned long long* total_iters;
  const float* alpha_in;     // alpha_mode 1
  unsigned int* counter;     // tensor counter (zeroed by the host)
  long long N;
  int m, U, S, L, Q, P;
  int low;                   // monomials of degree 1..m-2 in the recipe (L - Q)
  int mono_words;            // per-lane shared words: degrees 1..m-3 (mono[0..n) = x), at least n
  int buf_words;             // words of one B buffer (Q * round4(n), + 4 for the buffer's shift)
  float alpha, tol;
  int alpha_mode, maxit, refill_k;
};

__device__ __forceinline__ float blk_rsqrt_ftz(float v) {
  float r;
  asm("rsqrt.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(v));
  return r;
}

// Stage tensor t into buffer `buf` (warp-cooperative): B[q][j] = coef_q * a_{cls(q,j)}, rows padded to
// NP4 words with zeros; word Q*NP4 holds the tensor's shift (alpha modes 1-3).
template <int N>
__device__ void blk_stage(const BlkParams& p, long long t, float* buf, int lane) {
  constexpr int NP4 = (N + 3) / 4 * 4;
  const float* a = p.entries + t * p.U;
  const int words = p.Q * NP4;
  for (int w = lane; w < words; w += 32) {
    const int r = w / NP4, j = w - r * NP4;
    const int q = (int)__ldg(p.qperm + r);
    buf[w] = (j < N) ? __ldg(p.coef + q) * __ldg(a + __ldg(p.cls + q * N + j)) : 0.f;
  }
  if (p.alpha_mode >= 1) {
    float v;
    if (p.alpha_mode == 1) {
      v = __ldg(p.alpha_in + t);
    } else {                                                   // R17: (m-1) sum_c (m!/k!) |a_c|
      float b = 0.f;
      for (int c = lane; c < p.U; c += 32) b = fmaf((float)__ldg(p.cls_mult + c), fabsf(__ldg(a + c)), b);
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) b += __shfl_xor_sync(0xffffffffu, b, o);
      b *= (float)(p.m - 1);
      v = p.alpha_mode == 2 ? b : -b;
    }
    if (lane == 0) buf[words] = v;
  }
}

template <int N>
__global__ void __launch_bounds__(128) sshopm_blocked_kernel(const BlkParams p) {
  constexpr int NP4 = (N + 3) / 4 * 4;
  extern __shared__ float bsm[];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const uint32_t FULL = 0xffffffffu;
  uint32_t ltmask;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(ltmask));
  // CTA tables: recipe [L], grouped prefixes [P], group sizes [N]
  uint32_t* t_rec = reinterpret_cast<uint32_t*>(bsm);
  uint32_t* t_pidx = t_rec + p.L;
  uint32_t* t_gcnt = t_pidx + p.P;
  for (int i = threadIdx.x; i < p.L; i += blockDim.x) t_rec[i] = p.recipe[i];
  for (int i = threadIdx.x; i < p.P; i += blockDim.x) t_pidx[i] = p.pidx[i];
  for (int i = threadIdx.x; i < N; i += blockDim.x) t_gcnt[i] = p.gcnt[i];
  // per warp: two B buffers (16-byte aligned, the second offset by 16 bytes modulo 128 so the two
  // tensors' rows fall in different banks), then the lane-interleaved low monomials
  const int tab_words = (p.L + p.P + N + 3) / 4 * 4;
  const int bw = (p.buf_words + 3) / 4 * 4;
  const int warp_words = 2 * bw + 4 + 32 * p.mono_words;
  float* wb = bsm + tab_words + warp * warp_words;
  const int bstride = bw + 4;                                      // buffer b at wb + b * bstride
  char* mono = reinterpret_cast<char*>(wb + 2 * bstride - 4) + lane * 4;   // mono[i] at mono + 128 i; mono[0..N) = x
#define MONO(i) (*reinterpret_cast<float*>(mono + (size_t)(i) * 128))
  __syncthreads();

  const int m = p.m, S = p.S, Q = p.Q, P = p.P, low = p.low;
  const int offP = low - (m >= 3 ? P : 0);                         // stored monomials: degree 1..m-3 = [0, offP)
  // warp-uniform: tensor held by each buffer (-1: none), the buffer being filled and its next start
  long long bt0 = -1, bt1 = -1;
  int fb = 1, fill_s = S;
  bool exhausted = false;
  uint32_t k_eff = (uint32_t)p.refill_k;
  // lane state
  float x[N];
#pragma unroll
  for (int j = 0; j < N; ++j) x[j] = 0.f;
  float lam = 0.f, lamp = 0.f, la = 0.f, ls = 1.f;
  int k = 0, s = 0, b = 0;
  bool has = false, stop = true, conv = false;
  const float4* brow = reinterpret_cast<const float4*>(wb);
  uint32_t it_sum = 0;

  for (;;) {
    const uint32_t smask = __ballot_sync(FULL, stop);
    const uint32_t cnt = __popc(smask);
    if (cnt >= k_eff) {
      const long long mt = b ? bt1 : bt0;
      if (stop && has) {                                             // A7: outputs of the finished start
        const long long item = mt * S + s;
        p.out_lambda[item] = lam;
#pragma unroll
        for (int j = 0; j < N; ++j) p.out_x[item * N + j] = x[j];
        p.out_iters[item] = k;
        p.out_conv[item] = conv ? 1 : 0;
        it_sum += (uint32_t)k;
      }
      const uint32_t rank = __popc(smask & ltmask);
      uint32_t avail = (uint32_t)(S - fill_s);
      // the fill tensor cannot serve every idle lane: stage the next tensor into the other buffer
      // once no running lane uses it
      bool fresh = false;
      if (!exhausted && cnt > avail) {
        const int ob = fb ^ 1;
        const uint32_t busy = __ballot_sync(FULL, has && !stop && b == ob);
        if (busy == 0u) {
          unsigned int tn = 0;
          if (lane == 0) tn = atomicAdd(p.counter, 1u);
          tn = __shfl_sync(FULL, tn, 0);
          if ((long long)tn < p.N) {
            __syncwarp();
            blk_stage<N>(p, (long long)tn, wb + ob * bstride, lane);
            __syncwarp();
            if (ob) bt1 = tn; else bt0 = tn;
            fresh = true;
          } else {
            exhausted = true;
            k_eff = 32u;
          }
        }
      }
      const bool cur = rank < avail;
      const bool ok = stop && (cur || (fresh && rank - avail < (uint32_t)S));
      if (ok) {
        b = cur ? fb : (fb ^ 1);
        s = cur ? fill_s + (int)rank : (int)(rank - avail);
        const float* bb = wb + b * bstride;
        brow = reinterpret_cast<const float4*>(bb);
        float nn = 0.f;
#pragma unroll
        for (int j = 0; j < N; ++j) { x[j] = __ldg(p.starts + (size_t)s * N + j); nn = fmaf(x[j], x[j], nn); }
        const float r0 = nn > 0.f ? rsqrtf(nn) : 0.f;               // R7
#pragma unroll
        for (int j = 0; j < N; ++j) { x[j] *= r0; MONO(j) = x[j]; }
        const float a = p.alpha_mode >= 1 ? bb[Q * NP4] : p.alpha;
        ls = a >= 0.f ? 1.f : -1.f;                                  // R5
        la = fabsf(a);
        k = 0;
        lamp = __int_as_float(0x7fffffff);                          // NaN: the first test never fires (R2)
      }
      has = stop ? ok : has;
      if (fresh) {
        fb ^= 1;
        fill_s = (int)min((uint32_t)S, cnt - avail);
      } else {
        fill_s += (int)min(cnt, avail);
      }
      if (exhausted && __ballot_sync(FULL, has) == 0u) break;
    }

    // ---- one SS-HOPM step (Fig. 1) ----
    for (int i = N; i < offP; ++i) {                                // monomials of degree 2..m-3
      const uint32_t r = t_rec[i];
      MONO(i) = MONO(r & 0xffffu) * MONO(r >> 16);
    }
    float g[N];
#pragma unroll
    for (int j = 0; j < N; ++j) g[j] = 0.f;
    // blocks grouped by the prefix's last index l (compile-time in the unrolled l loop), so each
    // block's rows i = l..N-1 are straight-line code: no branch between its broadcast loads and FMAs
    const float4* row = brow;
    int pp = 0;
#pragma unroll
    for (int l = 0; l < N; ++l) {
      const int cnt = (int)t_gcnt[l];
      // x^p = x^{p - e_l} x_l: the prefix's own prefix from shared memory (prefetched one block
      // ahead), x_l from a register (l is compile-time here); m = 3: x^p = x_l, m = 2: x^p = 1
      float mpn = (m >= 4 && cnt > 0) ? MONO((int)t_pidx[pp]) : 1.f;
      for (int c = 0; c < cnt; ++c, ++pp) {
        const float mp = (m >= 4) ? mpn * x[l] : (m == 3 ? x[l] : 1.f);
        if (m >= 4 && c + 1 < cnt) mpn = MONO((int)t_pidx[pp + 1]);
#pragma unroll
        for (int i = l; i < N; ++i) {
          const float cm = mp * x[i];
          float4 w[NP4 / 4];
#pragma unroll
          for (int v = 0; v < NP4 / 4; ++v) w[v] = row[v];
#pragma unroll
          for (int j = 0; j < N; ++j) {
            const float bj = (j % 4 == 0) ? w[j / 4].x : (j % 4 == 1) ? w[j / 4].y : (j % 4 == 2) ? w[j / 4].z : w[j / 4].w;
            g[j] = fmaf(bj, cm, g[j]);
          }
          row += NP4 / 4;
        }
      }
    }
    lam = 0.f;
#pragma unroll
    for (int j = 0; j < N; ++j) lam = fmaf(x[j], g[j], lam);       // lambda_k = x_k . g
    conv = fabsf(lam - lamp) <= p.tol * fmaxf(1.0f, fabsf(lam));    // R2
    float nn = 0.f;
#pragma unroll
    for (int j = 0; j < N; ++j) { g[j] = fmaf(la, x[j], ls * g[j]); nn = fmaf(g[j], g[j], nn); }   // +-(g + alpha x)
    const bool deg = !(nn >= 1.17549435e-38f);                     // R6
    stop = (!has) | conv | (k >= p.maxit) | deg;
    const float r = blk_rsqrt_ftz(nn);
    if (!stop) {
#pragma unroll
      for (int j = 0; j < N; ++j) { x[j] = g[j] * r; MONO(j) = x[j]; }
      lamp = lam;
      ++k;
    }
  }
#undef MONO
  if (p.total_iters) {
    unsigned long long ws = it_sum;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) ws += __shfl_xor_sync(FULL, ws, o);
    if (lane == 0) atomicAdd(p.total_iters, ws);
  }
}

// ------------------------------------------------------------------ host --
static int blk_smem(const GeneralTables* t, int warps) {
  const int NP4 = (t->n + 3) / 4 * 4;
  const int tab_words = (t->L + t->P + t->n + 3) / 4 * 4;
  const int bw = (t->Q * NP4 + 4 + 3) / 4 * 4;
  const int stored = t->L - t->Q - (t->m >= 3 ? t->P : 0);           // degrees 1..m-3
  const int mono = stored > t->n ? stored : t->n;
  return 4 * (tab_words + warps * (2 * bw + 4 + 32 * mono));
}

bool blocked_fits(const GeneralTables* t) { return t && t->recipe && t->qperm && blk_smem(t, 1) <= 200 * 1024; }

// CTA size: the one of 4 / 2 / 1 warps that keeps the most warps resident per SM (each warp holds
// its own two tensor buffers, so shared memory, not registers, usually bounds the occupancy)
template <int N>
static cudaError_t launch_blocked(const BlkParams& p, const GeneralTables* t, cudaStream_t st) {
  int warps = 0, bps = 0, smem = 0;
  for (int w = 4; w >= 1; w >>= 1) {
    const int sm = blk_smem(t, w);
    if (sm > 200 * 1024) continue;
    cudaError_t e = cudaFuncSetAttribute(sshopm_blocked_kernel<N>, cudaFuncAttributeMaxDynamicSharedMemorySize, sm);
    if (e != cudaSuccess) return e;
    int b = 0;
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, sshopm_blocked_kernel<N>, 32 * w, sm);
    if (e != cudaSuccess) return e;
    if (b * w > bps * warps) { warps = w; bps = b; smem = sm; }
  }
  if (bps < 1) return cudaErrorInvalidConfiguration;
  cudaError_t e = cudaFuncSetAttribute(sshopm_blocked_kernel<N>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  if (e != cudaSuccess) return e;
  long long grid = (long long)device_sms() * bps;
  const long long need = (p.N + 2LL * warps - 1) / (2LL * warps);   // >= 2 tensors per warp
  if (grid > need) grid = need > 0 ? need : 1;
  sshopm_blocked_kernel<N><<<(int)grid, 32 * warps, smem, st>>>(p);
  return cudaGetLastError();
}

int blocked_solve(const GeneralTables* t, int64_t N, const float* d_entries, int S, const float* d_starts, float alpha,
                  float tol, int maxit, float* d_lambda, float* d_x, int32_t* d_iters, uint8_t* d_conv,
                  const sshopm_solve_opts* opts, cudaStream_t st) {
  if (!blocked_fits(t)) return SSHOPM_EUNSUPPORTED;
  const int alpha_mode = opts ? opts->alpha_mode : 0;
  if (alpha_mode < 0 || alpha_mode > 3 || (alpha_mode == 1 && !opts->d_alpha)) return SSHOPM_EINVAL;
  const int n = t->n;
  auto al = [](size_t v) { return (v + 255) / 256 * 256; };
  const size_t b_rec = al((size_t)t->L * 4), b_coef = al((size_t)t->Q * 4), b_cls = al((size_t)t->Q * n * 4);
  const size_t b_mult = al((size_t)t->U * 4), b_pidx = al((size_t)t->P * 4), b_gcnt = al((size_t)n * 4);
  const size_t b_qperm = al((size_t)t->Q * 4);
  char* tab = nullptr;
  cudaError_t e = cudaMallocAsync(reinterpret_cast<void**>(&tab), 256 + b_rec + b_coef + b_cls + b_mult + b_pidx + b_gcnt + b_qperm, st);
  if (e != cudaSuccess) return e == cudaErrorMemoryAllocation ? SSHOPM_ENOMEM : cuda_fail(e, "blocked: malloc");
  BlkParams p;
  memset(&p, 0, sizeof(p));
  char* o = tab;
  p.counter = reinterpret_cast<unsigned int*>(o); o += 256;
  p.recipe = reinterpret_cast<const uint32_t*>(o); o += b_rec;
  p.coef = reinterpret_cast<const float*>(o); o += b_coef;
  p.cls = reinterpret_cast<const uint32_t*>(o); o += b_cls;
  p.cls_mult = reinterpret_cast<const int*>(o); o += b_mult;
  p.pidx = reinterpret_cast<const uint32_t*>(o); o += b_pidx;
  p.gcnt = reinterpret_cast<const uint32_t*>(o); o += b_gcnt;
  p.qperm = reinterpret_cast<const uint32_t*>(o);
  e = cudaMemsetAsync(tab, 0, 256, st);
  if (e == cudaSuccess) e = cudaMemcpyAsync((void*)p.recipe, t->recipe, (size_t)t->L * 4, cudaMemcpyHostToDevice, st);
  if (e == cudaSuccess) e = cudaMemcpyAsync((void*)p.coef, t->coef, (size_t)t->Q * 4, cudaMemcpyHostToDevice, st);
  if (e == cudaSuccess) e = cudaMemcpyAsync((void*)p.cls, t->cls_idx, (size_t)t->Q * n * 4, cudaMemcpyHostToDevice, st);
  if (e == cudaSuccess) e = cudaMemcpyAsync((void*)p.cls_mult, t->mult, (size_t)t->U * 4, cudaMemcpyHostToDevice, st);
  if (e == cudaSuccess) e = cudaMemcpyAsync((void*)p.pidx, t->ppar, (size_t)t->P * 4, cudaMemcpyHostToDevice, st);
  if (e == cudaSuccess) e = cudaMemcpyAsync((void*)p.gcnt, t->gcnt, (size_t)n * 4, cudaMemcpyHostToDevice, st);
  if (e == cudaSuccess) e = cudaMemcpyAsync((void*)p.qperm, t->qperm, (size_t)t->Q * 4, cudaMemcpyHostToDevice, st);
  if (e != cudaSuccess) { cudaFreeAsync(tab, st); return cuda_fail(e, "blocked: table upload"); }
  p.entries = d_entries;
  p.starts = d_starts;
  p.out_lambda = d_lambda;
  p.out_x = d_x;
  p.out_iters = d_iters;
  p.out_conv = d_conv;
  p.total_iters = opts ? opts->d_total_iters : nullptr;
  p.alpha_in = alpha_mode == 1 ? opts->d_alpha : nullptr;
  p.N = N;
  p.m = t->m;
  p.U = t->U;
  p.S = S;
  p.L = t->L;
  p.Q = t->Q;
  p.P = t->P;
  p.low = t->L - t->Q;
  const int stored = p.low - (t->m >= 3 ? t->P : 0);
  p.mono_words = stored > n ? stored : n;
  p.buf_words = t->Q * ((n + 3) / 4 * 4) + 4;
  p.alpha = alpha;
  p.tol = tol;
  p.alpha_mode = alpha_mode;
  p.maxit = maxit;
  const int k = (opts && opts->refill_threshold > 0) ? opts->refill_threshold : 4;
  p.refill_k = k < 1 ? 1 : (k > 32 ? 32 : k);
  switch (n) {
#define BLK_CASE(NN) case NN: e = launch_blocked<NN>(p, t, st); break;
    BLK_CASE(1) BLK_CASE(2) BLK_CASE(3) BLK_CASE(4) BLK_CASE(5) BLK_CASE(6) BLK_CASE(7) BLK_CASE(8)
    BLK_CASE(9) BLK_CASE(10) BLK_CASE(11) BLK_CASE(12) BLK_CASE(13) BLK_CASE(14) BLK_CASE(15) BLK_CASE(16)
#undef BLK_CASE
    default: e = cudaErrorInvalidValue;
  }
  cudaFreeAsync(tab, st);
  if (e != cudaSuccess) return cuda_fail(e, "blocked: launch");
  return SSHOPM_OK;
}

}  // namespace sshopm
