// general.cu — table-driven SS-HOPM for any (m, n) (the paper's "general"
// implementation).
//
// Mapping as in the paper: one block per tensor (grid-stride),
// its U entries and the shared index/multinomial tables in shared memory
// ("the index information is stored as an array of size m x U and can
// be shared by all threads ... We store the multinomial coefficient for each
// unique tensor value"), one thread per start.  Per evaluation each thread
// walks the U classes (Fig. 2/3 order); for the first occurrence t of each
// index i in the class it adds sigma(i) a_c x^{k - e_i} with
// sigma(i) = c * k_i / m and x^{k - e_i} = prefix(t) * suffix(t) (the
// product without one occurrence of i — never a division, reading R10).
// lambda = x . g (Euler identity).  Stopping rule, shift and outputs are
// exactly those of the specialised kernels (readings R1-R7).
#include <cstdio>
#include <cstring>
#include <new>

#include "api_internal.h"
#include "general.h"
#include "sshopm.h"

namespace sshopm {

struct GenParams {
  const float* entries;      // [N][U]
  const float* starts;       // [S][n] raw
  const uint8_t* cls_idx;    // [U][m] 0-based
  const int* cls_mult;       // [U]  m!/k!
  float* out_lambda;
  float* out_x;
  int32_t* out_iters;
  uint8_t* out_conv;
  unsigned long long* total_iters;
  const float* alpha_in;     // alpha_mode 1
  long long N;
  int m, n, U, S;
  float alpha, tol;
  int alpha_mode, maxit;
};

// g = A x^{m-1} (Eq. 6 by classes) for this thread; x, g in the thread's shared slots
__device__ __forceinline__ void gen_eval(const GenParams& p, const float* __restrict__ ent, const uint8_t* __restrict__ idx,
                                         const int* __restrict__ mult, const float* x, float* g) {
  const int m = p.m, n = p.n;
  for (int j = 0; j < n; ++j) g[j] = 0.f;
  float suf[kGenMaxM + 1];
  for (int c = 0; c < p.U; ++c) {
    const uint8_t* I = idx + c * m;
    suf[m] = 1.f;
    for (int t = m - 1; t >= 0; --t) suf[t] = suf[t + 1] * x[I[t]];
    const float ca = (float)mult[c] * ent[c] / (float)m;        // c * a_c / m
    float pre = 1.f;
    int t = 0;
    while (t < m) {
      const int i = I[t];
      int k = 1;
      while (t + k < m && I[t + k] == i) ++k;
      g[i] = fmaf(ca * (float)k, pre * suf[t + 1], g[i]);      // sigma(i) a_c x^{k - e_i}
      for (int r = 0; r < k; ++r) pre *= x[i];
      t += k;
    }
  }
}

__global__ void __launch_bounds__(128) sshopm_general_kernel(const GenParams p) {
  extern __shared__ float gsm[];
  const int m = p.m, n = p.n, U = p.U;
  float* ent = gsm;                                                   // [U]
  int* mult = reinterpret_cast<int*>(ent + U);                        // [U]
  float* xs = reinterpret_cast<float*>(mult + U) + threadIdx.x * (2 * n + 1);
  float* g = xs + n;
  uint8_t* idx = reinterpret_cast<uint8_t*>(reinterpret_cast<float*>(mult + U) + blockDim.x * (2 * n + 1));
  for (int i = threadIdx.x; i < U * m; i += blockDim.x) idx[i] = p.cls_idx[i];
  for (int i = threadIdx.x; i < U; i += blockDim.x) mult[i] = p.cls_mult[i];
  unsigned long long it_sum = 0;
  for (long long v = blockIdx.x; v < p.N; v += gridDim.x) {
    __syncthreads();
    for (int i = threadIdx.x; i < U; i += blockDim.x) ent[i] = p.entries[v * U + i];
    __syncthreads();
    float alpha = p.alpha;
    if (p.alpha_mode == 1) {
      alpha = p.alpha_in[v];
    } else if (p.alpha_mode >= 2) {
      float b = 0.f;
      for (int c = 0; c < U; ++c) b = fmaf((float)mult[c], fabsf(ent[c]), b);
      alpha = (p.alpha_mode == 2 ? 1.f : -1.f) * (float)(m - 1) * b;
    }
    const float sg = alpha >= 0.f ? 1.f : -1.f;                      // Fig. 1 lines 2-5 (R5)
    for (int s = threadIdx.x; s < p.S; s += blockDim.x) {
      float nn = 0.f;
      for (int j = 0; j < n; ++j) { xs[j] = p.starts[(size_t)s * n + j]; nn = fmaf(xs[j], xs[j], nn); }
      const float r0 = nn > 0.f ? rsqrtf(nn) : 0.f;                  // R7
      for (int j = 0; j < n; ++j) xs[j] *= r0;
      float lamp = __int_as_float(0x7fffffff), lam = 0.f;
      int k = 0;
      bool conv = false;
      for (;;) {
        gen_eval(p, ent, idx, mult, xs, g);
        lam = 0.f;
        for (int j = 0; j < n; ++j) lam = fmaf(xs[j], g[j], lam);   // lambda_k = x_k . g
        conv = fabsf(lam - lamp) <= p.tol * fmaxf(1.0f, fabsf(lam)); // R2
        if (conv || k >= p.maxit) break;
        float h2 = 0.f;
        for (int j = 0; j < n; ++j) { g[j] = sg * fmaf(alpha, xs[j], g[j]); h2 = fmaf(g[j], g[j], h2); }
        if (!(h2 >= 1.17549435e-38f)) break;                         // R6
        const float r = rsqrtf(h2);
        for (int j = 0; j < n; ++j) xs[j] = g[j] * r;
        lamp = lam;
        ++k;
      }
      const long long item = v * p.S + s;
      p.out_lambda[item] = lam;
      for (int j = 0; j < n; ++j) p.out_x[item * n + j] = xs[j];
      p.out_iters[item] = k;
      p.out_conv[item] = conv ? 1 : 0;
      it_sum += (unsigned long long)k;
    }
  }
  if (p.total_iters && it_sum) atomicAdd(p.total_iters, it_sum);
}

// test hook: g = A x^{m-1}, lambda = x . g for N (tensor, x) pairs (thread per pair)
__global__ void __launch_bounds__(128) sshopm_general_apply_kernel(const GenParams p, const float* __restrict__ x,
                                                                   float* __restrict__ out_g, float* __restrict__ out_lam) {
  extern __shared__ float gsm[];
  const int m = p.m, n = p.n, U = p.U;
  int* mult = reinterpret_cast<int*>(gsm);
  float* xs = reinterpret_cast<float*>(mult + U) + threadIdx.x * (2 * n + 1);
  float* g = xs + n;
  uint8_t* idx = reinterpret_cast<uint8_t*>(reinterpret_cast<float*>(mult + U) + blockDim.x * (2 * n + 1));
  for (int i = threadIdx.x; i < U * m; i += blockDim.x) idx[i] = p.cls_idx[i];
  for (int i = threadIdx.x; i < U; i += blockDim.x) mult[i] = p.cls_mult[i];
  __syncthreads();
  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < p.N; i += (long long)gridDim.x * blockDim.x) {
    for (int j = 0; j < n; ++j) xs[j] = x[i * n + j];
    gen_eval(p, p.entries + i * U, idx, mult, xs, g);
    float lam = 0.f;
    for (int j = 0; j < n; ++j) { out_g[i * n + j] = g[j]; lam = fmaf(xs[j], g[j], lam); }
    out_lam[i] = lam;
  }
}

// ------------------------------------------------ item-per-lane general kernel --
// The default table-driven path (any (m, n) whose per-lane arrays fit in shared
// memory).  Same stopping rule, shift and outputs as every other kernel, but
// scheduled like the unrolled solve kernel: persistent warps claim chunks of
// whole tensors, one lane = one (tensor, start) item, stopped lanes are refilled
// in batches.  Evaluation is Eq. 6 regrouped by the degree-(m-1) monomial q
// (DESIGN.md "Evaluation"): (A x^{m-1})_j = sum_q [(m-1)!/q!] a_{class(q+e_j)} x^q,
// with every monomial of degree 1..m-1 built from its prefix by one multiply
// (table `recipe`, lexicographic within a degree; degree 1 is x itself).
// Per-lane arrays live in shared memory, lane-interleaved (element c of lane l at
// word 32 c + l) so every access is bank-conflict free: the tensor row (U
// entries) and the monomials (L words, the first n of which hold x).
struct Gen2Params {
  const float* entries;      // [N][U]
  const float* starts;       // [S][n] raw
  const uint32_t* recipe;    // [L]: (parent | var << 16) for i >= n (degree >= 2)
  const float* coef;         // [Q]: (m-1)!/q!
  const uint32_t* cls;       // [Q][n]: byte offset 128 * class(q + e_j) in the lane-interleaved row
  const int* cls_mult;       // [U]: m!/k! (automatic shift)
  float* out_lambda;
  float* out_x;
  int32_t* out_iters;
  uint8_t* out_conv;
  unsigned long long* total_iters;
  const float* alpha_in;     // alpha_mode 1
  unsigned int* counter;     // chunk counter (zeroed by the host)
  long long N, n_chunks;
  int chunk_tensors;
  int m, n, U, S, L, Q;
  float alpha, tol;
  int alpha_mode, maxit, refill_k;
};

__device__ __forceinline__ float gen_rsqrt_ftz(float v) {
  float r;
  asm("rsqrt.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(v));
  return r;
}

template <int NMAX>
__global__ void __launch_bounds__(256) sshopm_general2_kernel(const Gen2Params p) {
  extern __shared__ float gsm[];
  const int n = p.n, U = p.U, L = p.L, Q = p.Q;
  const int lane = threadIdx.x & 31;
  const uint32_t FULL = 0xffffffffu;
  uint32_t ltmask;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(ltmask));
  // tables (shared by the CTA), then per-warp lane-interleaved arrays
  uint32_t* t_rec = reinterpret_cast<uint32_t*>(gsm);
  float* t_coef = reinterpret_cast<float*>(t_rec + L);
  uint32_t* t_cls = reinterpret_cast<uint32_t*>(t_coef + Q);
  int* t_mult = reinterpret_cast<int*>(t_cls + Q * n);
  for (int i = threadIdx.x; i < L; i += blockDim.x) t_rec[i] = p.recipe[i];
  for (int i = threadIdx.x; i < Q; i += blockDim.x) t_coef[i] = p.coef[i];
  for (int i = threadIdx.x; i < Q * n; i += blockDim.x) t_cls[i] = p.cls[i];
  for (int i = threadIdx.x; i < U; i += blockDim.x) t_mult[i] = p.cls_mult[i];
  __syncthreads();
  char* wbase = reinterpret_cast<char*>(t_mult + U) + (size_t)(threadIdx.x >> 5) * 32 * (U + L) * 4 + lane * 4;
  char* row = wbase;                                   // row[c] at row + 128 c
  char* mono = wbase + (size_t)U * 128;                // mono[i] at mono + 128 i; mono[0..n) = x
#define ROW(c) (*reinterpret_cast<float*>(row + (size_t)(c) * 128))
#define MONO(i) (*reinterpret_cast<float*>(mono + (size_t)(i) * 128))

  // warp-uniform chunk state (global item indices)
  long long c_next = 0, c_end = 0;
  bool exhausted = false;
  uint32_t k_eff = (uint32_t)p.refill_k;
  float x[NMAX];
#pragma unroll
  for (int j = 0; j < NMAX; ++j) x[j] = 0.f;
  float lam = 0.f, lamp = 0.f, la = 0.f, ls = 1.f;
  int k = 0;
  bool has = false, stop = true, conv = false;
  long long item = 0;
  uint32_t it_sum = 0;
  const long long S = p.S;
  const int offD = L - Q;

  for (;;) {
    const uint32_t smask = __ballot_sync(FULL, stop);
    const uint32_t cnt = __popc(smask);
    if (cnt >= k_eff) {
      if (stop && has) {
        p.out_lambda[item] = lam;
#pragma unroll
        for (int j = 0; j < NMAX; ++j)
          if (j < n) p.out_x[item * n + j] = x[j];
        p.out_iters[item] = k;
        p.out_conv[item] = conv ? 1 : 0;
        it_sum += (uint32_t)k;
      }
      const long long avail = c_end - c_next;
      long long n_begin = 0, n_end = 0;
      if (!exhausted && (long long)cnt > avail) {
        unsigned int ch = 0;
        if (lane == 0) ch = atomicAdd(p.counter, 1u);
        ch = __shfl_sync(FULL, ch, 0);
        if ((long long)ch < p.n_chunks) {
          const long long t0 = (long long)ch * p.chunk_tensors;
          const long long t1 = min(p.N, t0 + p.chunk_tensors);
          n_begin = t0 * S;
          n_end = t1 * S;
        }
      }
      const long long rank = __popc(smask & ltmask);
      const long long t = rank < avail ? c_next + rank : n_begin + (rank - avail);
      const bool ok = stop && !exhausted && (rank < avail || t < n_end);
      if (ok) {
        item = t;
        const long long v = t / S;
        const int s = (int)(t - v * S);
        const float* e = p.entries + v * U;
        for (int c = 0; c < U; ++c) ROW(c) = __ldg(e + c);
        float nn = 0.f;
#pragma unroll
        for (int j = 0; j < NMAX; ++j)
          if (j < n) { x[j] = __ldg(p.starts + (size_t)s * n + j); nn = fmaf(x[j], x[j], nn); }
        const float r0 = nn > 0.f ? rsqrtf(nn) : 0.f;                          // R7
#pragma unroll
        for (int j = 0; j < NMAX; ++j)
          if (j < n) { x[j] *= r0; MONO(j) = x[j]; }
        float a = p.alpha;
        if (p.alpha_mode == 1) {
          a = __ldg(p.alpha_in + v);
        } else if (p.alpha_mode >= 2) {                                       // R17 bound
          float b = 0.f;
          for (int c = 0; c < U; ++c) b = fmaf((float)t_mult[c], fabsf(ROW(c)), b);
          b *= (float)(p.m - 1);
          a = p.alpha_mode == 2 ? b : -b;
        }
        ls = a >= 0.f ? 1.f : -1.f;                                           // R5
        la = fabsf(a);
        k = 0;
        lamp = __int_as_float(0x7fffffff);                                    // NaN: first test never fires
      }
      has = stop ? ok : has;
      if (!exhausted) {
        if ((long long)cnt > avail) {
          if (n_end == 0) { exhausted = true; k_eff = 32u; }
          c_next = min(n_begin + ((long long)cnt - avail), n_end);
          c_end = n_end;
        } else {
          c_next += cnt;
        }
      }
      if (exhausted && __ballot_sync(FULL, has) == 0u) break;
    }

    // ---- one SS-HOPM step (Fig. 1) ----
#pragma unroll 4
    for (int i = n; i < L; ++i) {                                             // monomials of degree 2..m-1
      const uint32_t r = t_rec[i];
      MONO(i) = MONO(r & 0xffffu) * MONO(r >> 16);
    }
    float g[NMAX];
#pragma unroll
    for (int j = 0; j < NMAX; ++j) g[j] = 0.f;
    for (int q = 0; q < Q; ++q) {                                             // Eq. 6 by monomial
      const float cm = t_coef[q] * MONO(offD + q);
      const uint32_t* cq = t_cls + q * n;
#pragma unroll
      for (int j = 0; j < NMAX; ++j)
        if (j < n) g[j] = fmaf(*reinterpret_cast<const float*>(row + cq[j]), cm, g[j]);
    }
    lam = 0.f;
#pragma unroll
    for (int j = 0; j < NMAX; ++j)
      if (j < n) lam = fmaf(x[j], g[j], lam);                                // lambda_k = x_k . g
    conv = fabsf(lam - lamp) <= p.tol * fmaxf(1.0f, fabsf(lam));              // R2
    float nn = 0.f;
#pragma unroll
    for (int j = 0; j < NMAX; ++j)
      if (j < n) { g[j] = fmaf(la, x[j], ls * g[j]); nn = fmaf(g[j], g[j], nn); }   // xhat = +-(g + alpha x)
    const bool deg = !(nn >= 1.17549435e-38f);                               // R6
    stop = (!has) | conv | (k >= p.maxit) | deg;
    const float r = gen_rsqrt_ftz(nn);
    if (!stop) {
#pragma unroll
      for (int j = 0; j < NMAX; ++j)
        if (j < n) { x[j] = g[j] * r; MONO(j) = x[j]; }
      lamp = lam;
      ++k;
    }
  }
#undef ROW
#undef MONO
  if (p.total_iters) {
    unsigned long long ws = it_sum;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) ws += __shfl_xor_sync(FULL, ws, o);
    if (lane == 0) atomicAdd(p.total_iters, ws);
  }
}

// ------------------------------------------------------------------ host --
static long long binom_ll(int a, int b) {
  if (b < 0 || b > a) return 0;
  long long r = 1;
  for (int i = 1; i <= b; ++i) r = r * (a - b + i) / i;
  return r;
}

// lexicographic rank of a nondecreasing length-d tuple over {0..n-1} among all such tuples
static long long lex_rank(const int* I, int d, int n) {
  long long r = 0;
  int lo = 0;
  for (int p = 0; p < d; ++p) {
    for (int v = lo; v < I[p]; ++v) r += binom_ll((d - p - 1) + (n - v) - 1, d - p - 1);
    lo = I[p];
  }
  return r;
}

GeneralTables* general_create(int m, int n) {
  if (m < 2 || n < 1 || m > kGenMaxM || n > kGenMaxN) return nullptr;
  const long long U = binom_ll(m + n - 1, m);
  if (U > kGenMaxU) return nullptr;
  GeneralTables* t = new (std::nothrow) GeneralTables;
  if (!t) return nullptr;
  t->m = m;
  t->n = n;
  t->U = (int)U;
  t->idx = new (std::nothrow) uint8_t[U * m];
  t->mult = new (std::nothrow) int[U];
  if (!t->idx || !t->mult) { general_destroy(t); return nullptr; }
  // Fig. 4 UPDATEINDEX walk from [0..0]; multinomial by one pass
  int I[kGenMaxM] = {};
  long long fm = 1;
  for (int i = 2; i <= m; ++i) fm *= i;
  for (long long c = 0; c < U; ++c) {
    long long den = 1;
    int run = 1;
    for (int k = 0; k < m; ++k) {
      t->idx[c * m + k] = (uint8_t)I[k];
      if (k > 0 && I[k] == I[k - 1]) { ++run; den *= run; } else run = 1;
    }
    t->mult[c] = (int)(fm / den);
    int j = m - 1;
    while (j >= 0 && I[j] == n - 1) --j;
    if (j < 0) break;
    I[j] += 1;
    for (int k = j + 1; k < m; ++k) I[k] = I[j];
  }
  const long long Q = binom_ll(m + n - 2, m - 1);
  // item-per-lane kernel: monomials of degree 1..m-1 (lexicographic within a degree) built from
  // their prefix, and for each degree-(m-1) monomial q its coefficient (m-1)!/q! and the classes
  // of q + e_j (P:L180 for sigma)
  const int D = m - 1;
  const long long L = binom_ll(D + n, D) - 1;
  if (Q * n <= kBlkMaxT1 && L < 65536) {
    t->L = (int)L;
    t->Q = (int)Q;
    t->gen2 = (L + U <= kGen2MaxWords);
    t->P = m >= 3 ? (int)binom_ll(m - 2 + n - 1, m - 2) : 1;
    t->recipe = new (std::nothrow) uint32_t[L];
    t->coef = new (std::nothrow) float[Q];
    t->cls = new (std::nothrow) uint32_t[Q * n];
    t->cls_idx = new (std::nothrow) uint32_t[Q * n];
    t->plast = new (std::nothrow) uint32_t[t->P];
    if (!t->recipe || !t->coef || !t->cls || !t->cls_idx || !t->plast) { general_destroy(t); return nullptr; }
    t->plast[0] = 0;                                     // m = 2: the empty prefix (x^0 = 1)
    long long off = 0, prev_off = 0;
    for (int d = 1; d <= D; ++d) {
      int T[kGenMaxM] = {};
      const long long cnt = binom_ll(d + n - 1, d);
      for (long long i = 0; i < cnt; ++i) {
        if (d == m - 2) t->plast[i] = (uint32_t)T[d - 1];  // blocked kernel: last index of each prefix
        if (d == 1) t->recipe[off + i] = 0;
        else t->recipe[off + i] = (uint32_t)(prev_off + lex_rank(T, d - 1, n)) | ((uint32_t)T[d - 1] << 16);
        if (d == D) {
          const long long q = i;
          long long den = 1;
          int run = 1;
          for (int k = 1; k < d; ++k) { if (T[k] == T[k - 1]) { ++run; den *= run; } else run = 1; }
          long long fd = 1;
          for (int k = 2; k <= D; ++k) fd *= k;
          t->coef[q] = (float)((double)fd / (double)den);
          for (int j = 0; j < n; ++j) {                    // class of q + e_j: insert j into the sorted tuple
            int C[kGenMaxM + 1];
            int w = 0;
            bool put = false;
            for (int k = 0; k < d; ++k) {
              if (!put && j <= T[k]) { C[w++] = j; put = true; }
              C[w++] = T[k];
            }
            if (!put) C[w++] = j;
            t->cls_idx[q * n + j] = (uint32_t)lex_rank(C, m, n);
            t->cls[q * n + j] = 128u * t->cls_idx[q * n + j];
          }
        }
        int k2 = d - 1;                                     // Fig. 4 successor
        while (k2 >= 0 && T[k2] == n - 1) --k2;
        if (k2 < 0) break;
        T[k2] += 1;
        for (int r = k2 + 1; r < d; ++r) T[r] = T[k2];
      }
      prev_off = off;
      off += cnt;
    }
  }
  if (t->recipe) {
    // blocked kernel order: prefixes grouped by their last index l (stable, lexicographic within a
    // group), each followed by its rows q = p + e_i, i = l..n-1 (blocked.cu)
    const int d = m - 2, P = t->P;
    t->porder = new (std::nothrow) uint32_t[P];
    t->gcnt = new (std::nothrow) uint32_t[n];
    t->qperm = new (std::nothrow) uint32_t[Q];
    uint32_t* tup = new (std::nothrow) uint32_t[(size_t)P * (d > 0 ? d : 1)];
    if (!t->porder || !t->gcnt || !t->qperm || !tup) { delete[] tup; general_destroy(t); return nullptr; }
    int T[kGenMaxM] = {};
    for (int pi = 0; pi < P; ++pi) {                      // degree-d tuples in lexicographic order (Fig. 4)
      for (int k = 0; k < d; ++k) tup[(size_t)pi * d + k] = (uint32_t)T[k];
      int k2 = d - 1;
      while (k2 >= 0 && T[k2] == n - 1) --k2;
      if (k2 < 0) break;
      T[k2] += 1;
      for (int r = k2 + 1; r < d; ++r) T[r] = T[k2];
    }
    int np = 0, nq = 0;
    for (int l = 0; l < n; ++l) {
      t->gcnt[l] = 0;
      for (int pi = 0; pi < P; ++pi) {
        if ((int)t->plast[pi] != l) continue;
        t->porder[np++] = (uint32_t)pi;
        ++t->gcnt[l];
        for (int i = l; i < n; ++i) {
          int C[kGenMaxM];
          for (int k = 0; k < d; ++k) C[k] = (int)tup[(size_t)pi * d + k];
          C[d] = i;
          t->qperm[nq++] = (uint32_t)lex_rank(C, m - 1, n);
        }
      }
    }
    delete[] tup;
    if (np != P || nq != Q) { general_destroy(t); return nullptr; }
    t->ppar = new (std::nothrow) uint32_t[P];
    if (!t->ppar) { general_destroy(t); return nullptr; }
    const long long offP = (L - Q) - P;                  // recipe index of the first degree-(m-2) monomial
    for (int k = 0; k < P; ++k)
      t->ppar[k] = m >= 4 ? (t->recipe[offP + t->porder[k]] & 0xffffu) : 0u;
  }
  t->paper_flops = (long long)(m + 2) * U + (long long)(m + 1) * n * Q + 5LL * n;
  // executed per update: per class ~ (m suffix + m prefix + 3 per unique index) + lambda/shift/normalise
  t->exec_flops = U * (2LL * m + 3LL * n / 2) + 7LL * n;
  return t;
}

void general_destroy(GeneralTables* t) {
  if (!t) return;
  delete[] t->idx;
  delete[] t->mult;
  delete[] t->recipe;
  delete[] t->coef;
  delete[] t->cls;
  delete[] t->cls_idx;
  delete[] t->plast;
  delete[] t->porder;
  delete[] t->ppar;
  delete[] t->gcnt;
  delete[] t->qperm;
  delete t;
}

size_t general_table_bytes(const GeneralTables* t) { return ((size_t)t->U * t->m + 255) / 256 * 256 + (size_t)t->U * 4; }

static int general_smem(const GeneralTables* t, int block, bool with_entries) {
  return (with_entries ? t->U * 4 : 0) + t->U * 4 + block * (2 * t->n + 1) * 4 + t->U * t->m;
}

int general_upload(const GeneralTables* t, void* dev, cudaStream_t st, const uint8_t** d_idx, const int** d_mult) {
  uint8_t* di = reinterpret_cast<uint8_t*>(dev);
  int* dm = reinterpret_cast<int*>(di + ((size_t)t->U * t->m + 255) / 256 * 256);
  cudaError_t e = cudaMemcpyAsync(di, t->idx, (size_t)t->U * t->m, cudaMemcpyHostToDevice, st);
  if (e == cudaSuccess) e = cudaMemcpyAsync(dm, t->mult, (size_t)t->U * 4, cudaMemcpyHostToDevice, st);
  if (e != cudaSuccess) return cuda_fail(e, "general: table upload");
  *d_idx = di;
  *d_mult = dm;
  return SSHOPM_OK;
}

template <int NMAX>
static cudaError_t launch_general2(const Gen2Params& p, int warps, int smem, cudaStream_t st) {
  cudaError_t e = cudaFuncSetAttribute(sshopm_general2_kernel<NMAX>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  if (e != cudaSuccess) return e;
  int bps = 0;
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, sshopm_general2_kernel<NMAX>, 32 * warps, smem);
  if (e != cudaSuccess) return e;
  if (bps < 1) return cudaErrorInvalidConfiguration;
  long long grid = (long long)device_sms() * bps;
  const long long need = (p.n_chunks + 3) / 4;            // >= 4 chunks per warp-group on average
  if (grid > need) grid = need > 0 ? need : 1;
  sshopm_general2_kernel<NMAX><<<(int)grid, 32 * warps, smem, st>>>(p);
  return cudaGetLastError();
}

// item-per-lane general kernel (tables in the handle's host copy, uploaded per call)
static int general2_solve(const GeneralTables* t, int64_t N, const float* d_entries, int S, const float* d_starts,
                          float alpha, float tol, int maxit, float* d_lambda, float* d_x, int32_t* d_iters,
                          uint8_t* d_conv, const sshopm_solve_opts* opts, cudaStream_t st, int warps, int smem) {
  const int alpha_mode = opts ? opts->alpha_mode : 0;
  if (alpha_mode < 0 || alpha_mode > 3 || (alpha_mode == 1 && !opts->d_alpha)) return SSHOPM_EINVAL;
  const size_t b_rec = ((size_t)t->L * 4 + 255) / 256 * 256, b_coef = ((size_t)t->Q * 4 + 255) / 256 * 256;
  const size_t b_cls = ((size_t)t->Q * t->n * 4 + 255) / 256 * 256, b_mult = ((size_t)t->U * 4 + 255) / 256 * 256;
  char* tab = nullptr;
  cudaError_t e = cudaMallocAsync(reinterpret_cast<void**>(&tab), 256 + b_rec + b_coef + b_cls + b_mult, st);
  if (e != cudaSuccess) return e == cudaErrorMemoryAllocation ? SSHOPM_ENOMEM : cuda_fail(e, "general: malloc");
  Gen2Params p;
  memset(&p, 0, sizeof(p));
  p.counter = reinterpret_cast<unsigned int*>(tab);
  p.recipe = reinterpret_cast<const uint32_t*>(tab + 256);
  p.coef = reinterpret_cast<const float*>(tab + 256 + b_rec);
  p.cls = reinterpret_cast<const uint32_t*>(tab + 256 + b_rec + b_coef);
  p.cls_mult = reinterpret_cast<const int*>(tab + 256 + b_rec + b_coef + b_cls);
  e = cudaMemsetAsync(tab, 0, 256, st);
  if (e == cudaSuccess) e = cudaMemcpyAsync((void*)p.recipe, t->recipe, (size_t)t->L * 4, cudaMemcpyHostToDevice, st);
  if (e == cudaSuccess) e = cudaMemcpyAsync((void*)p.coef, t->coef, (size_t)t->Q * 4, cudaMemcpyHostToDevice, st);
  if (e == cudaSuccess) e = cudaMemcpyAsync((void*)p.cls, t->cls, (size_t)t->Q * t->n * 4, cudaMemcpyHostToDevice, st);
  if (e == cudaSuccess) e = cudaMemcpyAsync((void*)p.cls_mult, t->mult, (size_t)t->U * 4, cudaMemcpyHostToDevice, st);
  if (e != cudaSuccess) { cudaFreeAsync(tab, st); return cuda_fail(e, "general: table upload"); }
  p.entries = d_entries;
  p.starts = d_starts;
  p.out_lambda = d_lambda;
  p.out_x = d_x;
  p.out_iters = d_iters;
  p.out_conv = d_conv;
  p.total_iters = opts ? opts->d_total_iters : nullptr;
  p.alpha_in = alpha_mode == 1 ? opts->d_alpha : nullptr;
  p.N = N;
  p.chunk_tensors = chunk_tensors_for(S);
  p.n_chunks = (N + p.chunk_tensors - 1) / p.chunk_tensors;
  p.m = t->m;
  p.n = t->n;
  p.U = t->U;
  p.S = S;
  p.L = t->L;
  p.Q = t->Q;
  p.alpha = alpha;
  p.tol = tol;
  p.alpha_mode = alpha_mode;
  p.maxit = maxit;
  const int k = (opts && opts->refill_threshold > 0) ? opts->refill_threshold : 4;
  p.refill_k = k < 1 ? 1 : (k > 32 ? 32 : k);
  e = t->n <= 4 ? launch_general2<4>(p, warps, smem, st)
    : t->n <= 8 ? launch_general2<8>(p, warps, smem, st) : launch_general2<16>(p, warps, smem, st);
  cudaFreeAsync(tab, st);
  if (e != cudaSuccess) return cuda_fail(e, "general: launch");
  return SSHOPM_OK;
}

int general_solve(const GeneralTables* t, int64_t N, const float* d_entries, int S, const float* d_starts, float alpha,
                  float tol, int maxit, float* d_lambda, float* d_x, int32_t* d_iters, uint8_t* d_conv,
                  const sshopm_solve_opts* opts, cudaStream_t st) {
  // kernel choice: opts->schedule 3 = item per lane (general2), 5 = blocked (warp per tensor, blocked.cu),
  // 4 = block per tensor (the paper's mapping); default: blocked (measured faster than the item-per-lane
  // kernel on every uncompiled shape tried, 2x at (5,4) to 47x at (4,10): profiles/r1/large_shapes.txt),
  // else item per lane, else block per tensor
  const int sched = opts ? opts->schedule : 0;
  if (sched == 5 || sched == 0 || sched == 3) {
    int warps2 = 0, smem2 = 0;
    if (t->recipe && t->gen2) {
      const int tables = (t->L + t->Q + t->Q * t->n + t->U) * 4;
      const int per_warp = 32 * (t->U + t->L) * 4;
      warps2 = (200 * 1024 - tables) / per_warp;
      if (warps2 > 8) warps2 = 8;
      smem2 = tables + warps2 * per_warp;
    }
    const bool use2 = warps2 >= 1 && (sched == 3 || (sched == 0 && !blocked_fits(t)));
    if (use2)
      return general2_solve(t, N, d_entries, S, d_starts, alpha, tol, maxit, d_lambda, d_x, d_iters, d_conv, opts, st,
                            warps2, smem2);
    if (sched != 3 && blocked_fits(t))
      return blocked_solve(t, N, d_entries, S, d_starts, alpha, tol, maxit, d_lambda, d_x, d_iters, d_conv, opts, st);
    if (sched == 5) return SSHOPM_EUNSUPPORTED;
  }
  const int block = 128;
  const int smem = general_smem(t, block, true);
  if (smem > 200 * 1024) return SSHOPM_EUNSUPPORTED;
  const int alpha_mode = opts ? opts->alpha_mode : 0;
  if (alpha_mode < 0 || alpha_mode > 3 || (alpha_mode == 1 && !opts->d_alpha)) return SSHOPM_EINVAL;
  void* tab = nullptr;
  cudaError_t e = cudaMallocAsync(&tab, general_table_bytes(t), st);
  if (e != cudaSuccess) return e == cudaErrorMemoryAllocation ? SSHOPM_ENOMEM : cuda_fail(e, "general: malloc");
  GenParams p;
  int rc = general_upload(t, tab, st, &p.cls_idx, &p.cls_mult);
  if (rc != SSHOPM_OK) { cudaFreeAsync(tab, st); return rc; }
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
  p.n = t->n;
  p.U = t->U;
  p.S = S;
  p.alpha = alpha;
  p.tol = tol;
  p.alpha_mode = alpha_mode;
  p.maxit = maxit;
  if (smem > 48 * 1024) cudaFuncSetAttribute(sshopm_general_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  const int sms = device_sms();
  long long grid = N < (long long)sms * 16 ? N : (long long)sms * 16;
  sshopm_general_kernel<<<(int)grid, block, smem, st>>>(p);
  e = cudaGetLastError();
  cudaFreeAsync(tab, st);
  if (e != cudaSuccess) return cuda_fail(e, "general: launch");
  return SSHOPM_OK;
}

int general_apply(const GeneralTables* t, int64_t N, const float* d_entries, const float* d_x, float* d_g, float* d_lam,
                  cudaStream_t st) {
  const int block = 128;
  const int smem = general_smem(t, block, false);
  if (smem > 200 * 1024) return SSHOPM_EUNSUPPORTED;
  void* tab = nullptr;
  cudaError_t e = cudaMallocAsync(&tab, general_table_bytes(t), st);
  if (e != cudaSuccess) return e == cudaErrorMemoryAllocation ? SSHOPM_ENOMEM : cuda_fail(e, "general: malloc");
  GenParams p;
  memset(&p, 0, sizeof(p));
  int rc = general_upload(t, tab, st, &p.cls_idx, &p.cls_mult);
  if (rc != SSHOPM_OK) { cudaFreeAsync(tab, st); return rc; }
  p.entries = d_entries;
  p.N = N;
  p.m = t->m;
  p.n = t->n;
  p.U = t->U;
  if (smem > 48 * 1024) cudaFuncSetAttribute(sshopm_general_apply_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  const int sms = device_sms();
  long long grid = (N + block - 1) / block;
  if (grid > (long long)sms * 16) grid = (long long)sms * 16;
  sshopm_general_apply_kernel<<<(int)grid, block, smem, st>>>(p, d_x, d_g, d_lam);
  e = cudaGetLastError();
  cudaFreeAsync(tab, st);
  if (e != cudaSuccess) return cuda_fail(e, "general: apply launch");
  return SSHOPM_OK;
}

}  // namespace sshopm
