// sshopm_kernels.cuh — sm_100a kernels for batched SS-HOPM (templated on (M, N)).
//
// Paper: Fig. 1 SS-HOPM, Eq. 6 / Eq. 4 kernels,
// loop unrolling per (m, n) (Sec. V-D), data structures
// (Sec. V-C).  Design notes: DESIGN.md "Kernels".
//
// Mapping (differs from the paper's block-per-tensor / thread-per-start):
//   * one lane = one (tensor, start) work item at a time; a persistent grid of
//     warps, each owning a contiguous static range of items (tensor-major, so
//     a warp's consecutive items share a tensor);
//   * the whole iteration lives in registers: per-lane coefficient registers
//     (B-form: coefficient-folded entries, or raw entries), x, lambda_prev, k;
//   * lambda = x . (A x^{M-1}) (Euler identity), so one Eq. 6 evaluation per
//     iteration gives both kernels of Fig. 1;
//   * lanes that stop freeze (their state recomputes bit-identically) and the
//     warp refills them in batches: once >= K lanes are idle it writes their
//     results and hands them the next items of its range (warp ballot + popc,
//     no atomics, no block barriers);
//   * output pairs (g_0, g_1), (g_2, g_3), ... accumulate with packed FFMA2
//     (__ffma2_rn) so the FP32 pipe is saturated at half the issue slots.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>
#include "symm_tables.cuh"

namespace sshopm {

// ---------------------------------------------------------------- helpers --
struct FastDiv {        // n / d for 0 <= n < 2^31, d >= 1 (Granlund-Montgomery)
  uint32_t d, magic, shift;
};
__device__ __forceinline__ uint32_t fast_div(uint32_t n, const FastDiv& f) {
  return (__umulhi(n, f.magic) + n) >> f.shift;
}

template <int M, int N>
struct Shape {
  static constexpr Tables<M, N> T{};
  static constexpr int U = Tables<M, N>::U;
  static constexpr int Q = Tables<M, N>::Q;
  static constexpr int NL = Tables<M, N>::NL;
  static constexpr int NP = N / 2;          // packed output pairs
  static constexpr bool ODD = (N % 2) != 0;
  static constexpr int NX = (N + 1) / 2;    // float2 slots holding x
  // B-form keeps Q*N coefficient-folded entries per lane; raw form keeps U.
  static constexpr bool BFORM = (Q * N <= 64);
  // register budget -> min resident blocks of 256 threads (tuned on B200)
  static constexpr int MINB = BFORM ? (Q * N <= 32 ? 4 : 2) : (U <= 48 ? 2 : 1);
};

// -------------------------------------------------------- coefficient regs --
template <int M, int N, bool BF = Shape<M, N>::BFORM>
struct Coefs;

// B-form: bp[q][p] = ((M-1)!/q!) * (a_{class(q+e_{2p})}, a_{class(q+e_{2p+1})}),
//         bs[q]    = ((M-1)!/q!) * a_{class(q+e_{N-1})} (N odd).
template <int M, int N>
struct Coefs<M, N, true> {
  using S = Shape<M, N>;
  float2 bp[S::Q][S::NP > 0 ? S::NP : 1];
  float bs[S::Q];

  __device__ __forceinline__ void load(const float* __restrict__ e) {
    float a[S::U];
    static_for<S::U>([&](auto c) { a[decltype(c)::value] = __ldg(e + decltype(c)::value); });
    static_for<S::Q>([&](auto qq) {
      constexpr int q = decltype(qq)::value;
      constexpr float cf = (float)S::T.q_coef[q];
      static_for<S::NP>([&](auto pp) {
        constexpr int p = decltype(pp)::value;
        constexpr int c0 = S::T.q_cls[q][2 * p], c1 = S::T.q_cls[q][2 * p + 1];
        bp[q][p] = make_float2(cf * a[c0], cf * a[c1]);
      });
      if constexpr (S::ODD) {
        constexpr int c2 = S::T.q_cls[q][N - 1];
        bs[q] = cf * a[c2];
      }
    });
  }

  // g = A x^{M-1} from the Q monomials mq (coefficients already folded in)
  __device__ __forceinline__ void contract(const float (&mq)[S::Q], float2 (&gp)[S::NP > 0 ? S::NP : 1], float& gs) const {
    static_for<S::NP>([&](auto pp) {
      constexpr int p = decltype(pp)::value;
      gp[p] = __fmul2_rn(bp[0][p], make_float2(mq[0], mq[0]));
    });
    if constexpr (S::ODD) gs = bs[0] * mq[0];
    static_for<S::Q - 1>([&](auto qq) {
      constexpr int q = decltype(qq)::value + 1;
      const float2 mm = make_float2(mq[q], mq[q]);
      static_for<S::NP>([&](auto pp) {
        constexpr int p = decltype(pp)::value;
        gp[p] = __ffma2_rn(bp[q][p], mm, gp[p]);
      });
      if constexpr (S::ODD) gs = fmaf(bs[q], mq[q], gs);
    });
  }
};

// raw form: a[c] = entry of class c; coefficients multiply the monomials.
template <int M, int N>
struct Coefs<M, N, false> {
  using S = Shape<M, N>;
  float a[S::U];

  __device__ __forceinline__ void load(const float* __restrict__ e) {
    static_for<S::U>([&](auto c) { a[decltype(c)::value] = __ldg(e + decltype(c)::value); });
  }

  __device__ __forceinline__ void contract(const float (&mq)[S::Q], float2 (&gp)[S::NP > 0 ? S::NP : 1], float& gs) const {
    float g[N];
    static_for<S::Q>([&](auto qq) {
      constexpr int q = decltype(qq)::value;
      constexpr float cf = (float)S::T.q_coef[q];
      const float m = (cf == 1.0f) ? mq[q] : cf * mq[q];
      static_for<N>([&](auto jj) {
        constexpr int j = decltype(jj)::value;
        constexpr int c = S::T.q_cls[q][j];
        if constexpr (q == 0) g[j] = a[c] * m;
        else g[j] = fmaf(a[c], m, g[j]);
      });
    });
    static_for<S::NP>([&](auto pp) {
      constexpr int p = decltype(pp)::value;
      gp[p] = make_float2(g[2 * p], g[2 * p + 1]);
    });
    if constexpr (S::ODD) gs = g[N - 1];
  }
};

// x stored in float2 slots: x_i = xs[i/2].x or .y
template <int N>
__device__ __forceinline__ float xget(const float2 (&xs)[(N + 1) / 2], int i) {
  return (i & 1) ? xs[i >> 1].y : xs[i >> 1].x;
}

// degree-(M-1) monomials x^q (Tables: lower list up to degree H, then left*right)
template <int M, int N>
__device__ __forceinline__ void monomials(const float2 (&xs)[(N + 1) / 2], float (&mq)[Shape<M, N>::Q]) {
  using S = Shape<M, N>;
  float low[S::NL];
  static_for<S::NL>([&](auto tt) {
    constexpr int t = decltype(tt)::value;
    constexpr int par = S::T.low_parent[t], var = S::T.low_var[t];
    if constexpr (par < 0) low[t] = xget<N>(xs, var);
    else low[t] = low[par] * xget<N>(xs, var);
  });
  static_for<S::Q>([&](auto qq) {
    constexpr int q = decltype(qq)::value;
    constexpr int l = S::T.q_left[q], r = S::T.q_right[q];
    if constexpr (l < 0) mq[q] = low[r];
    else mq[q] = low[l] * low[r];
  });
}

// g = A x^{M-1} (pairs gp, odd tail gs) and lambda = x . g
template <int M, int N>
__device__ __forceinline__ float evaluate(const Coefs<M, N>& cf, const float2 (&xs)[(N + 1) / 2],
                                          float2 (&gp)[Shape<M, N>::NP > 0 ? Shape<M, N>::NP : 1], float& gs) {
  using S = Shape<M, N>;
  float mq[S::Q];
  monomials<M, N>(xs, mq);
  cf.contract(mq, gp, gs);
  float lam;
  if constexpr (S::NP > 0) {
    float2 t = __fmul2_rn(xs[0], gp[0]);
    static_for<S::NP - 1>([&](auto pp) {
      constexpr int p = decltype(pp)::value + 1;
      t = __ffma2_rn(xs[p], gp[p], t);
    });
    lam = t.x + t.y;
    if constexpr (S::ODD) lam = fmaf(xs[S::NX - 1].x, gs, lam);
  } else {
    lam = xs[0].x * gs;
  }
  return lam;
}

// ------------------------------------------------------------ solve kernel --
struct SolveParams {
  const float* entries;      // [N][U]
  const float* starts;       // [S][n] (raw; normalised in the kernel)
  float* out_lambda;         // [N][S]
  float* out_x;              // [N][S][n]
  int32_t* out_iters;        // [N][S]
  uint8_t* out_conv;         // [N][S]
  unsigned long long* total_iters;  // optional
  long long total_items;     // N*S
  long long items_per_warp;  // contiguous range per warp (< 2^30)
  int S;
  FastDiv divS;
  float alpha, tol;
  int maxit;
  int refill_k;              // refill threshold
  int starts_in_smem;        // 1: normalised starts cached in shared memory
};

__device__ __forceinline__ uint32_t lanemask_lt() {
  uint32_t r;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(r));
  return r;
}

template <int M, int N, bool NEG>
__global__ void __launch_bounds__(256, Shape<M, N>::MINB)
sshopm_solve_kernel(const SolveParams p) {
  using S = Shape<M, N>;
  extern __shared__ float s_starts[];   // [S][n] normalised starts (if starts_in_smem)

  if (p.starts_in_smem) {
    for (int s = threadIdx.x; s < p.S; s += blockDim.x) {
      float v[N];
      float nn = 0.f;
#pragma unroll
      for (int j = 0; j < N; ++j) { v[j] = __ldg(p.starts + (size_t)s * N + j); nn = fmaf(v[j], v[j], nn); }
      const float r = nn > 0.f ? rsqrtf(nn) : 0.f;
#pragma unroll
      for (int j = 0; j < N; ++j) s_starts[s * N + j] = v[j] * r;
    }
    __syncthreads();
  }

  const int lane = threadIdx.x & 31;
  const long long gwarp = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const long long base = gwarp * p.items_per_warp;
  if (base >= p.total_items) return;
  const long long span = min(p.items_per_warp, p.total_items - base);
  const uint32_t end = (uint32_t)span;
  const long long base_v = base / p.S;                 // tensor of the range's first item
  const uint32_t base_s = (uint32_t)(base - base_v * p.S);
  const uint32_t ltmask = lanemask_lt();

  Coefs<M, N> cf;
  float2 xs[S::NX];
#pragma unroll
  for (int i = 0; i < S::NX; ++i) xs[i] = make_float2(0.f, 0.f);
  float lamp = 0.f, lam = 0.f;
  int k = 0;
  bool has = false, stop = true, conv = false;
  uint32_t l = 0, next = 0;
  unsigned long long it_sum = 0;
  const float alpha = NEG ? -p.alpha : p.alpha;   // xhat = sgn*(g + alpha x) = sgn*g + (sgn*alpha) x

  for (;;) {
    // ---------------- refill (warp-uniform branch) ----------------
    const uint32_t smask = __ballot_sync(0xffffffffu, stop);
    const int cnt = __popc(smask);
    if ((cnt >= p.refill_k && next < end) || smask == 0xffffffffu) {
      if (stop && has) {
        const long long item = base + l;
        p.out_lambda[item] = lam;
#pragma unroll
        for (int j = 0; j < N; ++j) p.out_x[item * N + j] = xget<N>(xs, j);
        p.out_iters[item] = k;
        p.out_conv[item] = conv ? 1 : 0;
        it_sum += (unsigned long long)k;
      }
      const uint32_t nl = next + (uint32_t)__popc(smask & ltmask);
      if (stop) {
        has = nl < end;
        if (has) {
          l = nl;
          const uint32_t t = base_s + l;
          const uint32_t vq = fast_div(t, p.divS);
          const uint32_t s = t - vq * (uint32_t)p.S;
          cf.load(p.entries + (size_t)(base_v + vq) * S::U);
          float v[N];
          if (p.starts_in_smem) {
#pragma unroll
            for (int j = 0; j < N; ++j) v[j] = s_starts[s * N + j];
          } else {
            float nn = 0.f;
#pragma unroll
            for (int j = 0; j < N; ++j) { v[j] = __ldg(p.starts + (size_t)s * N + j); nn = fmaf(v[j], v[j], nn); }
            const float r = nn > 0.f ? rsqrtf(nn) : 0.f;
#pragma unroll
            for (int j = 0; j < N; ++j) v[j] *= r;
          }
#pragma unroll
          for (int i = 0; i < S::NX; ++i) xs[i] = make_float2(v[2 * i], (2 * i + 1 < N) ? v[2 * i + 1] : 0.f);
          k = 0;
          lamp = __int_as_float(0x7fffffff);   // NaN: the first test never fires (reading R2)
        }
      }
      next += (uint32_t)cnt;
      if (__ballot_sync(0xffffffffu, has) == 0u) break;
    }

    // ---------------- one SS-HOPM step (Fig. 1) ----------------
    float2 gp[S::NP > 0 ? S::NP : 1];
    float gs = 0.f;
    lam = evaluate<M, N>(cf, xs, gp, gs);                       // g = A x_k^{m-1}, lam_k = x_k . g
    conv = fabsf(lam - lamp) <= p.tol * fmaxf(1.0f, fabsf(lam)); // R2 (NaN lamp -> false)
    // xhat = +-(g + alpha x)   (Fig. 1 lines 2-5, R5)
    float2 hp[S::NX];
    static_for<S::NP>([&](auto qq) {
      constexpr int i = decltype(qq)::value;
      const float2 g = NEG ? make_float2(-gp[i].x, -gp[i].y) : gp[i];
      hp[i] = __ffma2_rn(make_float2(alpha, alpha), xs[i], g);
    });
    if constexpr (S::ODD) hp[S::NX - 1] = make_float2(fmaf(alpha, xs[S::NX - 1].x, NEG ? -gs : gs), 0.f);
    float nn;
    {
      float2 t = __fmul2_rn(hp[0], hp[0]);
      static_for<S::NX - 1>([&](auto qq) {
        constexpr int i = decltype(qq)::value + 1;
        t = __ffma2_rn(hp[i], hp[i], t);
      });
      nn = t.x + t.y;
    }
    const bool deg = !(nn > 0.f);                               // R6
    stop = !has || conv || k >= p.maxit || deg;
    if (!stop) {
      const float r = rsqrtf(nn);                               // line 7: x = xhat / ||xhat||
      const float2 rr = make_float2(r, r);
#pragma unroll
      for (int i = 0; i < S::NX; ++i) xs[i] = __fmul2_rn(hp[i], rr);
      lamp = lam;
      ++k;
    }
  }

  if (p.total_iters) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) it_sum += __shfl_xor_sync(0xffffffffu, it_sum, o);
    if (lane == 0) atomicAdd(p.total_iters, it_sum);
  }
}

// ------------------------------------------------------------ apply kernel --
template <int M, int N>
__global__ void __launch_bounds__(256)
sshopm_apply_kernel(long long n_items, const float* __restrict__ entries, const float* __restrict__ x,
                    float* __restrict__ out_g, float* __restrict__ out_lam) {
  using S = Shape<M, N>;
  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n_items; i += (long long)gridDim.x * blockDim.x) {
    Coefs<M, N> cf;
    cf.load(entries + (size_t)i * S::U);
    float2 xs[S::NX];
#pragma unroll
    for (int t = 0; t < S::NX; ++t)
      xs[t] = make_float2(__ldg(x + i * N + 2 * t), (2 * t + 1 < N) ? __ldg(x + i * N + 2 * t + 1) : 0.f);
    float2 gp[S::NP > 0 ? S::NP : 1];
    float gs = 0.f;
    const float lam = evaluate<M, N>(cf, xs, gp, gs);
    static_for<S::NP>([&](auto pp) {
      constexpr int q = decltype(pp)::value;
      out_g[i * N + 2 * q] = gp[q].x;
      out_g[i * N + 2 * q + 1] = gp[q].y;
    });
    if constexpr (S::ODD) out_g[i * N + N - 1] = gs;
    out_lam[i] = lam;
  }
}

}  // namespace sshopm
