// sshopm_kernels.cuh — sm_100a kernels for batched SS-HOPM (templated on (M, N)).
//
// Paper: Fig. 1 SS-HOPM, Eq. 6 / Eq. 4 kernels,
// loop unrolling per (m, n) (Sec. V-D), data structures
// (Sec. V-C), precomputed coefficient tables shared by all
// same-size tensors.  Design notes: DESIGN.md "Kernels".
//
// Mapping (differs from the paper's block-per-tensor / thread-per-start):
//   * a pack kernel rewrites each tensor's U entries once into a 16-byte
//     aligned row of coefficient-folded words (B-form) or padded raw entries;
//   * the solve kernel is a persistent grid of warps; one lane holds one
//     (tensor, start) item at a time; warps claim chunks of whole tensors
//     from a global atomic counter (dynamic load balance);
//   * the whole iteration lives in registers: coefficients (LDG.128 from the
//     packed row at refill), x, lambda_prev, k;
//   * lambda = x . (A x^{M-1}) (Euler identity), so one Eq. 6 evaluation per
//     iteration provides both kernels of Fig. 1;
//   * lanes that stop freeze (their state recomputes bit-identically) and the
//     warp refills them in batches once >= K lanes are idle (ballot + popc);
//   * output pairs (g_0, g_1), ... accumulate with packed FFMA2 (__ffma2_rn),
//     odd last output in q-pairs, so the FP32 pipe is fed at half the issue slots.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>
#ifdef SSHOPM_BOUNDS_CHECK
#include <cassert>
#define SSHOPM_CHECK(c) assert(c)   // debug builds (tools/gpu_bounds.sh): index bounds of the refill paths
#else
#define SSHOPM_CHECK(c) ((void)0)
#endif
#include <type_traits>
#include "symm_tables.cuh"
#include "sshopm_dedup.cuh"

namespace sshopm {

// ---------------------------------------------------------------- helpers --
struct FastDiv {        // n / d for 0 <= n < 2^31, d >= 1 (Granlund-Montgomery)
  uint32_t d, magic, shift;
};
__device__ __forceinline__ uint32_t fast_div(uint32_t n, const FastDiv& f) {
  return (__umulhi(n, f.magic) + n) >> f.shift;
}
__device__ __forceinline__ float rsqrt_ftz(float v) {
  float r;
  asm("rsqrt.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(v));
  return r;
}
__device__ __forceinline__ float2 f2(float a, float b) { return make_float2(a, b); }
__device__ __forceinline__ float2 bc(float a) { return make_float2(a, a); }
__device__ __forceinline__ float4 ldg4(const float4* p) { return __ldg(p); }
// Predicated global accesses as single predicated instructions (no divergent
// branch / BSSY region around the refill's stores and loads).
__device__ __forceinline__ void pst(bool p, float* a, float v) {
  asm volatile("{\n .reg .pred q;\n setp.ne.b32 q, %0, 0;\n @q st.global.f32 [%1], %2;\n}"
               :: "r"((int)p), "l"(a), "f"(v) : "memory");
}
__device__ __forceinline__ void pst(bool p, int32_t* a, int32_t v) {
  asm volatile("{\n .reg .pred q;\n setp.ne.b32 q, %0, 0;\n @q st.global.b32 [%1], %2;\n}"
               :: "r"((int)p), "l"(a), "r"(v) : "memory");
}
__device__ __forceinline__ void pst(bool p, uint8_t* a, uint32_t v) {
  asm volatile("{\n .reg .pred q;\n .reg .b16 t;\n setp.ne.b32 q, %0, 0;\n cvt.u16.u32 t, %2;\n @q st.global.b8 [%1], t;\n}"
               :: "r"((int)p), "l"(a), "r"(v) : "memory");
}
__device__ __forceinline__ void pld4(bool p, const float4* a, float4& v) {
  asm("{\n .reg .pred q;\n setp.ne.b32 q, %4, 0;\n @q ld.global.nc.v4.f32 {%0, %1, %2, %3}, [%5];\n}"
      : "+f"(v.x), "+f"(v.y), "+f"(v.z), "+f"(v.w) : "r"((int)p), "l"(a));
}
__device__ __forceinline__ unsigned int atom_add1(unsigned int* a) {   // plain (not warp-aggregated) atomic
  unsigned int r;
  asm volatile("atom.global.add.u32 %0, [%1], 1;" : "=r"(r) : "l"(a) : "memory");
  return r;
}

constexpr int round4(int v) { return (v + 3) / 4 * 4; }
// SS-HOPM steps per refill check (trip).  More steps amortise the ballot and
// branch over more arithmetic but let stopped lanes idle longer; measured on
// B200 (C2, (4,3)): 1 step 4.90 ms, 2 steps 4.60, 3 steps 4.45, 4 steps 4.58
// (best refill threshold each).  Shapes with costlier steps keep 2.
// Round 2, (4,3) with the scalar-tail step: 4 steps per trip (C2 4.14 ms at K = 10; 3 steps 4.22 at K = 8,
// 5 steps 4.34, 6 steps 4.34: profiles/r2/solve_variants_s6.jsonl).
template <int M, int N>
constexpr int steps_per_trip() {
#ifdef SSHOPM_STEPS
  return SSHOPM_STEPS;
#else
  // n = 3, m >= 6 (Horner step): 3 steps per trip (C3 10.75 -> 10.71 ms, C4a 5.37 -> 5.32 ms at K = 6)
  return (M == 4 && N == 3) ? 4 : ((binom(M + N - 2, M - 1) * N <= 30 || (N == 3 && M >= 6)) ? 3 : 2);
#endif
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
  static constexpr int QP = Q / 2;          // q-pairs of the odd output (leftover q handled scalar)
  // B-form keeps Q*N coefficient-folded entries per lane; raw form keeps U.
#ifndef SSHOPM_BFORM_MAX
#define SSHOPM_BFORM_MAX 64
#endif
#ifndef SSHOPM_RAW_MINB_SMALL
#define SSHOPM_RAW_MINB_SMALL 3   // raw rows of <= 48 words ((8,3)): 80 registers, 3 CTAs per SM with the Horner step
                                  // (C4a 5.32 -> 5.27 ms, no spills; (6,3) at 3 CTAs spills and is slower: 11.42 ms)
#endif
  static constexpr bool BFORM = (Q * N <= SSHOPM_BFORM_MAX);   // (8,3) B-form (108 words, 186 regs) measured slower: 7.5 vs 6.3 ms
  static constexpr int PW_B = Q * NP * 2 + (ODD ? 2 * QP + (Q % 2) : 0);
  static constexpr int PW = round4(BFORM ? PW_B : U);   // packed words per tensor
#ifndef SSHOPM_BFORM32_MINB
#define SSHOPM_BFORM32_MINB 4
#endif
#ifndef SSHOPM_BFORM64_MINB
#define SSHOPM_BFORM64_MINB 2
#endif
  static constexpr int MINB = BFORM ? (Q * N <= 32 ? SSHOPM_BFORM32_MINB : (Q * N <= 64 ? SSHOPM_BFORM64_MINB : 1)) : (U <= 48 ? SSHOPM_RAW_MINB_SMALL : 1);
  // threads per CTA of the non-fused schedule-1 solve kernel (knob): 128-thread CTAs for n = 3, m >= 6
  // B-form rows fit a fifth CTA at <= 96 registers (20 instead of 16 warps per SM) but measured no faster
  // at C3 (10.78 vs 10.70 ms), so the default stays 256
#ifndef SSHOPM_TPB_BFORM63
#define SSHOPM_TPB_BFORM63 256
#endif
  static constexpr int TPB = (N == 3 && M >= 6 && BFORM && Q * N > 32) ? SSHOPM_TPB_BFORM63 : 256;
  static constexpr int MINB_T = TPB == 256 ? MINB : (65536 / (TPB * 96));   // <= 96 registers at 128 threads
};

// State layout of x (see xget below): slot of component i.
#ifndef SSHOPM_43_FORM
#define SSHOPM_43_FORM 2   // (4,3) step: 2 = (x0,x1),(x2,x1) layout, 8 FMUL2 monomials, scalar FFMA contraction (default:
                           // C2 4.26 ms); 1 = natural layout, (g0,g1) FFMA2 + g2 FFMA (4.44); 0 = X02 layout, scalar (4.43);
                           // 3 = form 2 without the (x1,x2) moves (4.26); 4 = all scalar (4.79).  DESIGN.md "Round 2".
#endif
template <int M, int N>
struct X02 { static constexpr bool v = (M == 4 && N == 3 && SSHOPM_43_FORM == 0); };
template <int M, int N>
struct N43 { static constexpr bool v = (M == 4 && N == 3 && SSHOPM_43_FORM == 1); };
// form 4: natural layout, every FP32 operation scalar (FMUL / FFMA / FADD only: no packed FP32 in the step)
template <int M, int N>
struct S43 { static constexpr bool v = (M == 4 && N == 3 && SSHOPM_43_FORM == 4); };
// form 2: the round-1 layout, x held as (x0, x1), (x2, x1) (slot 3 duplicates x1), monomials as 8 FMUL2
template <int M, int N>
struct X21 { static constexpr bool v = (M == 4 && N == 3 && (SSHOPM_43_FORM == 2 || SSHOPM_43_FORM == 3 || SSHOPM_43_FORM == 5)); };
// form 5: the form-2 layout, g by Horner in x0 over shared (x1, x2) monomials, (g0, g1) as FFMA2, g2 scalar
template <int M, int N>
struct H43 { static constexpr bool v = (M == 4 && N == 3 && SSHOPM_43_FORM == 5); };
#ifndef SSHOPM_GEN_TAIL
#define SSHOPM_GEN_TAIL 1   // other n = 3 shapes with rows of <= 64 words: scalar lambda / ||xhat||^2 / update
                            // (C3 (6,3) solve 11.85 -> 11.60 ms; (8,3) is 0.9% slower with it, so excluded)
#endif
#ifndef SSHOPM_HORNER3
#define SSHOPM_HORNER3 1   // n = 3, m >= 6 shapes evaluate Eq. 6 by Horner in x0 (horner3): C3 11.61 -> 10.75 ms,
                           // C4a 5.87 -> 5.37 ms (profiles/r2/horner3.md); (4,3) keeps form 2 (form 5 measured slower);
                           // (5,3) keeps the monomial form (one chaotic stress lane left the parity contract)
#endif
#ifndef SSHOPM_X21_TAIL
#define SSHOPM_X21_TAIL 1   // 1 (default): forms 2/3 with lambda, ||xhat||^2 and the update in scalar FP32 (C2 4.26 -> 4.22 ms)
#endif
template <int M, int N>
__host__ __device__ constexpr int xslot(int i) {
  return X02<M, N>::v ? (i == 0 ? 0 : (i == 1 ? 2 : 1)) : i;
}

// ---------------------------------------------------------- pack kernel ----
// B-form row:  [ (B_{q,2p}, B_{q,2p+1}) for q, p ] [ (B_{2t,N-1}, B_{2t+1,N-1}) for t < QP ] [B_{Q-1,N-1} if Q odd] [0 pad]
// with B_{q,j} = ((M-1)!/q!) * a_{class(q + e_j)}   (Eq. 6 regrouped by monomial)
// raw row:     [ a_0 .. a_{U-1} ] [0 pad]
template <int M, int N>
__global__ void __launch_bounds__(256)
sshopm_pack_kernel(long long n_tensors, const float* __restrict__ entries, float4* __restrict__ packed,
                   unsigned int* __restrict__ counter, int n_starts, const float* __restrict__ starts,
                   float* __restrict__ starts_n, int alpha_mode, const float* __restrict__ alpha_in,
                   float* __restrict__ alpha_t) {
  using S = Shape<M, N>;
  if (counter && blockIdx.x == 0 && threadIdx.x == 0) { counter[0] = 0u; counter[1] = 0u; }   // solve's chunk / overflow counters
  // normalised starts x_0 = s / ||s|| in FP32 (reading R7), rows padded to SST floats, components in the
  // kernels' state slot order (xslot)
  constexpr int SST = round4(N);
  for (int s = blockIdx.x * blockDim.x + threadIdx.x; s < n_starts; s += gridDim.x * blockDim.x) {
    float v[N];
    float nn = 0.f;
#pragma unroll
    for (int j = 0; j < N; ++j) { v[j] = starts[(size_t)s * N + j]; nn = fmaf(v[j], v[j], nn); }
    const float r = nn > 0.f ? rsqrtf(nn) : 0.f;
#pragma unroll
    for (int j = 0; j < SST; ++j) starts_n[(size_t)s * SST + j] = 0.f;
#pragma unroll
    for (int j = 0; j < N; ++j) starts_n[(size_t)s * SST + xslot<M, N>(j)] = v[j] * r;   // state slot order
    if constexpr (X21<M, N>::v) starts_n[(size_t)s * SST + 3] = v[1] * r;                 // (x2, x1) pair
  }
  // one tensor: coefficient-folded words w from its entries a, and its shift (alpha modes 1-3)
  auto row = [&](long long t, const float (&a)[S::U], float (&w)[S::PW]) {
#pragma unroll
    for (int i = 0; i < S::PW; ++i) w[i] = 0.f;
    if constexpr (S::BFORM) {
      static_for<S::Q>([&](auto qq) {
        constexpr int q = decltype(qq)::value;
        constexpr float cf = (float)S::T.q_coef[q];
        static_for<S::NP>([&](auto pp) {
          constexpr int p = decltype(pp)::value;
          constexpr int c0 = S::T.q_cls[q][2 * p], c1 = S::T.q_cls[q][2 * p + 1];
          w[(q * S::NP + p) * 2 + 0] = cf * a[c0];
          w[(q * S::NP + p) * 2 + 1] = cf * a[c1];
        });
        if constexpr (S::ODD) {
          constexpr int c2 = S::T.q_cls[q][N - 1];
          w[S::Q * S::NP * 2 + q] = cf * a[c2];
        }
      });
    } else {
#pragma unroll
      for (int c = 0; c < S::U; ++c) w[c] = a[c];
    }
    if (alpha_mode == 1) {
      alpha_t[t] = alpha_in[t];
    } else if (alpha_mode >= 2) {
      // convexity shift bound beta(A) <= (m-1) sum_{i_1..i_m} |a| = (m-1) sum_c (m!/k!) |a_c| (R17)
      float b = 0.f;
      static_for<S::U>([&](auto cc) {
        constexpr int c = decltype(cc)::value;
        constexpr float mult = (float)S::T.cls_mult[c];
        b = fmaf(mult, fabsf(a[c]), b);
      });
      b *= (float)(M - 1);
      alpha_t[t] = (alpha_mode == 2) ? b : -b;
    }
  };
  // Small rows: a warp packs 32 consecutive tensors through shared memory, so both the entry reads
  // and the row writes are contiguous, fully coalesced warp accesses (the thread-per-tensor form
  // reads at a U-word and writes at a PW-word stride: 3.5 TB/s at C2).
  constexpr int TW = (S::U > S::PW + 1) ? S::U : S::PW + 1;
  constexpr bool TILE = 8 * 32 * TW * 4 <= 40 * 1024;
  if constexpr (TILE) {
    __shared__ float tsm[8][32 * TW];
    float* my = tsm[threadIdx.x >> 5];
    const int lane = threadIdx.x & 31;
    const long long nw = (long long)gridDim.x * (blockDim.x >> 5);
    for (long long tile = (long long)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); tile * 32 < n_tensors;
         tile += nw) {
      const long long t0 = tile * 32;
      const int cnt = (int)((n_tensors - t0) < 32 ? (n_tensors - t0) : 32);
      const float* src = entries + t0 * S::U;
      for (int i = lane; i < cnt * S::U; i += 32) my[i] = __ldg(src + i);
      __syncwarp();
      float a[S::U], w[S::PW];
#pragma unroll
      for (int c = 0; c < S::U; ++c) a[c] = (lane < cnt) ? my[lane * S::U + c] : 0.f;
      __syncwarp();
      if (lane < cnt) {
        row(t0 + lane, a, w);
#pragma unroll
        for (int i = 0; i < S::PW; ++i) my[lane * (S::PW + 1) + i] = w[i];   // padded stride: no bank conflicts
      }
      __syncwarp();
      float4* dst = packed + t0 * (S::PW / 4);
      for (int f = lane; f < cnt * (S::PW / 4); f += 32) {
        const int r = (4 * f) / S::PW, c = (4 * f) % S::PW;
        const float* q = my + r * (S::PW + 1) + c;
        dst[f] = make_float4(q[0], q[1], q[2], q[3]);
      }
      __syncwarp();
    }
  } else {
    for (long long t = (long long)blockIdx.x * blockDim.x + threadIdx.x; t < n_tensors;
         t += (long long)gridDim.x * blockDim.x) {
      float a[S::U], w[S::PW];
      static_for<S::U>([&](auto c) { a[decltype(c)::value] = __ldg(entries + t * S::U + decltype(c)::value); });
      row(t, a, w);
      float4* dst = packed + t * (S::PW / 4);
#pragma unroll
      for (int i = 0; i < S::PW / 4; ++i) dst[i] = make_float4(w[4 * i], w[4 * i + 1], w[4 * i + 2], w[4 * i + 3]);
    }
  }
}

// -------------------------------------------------------- coefficient regs --
template <int M, int N, bool BF = Shape<M, N>::BFORM>
struct Coefs {
  using S = Shape<M, N>;
  float4 w[S::PW / 4];

  __device__ __forceinline__ void load(const float4* __restrict__ src) {
#pragma unroll
    for (int i = 0; i < S::PW / 4; ++i) w[i] = ldg4(src + i);
  }
  __device__ __forceinline__ void load_if(bool p, const float4* __restrict__ src) {
#pragma unroll
    for (int i = 0; i < S::PW / 4; ++i) pld4(p, src + i, w[i]);
  }
  template <int I>
  __device__ __forceinline__ float word() const {
    constexpr int v = I / 4, c = I % 4;
    if constexpr (c == 0) return w[v].x;
    else if constexpr (c == 1) return w[v].y;
    else if constexpr (c == 2) return w[v].z;
    else return w[v].w;
  }
  template <int I>   // aligned pair of words (I even)
  __device__ __forceinline__ float2 pair() const {
    constexpr int v = I / 4;
    if constexpr ((I % 4) == 0) return f2(w[v].x, w[v].y);
    else return f2(w[v].z, w[v].w);
  }

  // g = A x^{M-1} from the Q monomials mq.
  __device__ __forceinline__ void contract(const float (&mq)[S::Q], float2 (&gp)[S::NP > 0 ? S::NP : 1], float& gs) const {
#ifndef SSHOPM_PAIRED_CONTRACT
    // small rows: scalar FFMA, q outer / j inner (the monomial is the operand every output of a q shares,
    // reused from the operand cache); measured faster than the FFMA2 forms below on B200 for (4,3)
    // (C2 solve 4.43 -> 4.32 ms, C2a 7.41 -> 7.25) but slower for (6,3) (C3 11.98 -> 12.14):
    // profiles/r1/solve_variants.txt.  Outputs g_j as independent chains; the odd last output sequential.
    if constexpr (BF && S::Q * N <= 30) {
      constexpr int base = S::Q * S::NP * 2;
      float g[N];
      static_for<S::Q>([&](auto qq) {
        constexpr int q = decltype(qq)::value;
        static_for<S::NP>([&](auto pp) {
          constexpr int p = decltype(pp)::value;
          if constexpr (q == 0) {
            g[2 * p] = word<(q * S::NP + p) * 2>() * mq[q];
            g[2 * p + 1] = word<(q * S::NP + p) * 2 + 1>() * mq[q];
          } else {
            g[2 * p] = fmaf(word<(q * S::NP + p) * 2>(), mq[q], g[2 * p]);
            g[2 * p + 1] = fmaf(word<(q * S::NP + p) * 2 + 1>(), mq[q], g[2 * p + 1]);
          }
        });
        if constexpr (S::ODD) {
          if constexpr (q == 0) g[N - 1] = word<base>() * mq[0];
          else g[N - 1] = fmaf(word<base + q>(), mq[q], g[N - 1]);
        }
      });
      static_for<S::NP>([&](auto pp) {
        constexpr int p = decltype(pp)::value;
        gp[p] = f2(g[2 * p], g[2 * p + 1]);
      });
      if constexpr (S::ODD) gs = g[N - 1];
      return;
    }
#endif
    if constexpr (BF) {
      static_for<S::NP>([&](auto pp) {
        constexpr int p = decltype(pp)::value;
        gp[p] = __fmul2_rn(pair<2 * p>(), bc(mq[0]));
      });
      static_for<S::Q - 1>([&](auto qq) {
        constexpr int q = decltype(qq)::value + 1;
        static_for<S::NP>([&](auto pp) {
          constexpr int p = decltype(pp)::value;
          gp[p] = __ffma2_rn(pair<(q * S::NP + p) * 2>(), bc(mq[q]), gp[p]);
        });
      });
      if constexpr (S::ODD) {
        constexpr int base = S::Q * S::NP * 2;
        if constexpr (S::QP > 0) {
          float2 h = __fmul2_rn(pair<base>(), f2(mq[0], mq[1]));
          static_for<S::QP - 1>([&](auto tt) {
            constexpr int t = decltype(tt)::value + 1;
            h = __ffma2_rn(pair<base + 2 * t>(), f2(mq[2 * t], mq[2 * t + 1]), h);
          });
          gs = h.x + h.y;
          if constexpr (S::Q % 2) gs = fmaf(word<base + S::Q - 1>(), mq[S::Q - 1], gs);
        } else {
          gs = word<base>() * mq[0];
        }
      }
    } else {
      float g[N];
      static_for<S::Q>([&](auto qq) {
        constexpr int q = decltype(qq)::value;
        constexpr float cf = (float)S::T.q_coef[q];
        const float m = (cf == 1.0f) ? mq[q] : cf * mq[q];
        static_for<N>([&](auto jj) {
          constexpr int j = decltype(jj)::value;
          constexpr int c = S::T.q_cls[q][j];
          if constexpr (q == 0) g[j] = word<c>() * m;
          else g[j] = fmaf(word<c>(), m, g[j]);
        });
      });
      static_for<S::NP>([&](auto pp) {
        constexpr int p = decltype(pp)::value;
        gp[p] = f2(g[2 * p], g[2 * p + 1]);
      });
      if constexpr (S::ODD) gs = g[N - 1];
    }
  }
};

// State layout.  The N components of x live in the float2 slots xs[NX]:
// generic shapes keep x_i in slot i (xs[i/2].x / .y); (4,3) keeps (x0, x2) in
// xs[0] and x1 in xs[1].x ("X02"), so its degree-2/3 monomials are 7 FMUL2 +
// 2 FMUL with no layout moves and the update is one FMUL2 + one FMUL
// (tools/sassmodel: 75 instead of 88 modeled cycles per step on B200).  The
// pack kernel writes the normalised starts in this slot order.
template <int M, int N>
__device__ __forceinline__ float xget(const float2 (&xs)[(N + 1) / 2], int i) {
  const int s = xslot<M, N>(i);
  return (s & 1) ? xs[s >> 1].y : xs[s >> 1].x;
}

// degree-(M-1) monomials x^q (lower list up to degree H, then left * right)
template <int M, int N>
__device__ __forceinline__ void monomials(const float2 (&xs)[(N + 1) / 2], float (&mq)[Shape<M, N>::Q]) {
  using S = Shape<M, N>;
  float low[S::NL];
  static_for<S::NL>([&](auto tt) {
    constexpr int t = decltype(tt)::value;
    constexpr int par = S::T.low_parent[t], var = S::T.low_var[t];
    if constexpr (par < 0) low[t] = xget<M, N>(xs, var);
    else low[t] = low[par] * xget<M, N>(xs, var);
  });
  static_for<S::Q>([&](auto qq) {
    constexpr int q = decltype(qq)::value;
    constexpr int l = S::T.q_left[q], r = S::T.q_right[q];
    if constexpr (l < 0) mq[q] = low[r];
    else mq[q] = low[l] * low[r];
  });
}

// (4,3): the paper's hand-unrolled case (Sec. V-D).  With x in the X02
// layout the ten degree-3 monomials (lex order q = 000 001 002 011 012 022 111
// 112 122 222) come from 7 FMUL2 + 2 FMUL; Eq. 6 is scalar FFMA, q outer / j
// inner (the monomial is the operand the three outputs share, so it is read
// once); lambda = x . g as a scalar FMA chain (Definition 2).
__device__ __forceinline__ float eval43(const Coefs<4, 3>& cf, const float2 (&xs)[2], float& g0, float& g1, float& g2) {
  const float2 xq = xs[0];                    // (x0, x2)
  const float x0 = xq.x, x2 = xq.y, x1 = xs[1].x;
  const float2 a = __fmul2_rn(bc(x0), xq);    // x0x0, x0x2
  const float2 b = __fmul2_rn(bc(x1), xq);    // x0x1, x1x2
  const float2 c = f2(x1 * x1, x2 * x2);      // x1x1, x2x2
  const float2 m0 = __fmul2_rn(bc(x0), a);    // q0 = 000, q2 = 002
  const float2 m1 = __fmul2_rn(bc(x1), a);    // q1 = 001, q4 = 012
  const float2 m2 = __fmul2_rn(bc(x1), b);    // q3 = 011, q7 = 112
  const float2 m3 = __fmul2_rn(bc(c.y), xq);  // q5 = 022, q9 = 222
  const float2 m4 = __fmul2_rn(bc(x1), c);    // q6 = 111, q8 = 122
  const float mq[10] = {m0.x, m1.x, m0.y, m2.x, m1.y, m3.x, m4.x, m2.y, m4.y, m3.y};
  // B-form words: (B_{q,0}, B_{q,1}) at 2q, B_{q,2} at 20 + q (Shape<4,3>: NP = 1, base = Q * NP * 2)
  g0 = cf.template word<0>() * mq[0];
  g1 = cf.template word<1>() * mq[0];
  g2 = cf.template word<20>() * mq[0];
  static_for<9>([&](auto qq) {
    constexpr int q = decltype(qq)::value + 1;
    g0 = fmaf(cf.template word<2 * q>(), mq[q], g0);
    g1 = fmaf(cf.template word<2 * q + 1>(), mq[q], g1);
    g2 = fmaf(cf.template word<20 + q>(), mq[q], g2);
  });
  return fmaf(x2, g2, fmaf(x1, g1, x0 * g0));
}

#ifndef SSHOPM_MONO_MIX
#define SSHOPM_MONO_MIX 0   // form 2 monomials: 0 = 8 FMUL2; 1 = 3 FMUL2 (degree 2) + 10 FMUL; 2 = 6 FMUL + 5 FMUL2
#endif
#if SSHOPM_43_FORM == 2 && !defined(SSHOPM_SCALAR_MONO) && SSHOPM_MONO_MIX == 1
template <>
__device__ __forceinline__ void monomials<4, 3>(const float2 (&xs)[2], float (&mq)[10]) {
  const float2 x01 = xs[0], x21 = xs[1];
  const float x0 = x01.x, x1 = x01.y, x2 = x21.x;
  const float2 s0 = __fmul2_rn(bc(x0), x01);      // (x0x0, x0x1)
  const float2 s1 = __fmul2_rn(x01, x21);         // (x0x2, x1x1)
  const float2 s2 = __fmul2_rn(bc(x2), x21);      // (x2x2, x2x1)
  mq[0] = x0 * s0.x; mq[1] = x0 * s0.y; mq[2] = x0 * s1.x; mq[3] = x0 * s1.y; mq[4] = x0 * s2.y;
  mq[5] = x0 * s2.x; mq[6] = x1 * s1.y; mq[7] = x2 * s1.y; mq[8] = x1 * s2.x; mq[9] = x2 * s2.x;
}
#elif SSHOPM_43_FORM == 2 && !defined(SSHOPM_SCALAR_MONO) && SSHOPM_MONO_MIX == 2
template <>
__device__ __forceinline__ void monomials<4, 3>(const float2 (&xs)[2], float (&mq)[10]) {
  const float x0 = xs[0].x, x1 = xs[0].y, x2 = xs[1].x;
  const float2 d0 = f2(x0 * x0, x0 * x1), d1 = f2(x0 * x2, x1 * x1), d2 = f2(x1 * x2, x2 * x2);
  const float2 m01 = __fmul2_rn(bc(x0), d0);      // 000 001
  const float2 m23 = __fmul2_rn(bc(x0), d1);      // 002 011
  const float2 m45 = __fmul2_rn(bc(x0), d2);      // 012 022
  const float2 m67 = __fmul2_rn(bc(x1), f2(d1.y, d2.x));   // 111 112
  const float2 m89 = __fmul2_rn(bc(x2), d2);      // 122 222
  mq[0] = m01.x; mq[1] = m01.y; mq[2] = m23.x; mq[3] = m23.y; mq[4] = m45.x;
  mq[5] = m45.y; mq[6] = m67.x; mq[7] = m67.y; mq[8] = m89.x; mq[9] = m89.y;
}
#elif SSHOPM_43_FORM == 2 && !defined(SSHOPM_SCALAR_MONO)
template <>
__device__ __forceinline__ void monomials<4, 3>(const float2 (&xs)[2], float (&mq)[10]) {
  const float2 x01 = xs[0], x21 = xs[1];
  const float2 x12 = f2(x21.y, x21.x);
  const float2 s0 = __fmul2_rn(bc(x01.x), x01);   // (x0x0, x0x1)
  const float2 s1 = __fmul2_rn(x01, x21);         // (x0x2, x1x1)
  const float2 s2 = __fmul2_rn(bc(x21.x), x12);   // (x2x1, x2x2)
  const float2 m01 = __fmul2_rn(bc(x01.x), s0);   // 000 001
  const float2 m23 = __fmul2_rn(bc(x01.x), s1);   // 002 011
  const float2 m45 = __fmul2_rn(bc(x01.x), s2);   // 012 022
  const float2 m67 = __fmul2_rn(bc(s1.y), x12);   // 111 112
  const float2 m89 = __fmul2_rn(bc(s2.y), x12);   // 122 222
  mq[0] = m01.x; mq[1] = m01.y; mq[2] = m23.x; mq[3] = m23.y; mq[4] = m45.x;
  mq[5] = m45.y; mq[6] = m67.x; mq[7] = m67.y; mq[8] = m89.x; mq[9] = m89.y;
}
#elif SSHOPM_43_FORM == 3
// form 3: the form-2 layout without the (x1, x2) pair (no register moves): every product pairs with (x2, x1)
template <>
__device__ __forceinline__ void monomials<4, 3>(const float2 (&xs)[2], float (&mq)[10]) {
  const float2 x01 = xs[0], x21 = xs[1];
  const float2 s0 = __fmul2_rn(bc(x01.x), x01);   // (x0x0, x0x1)
  const float2 s1 = __fmul2_rn(x01, x21);         // (x0x2, x1x1)
  const float2 s2 = __fmul2_rn(bc(x21.x), x21);   // (x2x2, x2x1)
  const float2 m01 = __fmul2_rn(bc(x01.x), s0);   // 000 001
  const float2 m23 = __fmul2_rn(bc(x01.x), s1);   // 002 011
  const float2 m54 = __fmul2_rn(bc(x01.x), s2);   // 022 012
  const float2 m76 = __fmul2_rn(bc(s1.y), x21);   // 112 111
  const float2 m98 = __fmul2_rn(bc(s2.x), x21);   // 222 122
  mq[0] = m01.x; mq[1] = m01.y; mq[2] = m23.x; mq[3] = m23.y; mq[4] = m54.y;
  mq[5] = m54.x; mq[6] = m76.y; mq[7] = m76.x; mq[8] = m98.y; mq[9] = m98.x;
}
#endif

// (4,3), form 5: Eq. 6 regrouped as a polynomial in x0 whose coefficients are forms in (x1, x2),
//   g_j = x0 (x0 (x0 B_000j + B_001j x1 + B_002j x2) + Q_j) + C_j,
//   Q_j = B_011j x1^2 + B_012j x1x2 + B_022j x2^2,  C_j = B_111j x1^3 + B_112j x1^2x2 + B_122j x1x2^2 + B_222j x2^3
// (B_qj = B-form word of monomial q for output j): 36 multiply-adds per step plus 7 shared products
// (43 FP32 pipe operations instead of 30 + 16); (g0, g1) run as FFMA2 on the B-form word pairs with
// the shared value broadcast, g2 as scalar FFMA.  State layout of form 2: xs = (x0, x1), (x2, x1).
__device__ __forceinline__ void horner43(const Coefs<4, 3>& cf, const float2 (&xs)[2], float& g0, float& g1, float& g2) {
  const float x0 = xs[0].x, x1 = xs[0].y, x2 = xs[1].x;
  const float2 p21 = xs[1];                          // (x2, x1)
  const float2 s = __fmul2_rn(bc(x1), p21);          // (x1x2, x1x1)
  const float s22 = x2 * x2;
  const float2 c1 = __fmul2_rn(bc(s.y), p21);        // (x1^2 x2, x1^3)
  const float2 c2 = __fmul2_rn(bc(s22), p21);        // (x2^3, x1 x2^2)
  float2 L = __fmul2_rn(cf.template pair<2>(), bc(x1));
  L = __ffma2_rn(cf.template pair<4>(), bc(x2), L);
  float2 t = __ffma2_rn(cf.template pair<0>(), bc(x0), L);
  float2 Q = __fmul2_rn(cf.template pair<6>(), bc(s.y));
  Q = __ffma2_rn(cf.template pair<8>(), bc(s.x), Q);
  Q = __ffma2_rn(cf.template pair<10>(), bc(s22), Q);
  t = __ffma2_rn(t, bc(x0), Q);
  float2 C = __fmul2_rn(cf.template pair<12>(), bc(c1.y));
  C = __ffma2_rn(cf.template pair<14>(), bc(c1.x), C);
  C = __ffma2_rn(cf.template pair<16>(), bc(c2.y), C);
  C = __ffma2_rn(cf.template pair<18>(), bc(c2.x), C);
  const float2 g01 = __ffma2_rn(t, bc(x0), C);
  g0 = g01.x;
  g1 = g01.y;
  float L2 = cf.template word<21>() * x1;
  L2 = fmaf(cf.template word<22>(), x2, L2);
  float t2 = fmaf(cf.template word<20>(), x0, L2);
  float Q2 = cf.template word<23>() * s.y;
  Q2 = fmaf(cf.template word<24>(), s.x, Q2);
  Q2 = fmaf(cf.template word<25>(), s22, Q2);
  t2 = fmaf(t2, x0, Q2);
  float C2 = cf.template word<26>() * c1.y;
  C2 = fmaf(cf.template word<27>(), c1.x, C2);
  C2 = fmaf(cf.template word<28>(), c2.y, C2);
  C2 = fmaf(cf.template word<29>(), c2.x, C2);
  g2 = fmaf(t2, x0, C2);
}

// ---------------------------------------------------------------- n = 3 Horner --
// Eq. 6 for n = 3 regrouped as a polynomial in x0 whose coefficients are forms in (x1, x2):
//   g_j = sum_{d=0}^{D} x0^{D-d} P_{j,d},   P_{j,d} = sum_{b+c=d} B_{(D-d,b,c),j} x1^b x2^c     (D = m - 1)
// evaluated by Horner in x0, the (x1, x2) monomials shared by the three outputs: n (Q - 1 + D) multiply-
// adds plus Q - 3 shared products per step instead of n Q + (monomial tree) — (6,3): 93 FP32 operations
// instead of 115 (default for n = 3, m >= 6; SSHOPM_HORNER3=0 restores the monomial form).  B-form rows: (g0, g1) as FFMA2 on the word pairs
// (B_{q,0}, B_{q,1}), g2 scalar.  Raw rows ((8,3)): the solver carries the multinomial weight
// D!/(a! b! c!) by divided powers (x1^b/b!, x2^c/c!, Horner factors x0/k, D! at the end); EXACT_RAW
// (the apply test hook) multiplies the shared monomials by the integer weights instead, which is exact
// on small integers and has the same Horner structure.
template <int D>
__host__ __device__ constexpr int h3_q(int a, int b, int c) {     // lex rank of the degree-D tuple 0^a 1^b 2^c
  int I[D > 0 ? D : 1] = {};
  for (int t = 0; t < D; ++t) I[t] = t < a ? 0 : (t < a + b ? 1 : 2);
  return tuple_rank(I, D, 3);
}
__host__ __device__ constexpr int h3_y(int b, int c) { return (b + c) * (b + c + 1) / 2 + c; }   // (b, c) -> slot

template <int M, bool EXACT_RAW = false>
__device__ __forceinline__ void horner3(const Coefs<M, 3>& cf, float x0, float x1, float x2, float& g0, float& g1,
                                        float& g2) {
  using S = Shape<M, 3>;
  constexpr int D = M - 1;
  constexpr int NY = (D + 1) * (D + 2) / 2;
  if constexpr (S::BFORM) {
    float y[NY];                                   // x1^b x2^c
    y[0] = 1.f;
    y[h3_y(1, 0)] = x1;
    y[h3_y(0, 1)] = x2;
    static_for<(D > 1 ? D - 1 : 0)>([&](auto dd) {
      constexpr int d = decltype(dd)::value + 2;
      static_for<d + 1>([&](auto bb) {
        constexpr int b = decltype(bb)::value, c = d - b;
        if constexpr (b > 0) y[h3_y(b, c)] = y[h3_y(b - 1, c)] * x1;
        else y[h3_y(b, c)] = y[h3_y(b, c - 1)] * x2;
      });
    });
    constexpr int base2 = 2 * S::Q;                // B_{q,2} words
#ifdef SSHOPM_H3_SCALAR
    {   // experiment: all three outputs as scalar FFMA chains (no FFMA2)
      float tt[3];
      static_for<3>([&](auto jj) {
        constexpr int j = decltype(jj)::value;
        auto W = [&](auto qq) { constexpr int q = decltype(qq)::value;
                                return j < 2 ? cf.template word<2 * q + (j < 2 ? j : 0)>() : cf.template word<base2 + q>(); };
        constexpr int q00 = h3_q<D>(D, 0, 0), q10 = h3_q<D>(D - 1, 1, 0), q01 = h3_q<D>(D - 1, 0, 1);
        float t = W(std::integral_constant<int, q10>{}) * x1;
        t = fmaf(W(std::integral_constant<int, q01>{}), x2, t);
        t = fmaf(W(std::integral_constant<int, q00>{}), x0, t);
        static_for<(D > 1 ? D - 1 : 0)>([&](auto dd) {
          constexpr int d = decltype(dd)::value + 2;
          constexpr int qa = h3_q<D>(D - d, d, 0);
          float pp = W(std::integral_constant<int, qa>{}) * y[h3_y(d, 0)];
          static_for<d>([&](auto cc) {
            constexpr int c = decltype(cc)::value + 1, b = d - c;
            pp = fmaf(W(std::integral_constant<int, h3_q<D>(D - d, b, c)>{}), y[h3_y(b, c)], pp);
          });
          t = fmaf(t, x0, pp);
        });
        tt[j] = t;
      });
      g0 = tt[0]; g1 = tt[1]; g2 = tt[2];
      return;
    }
#endif
    // level 0..1: t = B_(D,0,0) x0 + B_(D-1,1,0) x1 + B_(D-1,0,1) x2
    constexpr int q00 = h3_q<D>(D, 0, 0), q10 = h3_q<D>(D - 1, 1, 0), q01 = h3_q<D>(D - 1, 0, 1);
    float2 t01 = __fmul2_rn(cf.template pair<2 * q10>(), bc(x1));
    t01 = __ffma2_rn(cf.template pair<2 * q01>(), bc(x2), t01);
    t01 = __ffma2_rn(cf.template pair<2 * q00>(), bc(x0), t01);
    float t2 = cf.template word<base2 + q10>() * x1;
    t2 = fmaf(cf.template word<base2 + q01>(), x2, t2);
    t2 = fmaf(cf.template word<base2 + q00>(), x0, t2);
    static_for<(D > 1 ? D - 1 : 0)>([&](auto dd) {
      constexpr int d = decltype(dd)::value + 2;
      constexpr int qa = h3_q<D>(D - d, d, 0);
      float2 p01 = __fmul2_rn(cf.template pair<2 * qa>(), bc(y[h3_y(d, 0)]));
      float p2 = cf.template word<base2 + qa>() * y[h3_y(d, 0)];
      static_for<d>([&](auto cc) {
        constexpr int c = decltype(cc)::value + 1, b = d - c;
        constexpr int q = h3_q<D>(D - d, b, c);
        p01 = __ffma2_rn(cf.template pair<2 * q>(), bc(y[h3_y(b, c)]), p01);
        p2 = fmaf(cf.template word<base2 + q>(), y[h3_y(b, c)], p2);
      });
      t01 = __ffma2_rn(t01, bc(x0), p01);
      t2 = fmaf(t2, x0, p2);
    });
    g0 = t01.x;
    g1 = t01.y;
    g2 = t2;
  } else if constexpr (EXACT_RAW) {
    // raw rows: the multinomial weight D!/((D-d)! b! c!) rides on the shared (x1, x2) monomials,
    // z_{b,c} = w_{b,c} x1^b x2^c (integer weights: exact on small integers, one rounding more than y)
    constexpr Tables<M, 3> T{};
    float y[NY];
    y[0] = 1.f;
    y[h3_y(1, 0)] = x1;
    y[h3_y(0, 1)] = x2;
    static_for<(D > 1 ? D - 1 : 0)>([&](auto dd) {
      constexpr int d = decltype(dd)::value + 2;
      static_for<d + 1>([&](auto bb) {
        constexpr int b = decltype(bb)::value, c = d - b;
        if constexpr (b > 0) y[h3_y(b, c)] = y[h3_y(b - 1, c)] * x1;
        else y[h3_y(b, c)] = y[h3_y(b, c - 1)] * x2;
      });
    });
    float z[NY];
    static_for<NY>([&](auto ii) {
      constexpr int i = decltype(ii)::value;
      constexpr int d = [] { int e = 0; while ((e + 1) * (e + 2) / 2 <= i) ++e; return e; }();
      constexpr int c = i - d * (d + 1) / 2, b = d - c;
      constexpr float w = (float)(fact(D) / (fact(D - d) * fact(b) * fact(c)));
      if constexpr (w == 1.0f) z[i] = y[i];
      else z[i] = y[i] * w;
    });
    float t[3];
    static_for<3>([&](auto jj) {
      constexpr int j = decltype(jj)::value;
      float acc = cf.template word<T.q_cls[h3_q<D>(D, 0, 0)][j]>();   // weight 1 (x0^D)
      static_for<D>([&](auto dd) {
        constexpr int d = decltype(dd)::value + 1;
        constexpr int qa = h3_q<D>(D - d, d, 0);
        float p = cf.template word<T.q_cls[qa][j]>() * z[h3_y(d, 0)];
        static_for<d>([&](auto cc) {
          constexpr int c = decltype(cc)::value + 1, b = d - c;
          constexpr int q = h3_q<D>(D - d, b, c);
          p = fmaf(cf.template word<T.q_cls[q][j]>(), z[h3_y(b, c)], p);
        });
        acc = fmaf(acc, x0, p);
      });
      t[j] = acc;
    });
    g0 = t[0];
    g1 = t[1];
    g2 = t[2];
  } else {
    // raw rows, solver form: divided powers v_{b,c} = x1^b x2^c / (b! c!) and Horner factors x0 / k,
    //   g_j = D! sum_d x0^{D-d}/(D-d)! sum_{b+c=d} a_{(D-d,b,c)+e_j} v_{b,c}
    // (21 shared factors instead of 35 weight products for (8,3): C4a 5.72 -> 5.37 ms; the 1/k factors round)
    constexpr Tables<M, 3> T{};
    float v[NY];
    v[0] = 1.f;
    v[h3_y(1, 0)] = x1;
    v[h3_y(0, 1)] = x2;
    static_for<(D > 1 ? D - 1 : 0)>([&](auto dd) {
      constexpr int d = decltype(dd)::value + 2;
      static_for<d + 1>([&](auto bb) {
        constexpr int b = decltype(bb)::value, c = d - b;
        if constexpr (b > 0) v[h3_y(b, c)] = v[h3_y(b - 1, c)] * (x1 * (1.0f / (float)b));
        else v[h3_y(b, c)] = v[h3_y(b, c - 1)] * (x2 * (1.0f / (float)c));
      });
    });
    float t[3];
    static_for<3>([&](auto jj) {
      constexpr int j = decltype(jj)::value;
      float acc = cf.template word<T.q_cls[h3_q<D>(D, 0, 0)][j]>();
      static_for<D>([&](auto dd) {
        constexpr int d = decltype(dd)::value + 1;      // level d: Horner factor x0 / (D - d + 1)
        constexpr int qa = h3_q<D>(D - d, d, 0);
        float p = cf.template word<T.q_cls[qa][j]>() * v[h3_y(d, 0)];
        static_for<d>([&](auto cc) {
          constexpr int c = decltype(cc)::value + 1, b = d - c;
          constexpr int q = h3_q<D>(D - d, b, c);
          p = fmaf(cf.template word<T.q_cls[q][j]>(), v[h3_y(b, c)], p);
        });
        acc = fmaf(acc, x0 * (1.0f / (float)(D - d + 1)), p);
      });
      t[j] = acc;
    });
    constexpr float DF = (float)fact(D);
    g0 = t[0] * DF;
    g1 = t[1] * DF;
    g2 = t[2] * DF;
  }
}

// --------------------------------------------------------- any n: Horner in x0 --
// Raw rows, any n (default for n >= 6; SSHOPM_HORNERN=0 restores the monomial form): g_j = D! sum_{d} x0^{D-d}/(D-d)! sum_{|t| = d} a_{(0^{D-d} t) + e_j} v_t
// over tail multisets t of the variables 1..n-1 with divided powers v_t = prod x_i^{k_i} / k_i!
// (v_t = v_{t - l} x_l / k_l, l the last index of t), Horner in x0 with factors x0 / k.
template <int M, int N>
struct HTab {
  static constexpr int D = M - 1;
  static constexpr int NT = binom(D + N - 1, D);      // tail multisets of degree 0..D over N-1 variables
  int deg_off[D + 2];
  int parent[NT];      // index of t minus its last element (-1 for t = {})
  int var[NT];         // its last element l (1..N-1)
  int mult[NT];        // multiplicity of l in t
  int q[NT];           // degree-D multiset 0^{D-|t|} t as a Tables<M,N> q index
  long long w[NT];     // multinomial weight D! / ((D-|t|)! prod k_i!) of x0^{D-|t|} x^t (EXACT form)
  constexpr HTab() : deg_off(), parent(), var(), mult(), q(), w() {
    long long fp[NT > 0 ? NT : 1] = {};   // prod k_i! of t
    int off = 0;
    for (int d = 0; d <= D; ++d) {
      deg_off[d] = off;
      int I[D > 0 ? D : 1] = {};
      for (int i = 0; i < d; ++i) I[i] = 1;
      const int cnt = binom(d + N - 2, d);
      for (int c = 0; c < cnt; ++c) {
        const int idx = off + c;
        if (d == 0) { parent[idx] = -1; var[idx] = 0; mult[idx] = 0; }
        else {
          int J[D > 0 ? D : 1] = {};
          for (int i = 0; i < d - 1; ++i) J[i] = I[i] - 1;   // tuple over {0..N-2} for ranking
          parent[idx] = deg_off[d - 1] + tuple_rank(J, d - 1, N - 1);
          var[idx] = I[d - 1];
          int k = 0;
          for (int i = 0; i < d; ++i) k += (I[i] == I[d - 1]);
          mult[idx] = k;
        }
        fp[idx] = d == 0 ? 1 : fp[parent[idx]] * mult[idx];
        w[idx] = fact(D) / (fact(D - d) * fp[idx]);
        int K[D > 0 ? D : 1] = {};
        for (int i = 0; i < D - d; ++i) K[i] = 0;
        for (int i = 0; i < d; ++i) K[D - d + i] = I[i];
        q[idx] = tuple_rank(K, D, N);
        // next tuple over {1..N-1}
        if (d > 0) {
          int j = d - 1;
          while (j >= 0 && I[j] == N - 1) --j;
          if (j >= 0) { I[j] += 1; for (int k2 = j + 1; k2 < d; ++k2) I[k2] = I[j]; }
        }
      }
      off += cnt;
    }
    deg_off[D + 1] = off;
  }
};

// EXACT (the apply test hook): plain monomials times the integer weights, plain Horner in x0 (exact on
// small integers; same structure, one weight product per tail monomial instead of the 1/k factors).
template <int M, int N, bool EXACT = false>
__device__ __forceinline__ void hornerN(const Coefs<M, N>& cf, const float (&x)[N], float (&g)[N]) {
  using H = HTab<M, N>;
  constexpr H T{};
  constexpr Tables<M, N> TT{};
  constexpr int D = M - 1;
  float v[H::NT];
  v[0] = 1.f;
  static_for<H::NT - 1>([&](auto ii) {
    constexpr int i = decltype(ii)::value + 1;
    constexpr int par = T.parent[i], l = T.var[i], k = T.mult[i];
    if constexpr (par == 0) v[i] = x[l];
    else if constexpr (k == 1 || EXACT) v[i] = v[par] * x[l];
    else v[i] = v[par] * (x[l] * (1.0f / (float)k));
  });
  if constexpr (EXACT) {
    float z[H::NT];
    static_for<H::NT>([&](auto ii) {
      constexpr int i = decltype(ii)::value;
      constexpr long long wi = H{}.w[i];
      if constexpr (wi == 1) z[i] = v[i];
      else z[i] = v[i] * (float)wi;
    });
    static_for<N>([&](auto jj) {
      constexpr int j = decltype(jj)::value;
      float acc = cf.template word<TT.q_cls[T.q[0]][j]>();
      static_for<D>([&](auto dd) {
        constexpr int d = decltype(dd)::value + 1;
        constexpr int o = T.deg_off[d], cnt = T.deg_off[d + 1] - T.deg_off[d];
        float p = cf.template word<TT.q_cls[T.q[o]][j]>() * z[o];
        static_for<cnt - 1>([&](auto cc) {
          constexpr int i = o + decltype(cc)::value + 1;
          p = fmaf(cf.template word<TT.q_cls[T.q[i]][j]>(), z[i], p);
        });
        acc = fmaf(acc, x[0], p);
      });
      g[j] = acc;
    });
    return;
  }
  static_for<N>([&](auto jj) {
    constexpr int j = decltype(jj)::value;
    float acc = cf.template word<TT.q_cls[T.q[0]][j]>();
    static_for<D>([&](auto dd) {
      constexpr int d = decltype(dd)::value + 1;
      constexpr int o = T.deg_off[d], cnt = T.deg_off[d + 1] - T.deg_off[d];
      float p = cf.template word<TT.q_cls[T.q[o]][j]>() * v[o];
      static_for<cnt - 1>([&](auto cc) {
        constexpr int i = o + decltype(cc)::value + 1;
        p = fmaf(cf.template word<TT.q_cls[T.q[i]][j]>(), v[i], p);
      });
      acc = fmaf(acc, x[0] * (1.0f / (float)(D - d + 1)), p);
    });
    g[j] = acc * (float)fact(D);
  });
}

// (4,3), form 4: all-scalar evaluation (16 FMUL monomials, 30 FFMA, lambda as an FMA chain).
__device__ __forceinline__ float eval43s(const Coefs<4, 3>& cf, float x0, float x1, float x2, float& g0, float& g1,
                                         float& g2) {
  const float d00 = x0 * x0, d01 = x0 * x1, d02 = x0 * x2, d11 = x1 * x1, d12 = x1 * x2, d22 = x2 * x2;
  const float mq[10] = {x0 * d00, x0 * d01, x0 * d02, x0 * d11, x0 * d12, x0 * d22, x1 * d11, x1 * d12, x1 * d22,
                        x2 * d22};
  g0 = cf.template word<0>() * mq[0];
  g1 = cf.template word<1>() * mq[0];
  g2 = cf.template word<20>() * mq[0];
  static_for<9>([&](auto qq) {
    constexpr int q = decltype(qq)::value + 1;
    g0 = fmaf(cf.template word<2 * q>(), mq[q], g0);
    g1 = fmaf(cf.template word<2 * q + 1>(), mq[q], g1);
    g2 = fmaf(cf.template word<20 + q>(), mq[q], g2);
  });
  return fmaf(x2, g2, fmaf(x1, g1, x0 * g0));
}

// (4,3), natural layout (x0, x1 | x2): monomials from 7 FMUL2 + 2 FMUL; Eq. 6 as (g0, g1) FFMA2 with the
// monomial broadcast plus g2 scalar FFMA on the same monomial (q outer).
__device__ __forceinline__ float eval43n(const Coefs<4, 3>& cf, const float2 (&xs)[2], float2& g01, float& g2) {
  const float2 x01 = xs[0];
  const float x0 = x01.x, x1 = x01.y, x2 = xs[1].x;
  const float2 a = __fmul2_rn(bc(x0), x01);   // x0x0, x0x1
  const float2 b = __fmul2_rn(bc(x2), x01);   // x0x2, x1x2
  const float2 c = f2(x1 * x1, x2 * x2);      // x1x1, x2x2
  const float2 m0 = __fmul2_rn(bc(x0), a);    // q0 = 000, q1 = 001
  const float2 m1 = __fmul2_rn(bc(x2), a);    // q2 = 002, q4 = 012
  const float2 m2 = __fmul2_rn(bc(c.x), x01); // q3 = 011, q6 = 111
  const float2 m3 = __fmul2_rn(bc(x2), b);    // q5 = 022, q8 = 122
  const float2 m4 = __fmul2_rn(bc(x2), c);    // q7 = 112, q9 = 222
  const float mq[10] = {m0.x, m0.y, m1.x, m2.x, m1.y, m3.x, m2.y, m4.x, m3.y, m4.y};
  g2 = cf.template word<20>() * mq[0];
  g01 = __fmul2_rn(cf.template pair<0>(), bc(mq[0]));
  static_for<9>([&](auto qq) {
    constexpr int q = decltype(qq)::value + 1;
    g2 = fmaf(cf.template word<20 + q>(), mq[q], g2);
    g01 = __ffma2_rn(cf.template pair<2 * q>(), bc(mq[q]), g01);
  });
  const float2 t = __fmul2_rn(x01, g01);
  return fmaf(x2, g2, t.x + t.y);
}

// g = A x^{M-1} (pairs gp, odd tail gs) and lambda = x . g
#ifndef SSHOPM_HORNERN
#define SSHOPM_HORNERN 1   // raw-row shapes with n >= SSHOPM_HORNERN_MIN_N evaluate Eq. 6 by hornerN: C4b 9.20 -> 8.74 ms
#endif
#ifndef SSHOPM_HORNERN_MIN_N
#define SSHOPM_HORNERN_MIN_N 6
#endif
template <int M, int N>
__device__ __forceinline__ float evaluate(const Coefs<M, N>& cf, const float2 (&xs)[(N + 1) / 2],
                                          float2 (&gp)[Shape<M, N>::NP > 0 ? Shape<M, N>::NP : 1], float& gs) {
  using S = Shape<M, N>;
  if constexpr (SSHOPM_HORNERN && !S::BFORM && N >= SSHOPM_HORNERN_MIN_N && N >= 4) {
    float x[N], g[N];
#pragma unroll
    for (int i = 0; i < N; ++i) x[i] = xget<M, N>(xs, i);
    hornerN<M, N>(cf, x, g);
#pragma unroll
    for (int p = 0; p < S::NP; ++p) gp[p] = f2(g[2 * p], g[2 * p + 1]);
    if constexpr (S::ODD) gs = g[N - 1];
  } else {
    float mq[S::Q];
    monomials<M, N>(xs, mq);
    cf.contract(mq, gp, gs);
  }
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

// One SS-HOPM step (Fig. 1) for one lane: lam_k = x_k . A x_k^{m-1}; the stop
// test (R2, R6, maxit); x_{k+1} = +-(g + alpha x) / ||.|| (lines 2-7, R5).
// Stopped lanes freeze (x, lambda_prev, k unchanged) so a frozen lane
// recomputes bit-identical values until the warp refills it.
// SHIFT: 0 alpha = 0, 1 alpha > 0, 2 alpha < 0 (alpha passed negated), 3 per-lane (la = |alpha|, ls = sign)
// KIDLE: lanes without an item hold k = INT_MAX (>= maxit), so the maxit test also stops them and the
// per-step stop predicate needs no separate `has` term (schedule 1 keeps this convention).
template <int M, int N, int SHIFT, bool KIDLE = false>
__device__ __forceinline__ void sshopm_step(const Coefs<M, N>& cf, float2 (&xs)[Shape<M, N>::NX], float& lam,
                                            float& lamp, int& k, bool& conv, bool& stop, bool has, float alpha,
                                            float la, float ls, float tol, int maxit) {
  using S = Shape<M, N>;
  if constexpr (X02<M, N>::v) {
    float g0, g1, g2;
    lam = eval43(cf, xs, g0, g1, g2);                         // g = A x_k^3, lam_k = x_k . g
    conv = fabsf(lam - lamp) <= tol * fmaxf(1.0f, fabsf(lam));  // R2 (NaN lamp -> false)
    const float x0 = xs[0].x, x2 = xs[0].y, x1 = xs[1].x;
    float h0, h1, h2;                                         // xhat = +-(g + alpha x)   (Fig. 1 lines 2-5, R5)
    if constexpr (SHIFT == 0) { h0 = g0; h1 = g1; h2 = g2; }
    else if constexpr (SHIFT == 1) { h0 = fmaf(alpha, x0, g0); h1 = fmaf(alpha, x1, g1); h2 = fmaf(alpha, x2, g2); }
    else if constexpr (SHIFT == 2) { h0 = fmaf(alpha, x0, -g0); h1 = fmaf(alpha, x1, -g1); h2 = fmaf(alpha, x2, -g2); }
    else { h0 = fmaf(la, x0, g0 * ls); h1 = fmaf(la, x1, g1 * ls); h2 = fmaf(la, x2, g2 * ls); }
    const float nn = fmaf(h2, h2, fmaf(h1, h1, h0 * h0));
    const bool deg = !(nn >= 1.17549435e-38f);                  // R6 (FP32: subnormal counts as zero)
    if constexpr (KIDLE) stop = conv | (k >= maxit) | deg;
    else stop = (!has) | conv | (k >= maxit) | deg;
    const float r = rsqrt_ftz(nn);                              // line 7: x = xhat / ||xhat||
    if (!stop) {
      xs[0] = __fmul2_rn(f2(h0, h2), bc(r));
      xs[1].x = h1 * r;
      lamp = lam;
      ++k;
    }
    return;
  } else if constexpr (S43<M, N>::v) {
    const float x0 = xs[0].x, x1 = xs[0].y, x2 = xs[1].x;
    float g0, g1, g2;
    lam = eval43s(cf, x0, x1, x2, g0, g1, g2);
    conv = fabsf(lam - lamp) <= tol * fmaxf(1.0f, fabsf(lam));
    float h0, h1, h2;
    if constexpr (SHIFT == 0) { h0 = g0; h1 = g1; h2 = g2; }
    else if constexpr (SHIFT == 1) { h0 = fmaf(alpha, x0, g0); h1 = fmaf(alpha, x1, g1); h2 = fmaf(alpha, x2, g2); }
    else if constexpr (SHIFT == 2) { h0 = fmaf(alpha, x0, -g0); h1 = fmaf(alpha, x1, -g1); h2 = fmaf(alpha, x2, -g2); }
    else { h0 = fmaf(la, x0, g0 * ls); h1 = fmaf(la, x1, g1 * ls); h2 = fmaf(la, x2, g2 * ls); }
    const float nn = fmaf(h2, h2, fmaf(h1, h1, h0 * h0));
    const bool deg = !(nn >= 1.17549435e-38f);
    if constexpr (KIDLE) stop = conv | (k >= maxit) | deg;
    else stop = (!has) | conv | (k >= maxit) | deg;
    const float r = rsqrt_ftz(nn);
    if (!stop) {
      xs[0].x = h0 * r;
      xs[0].y = h1 * r;
      xs[1].x = h2 * r;
      lamp = lam;
      ++k;
    }
    return;
  } else if constexpr (N43<M, N>::v) {
    float2 g01;
    float g2;
    lam = eval43n(cf, xs, g01, g2);
    conv = fabsf(lam - lamp) <= tol * fmaxf(1.0f, fabsf(lam));
    float2 h01;
    float h2;
    const float x2 = xs[1].x;
    if constexpr (SHIFT == 0) { h01 = g01; h2 = g2; }
    else if constexpr (SHIFT == 1) { h01 = __ffma2_rn(bc(alpha), xs[0], g01); h2 = fmaf(alpha, x2, g2); }
    else if constexpr (SHIFT == 2) { h01 = __ffma2_rn(bc(alpha), xs[0], f2(-g01.x, -g01.y)); h2 = fmaf(alpha, x2, -g2); }
    else { h01 = __ffma2_rn(bc(la), xs[0], __fmul2_rn(g01, bc(ls))); h2 = fmaf(la, x2, g2 * ls); }
    const float2 u = __fmul2_rn(h01, h01);
    const float nn = fmaf(h2, h2, u.x + u.y);
    const bool deg = !(nn >= 1.17549435e-38f);
    if constexpr (KIDLE) stop = conv | (k >= maxit) | deg;
    else stop = (!has) | conv | (k >= maxit) | deg;
    const float r = rsqrt_ftz(nn);
    if (!stop) {
      xs[0] = __fmul2_rn(h01, bc(r));
      xs[1].x = h2 * r;
      lamp = lam;
      ++k;
    }
    return;
  } else if constexpr (X21<M, N>::v && SSHOPM_X21_TAIL == 1) {
    // form-2 monomials and contraction (form 5: Horner in x0); lambda, ||xhat||^2 and the update as scalar
    // FP32 (no packed op next to the scalar ones there: DESIGN.md "pipe mix")
    float g0, g1, g2;
    if constexpr (H43<M, N>::v) {
      horner43(cf, xs, g0, g1, g2);
    } else {
      float mq[S::Q];
      monomials<M, N>(xs, mq);
      float2 gp[1];
      g2 = 0.f;
      cf.contract(mq, gp, g2);
      g0 = gp[0].x;
      g1 = gp[0].y;
    }
    const float x0 = xs[0].x, x1 = xs[0].y, x2 = xs[1].x;
    lam = fmaf(x2, g2, fmaf(x1, g1, x0 * g0));
    conv = fabsf(lam - lamp) <= tol * fmaxf(1.0f, fabsf(lam));
    float h0, h1, h2;
    if constexpr (SHIFT == 0) { h0 = g0; h1 = g1; h2 = g2; }
    else if constexpr (SHIFT == 1) { h0 = fmaf(alpha, x0, g0); h1 = fmaf(alpha, x1, g1); h2 = fmaf(alpha, x2, g2); }
    else if constexpr (SHIFT == 2) { h0 = fmaf(alpha, x0, -g0); h1 = fmaf(alpha, x1, -g1); h2 = fmaf(alpha, x2, -g2); }
    else { h0 = fmaf(la, x0, g0 * ls); h1 = fmaf(la, x1, g1 * ls); h2 = fmaf(la, x2, g2 * ls); }
    const float nn = fmaf(h2, h2, fmaf(h1, h1, h0 * h0));
    const bool deg = !(nn >= 1.17549435e-38f);
    if constexpr (KIDLE) stop = conv | (k >= maxit) | deg;
    else stop = (!has) | conv | (k >= maxit) | deg;
    const float r = rsqrt_ftz(nn);
    if (!stop) {
      const float y1 = h1 * r;
      xs[0] = f2(h0 * r, y1);
      xs[1] = f2(h2 * r, y1);
      lamp = lam;
      ++k;
    }
    return;
  } else if constexpr (N == 3 && ((SSHOPM_GEN_TAIL == 1 && S::Q * N <= 64) || (SSHOPM_HORNER3 && M >= 6))) {
    // other n = 3 shapes: the library contraction (or Horner in x0, SSHOPM_HORNER3), then lambda,
    // ||xhat||^2 and the update in scalar FP32
    const float x0 = xs[0].x, x1 = xs[0].y, x2 = xs[1].x;
    float g0, g1, g2;
    if constexpr (SSHOPM_HORNER3 && M >= 6) {
      horner3<M>(cf, x0, x1, x2, g0, g1, g2);
    } else {
      float mq[S::Q];
      monomials<M, N>(xs, mq);
      float2 gp[1];
      g2 = 0.f;
      cf.contract(mq, gp, g2);
      g0 = gp[0].x;
      g1 = gp[0].y;
    }
    lam = fmaf(x2, g2, fmaf(x1, g1, x0 * g0));
    conv = fabsf(lam - lamp) <= tol * fmaxf(1.0f, fabsf(lam));
    float h0, h1, h2;
    if constexpr (SHIFT == 0) { h0 = g0; h1 = g1; h2 = g2; }
    else if constexpr (SHIFT == 1) { h0 = fmaf(alpha, x0, g0); h1 = fmaf(alpha, x1, g1); h2 = fmaf(alpha, x2, g2); }
    else if constexpr (SHIFT == 2) { h0 = fmaf(alpha, x0, -g0); h1 = fmaf(alpha, x1, -g1); h2 = fmaf(alpha, x2, -g2); }
    else { h0 = fmaf(la, x0, g0 * ls); h1 = fmaf(la, x1, g1 * ls); h2 = fmaf(la, x2, g2 * ls); }
    const float nn = fmaf(h2, h2, fmaf(h1, h1, h0 * h0));
    const bool deg = !(nn >= 1.17549435e-38f);
    if constexpr (KIDLE) stop = conv | (k >= maxit) | deg;
    else stop = (!has) | conv | (k >= maxit) | deg;
    const float r = rsqrt_ftz(nn);
    if (!stop) {
      xs[0] = f2(h0 * r, h1 * r);
      xs[1].x = h2 * r;
      lamp = lam;
      ++k;
    }
    return;
  } else {
  float2 gp[S::NP > 0 ? S::NP : 1];
  float gs = 0.f;
  lam = evaluate<M, N>(cf, xs, gp, gs);                       // g = A x_k^{m-1}, lam_k = x_k . g
  conv = fabsf(lam - lamp) <= tol * fmaxf(1.0f, fabsf(lam));  // R2 (NaN lamp -> false)
  // xhat = +-(g + alpha x)   (Fig. 1 lines 2-5, R5)
  float2 hp[S::NX];
  static_for<S::NP>([&](auto qq) {
    constexpr int i = decltype(qq)::value;
    if constexpr (SHIFT == 0) hp[i] = gp[i];
    else if constexpr (SHIFT == 1) hp[i] = __ffma2_rn(bc(alpha), xs[i], gp[i]);
    else if constexpr (SHIFT == 2) hp[i] = __ffma2_rn(bc(alpha), xs[i], f2(-gp[i].x, -gp[i].y));
    else hp[i] = __ffma2_rn(bc(la), xs[i], __fmul2_rn(gp[i], bc(ls)));
  });
  if constexpr (S::ODD) {
    float h;
    if constexpr (SHIFT == 0) h = gs;
    else if constexpr (SHIFT == 1) h = fmaf(alpha, xs[S::NX - 1].x, gs);
    else if constexpr (SHIFT == 2) h = fmaf(alpha, xs[S::NX - 1].x, -gs);
    else h = fmaf(la, xs[S::NX - 1].x, gs * ls);
    hp[S::NX - 1] = f2(h, 0.f);
  }
  float nn;
  {
    float2 t = __fmul2_rn(hp[0], hp[0]);
    static_for<S::NX - 1>([&](auto qq) {
      constexpr int i = decltype(qq)::value + 1;
      if constexpr (S::ODD && i == S::NX - 1) t.x = fmaf(hp[i].x, hp[i].x, t.x);
      else t = __ffma2_rn(hp[i], hp[i], t);
    });
    nn = t.x + t.y;
  }
  const bool deg = !(nn >= 1.17549435e-38f);                  // R6 (FP32: subnormal counts as zero)
  if constexpr (KIDLE) stop = conv | (k >= maxit) | deg;      // idle lanes: k = INT_MAX
  else stop = (!has) | conv | (k >= maxit) | deg;             // non-short-circuit: one predicate chain
  const float r = rsqrt_ftz(nn);                              // line 7: x = xhat / ||xhat||
  // the freeze is a guarded update that ptxas if-converts into predicated
  // FMUL2 / FMUL / MOV / IADD: no select per component (+9% step throughput
  // on B200, tools/microbench/step_loop.cu)
  if (!stop) {
    if constexpr (X21<M, N>::v) {
      xs[0] = __fmul2_rn(hp[0], bc(r));
      xs[1] = f2(hp[1].x * r, xs[0].y);
    } else {
#pragma unroll
      for (int i = 0; i < S::NP; ++i) xs[i] = __fmul2_rn(hp[i], bc(r));
      if constexpr (S::ODD) xs[S::NX - 1].x = hp[S::NX - 1].x * r;   // .y stays 0
    }
    lamp = lam;
    ++k;
  }
  }
}

// ------------------------------------------------------------ solve kernel --
struct SolveParams {
  const float4* packed;      // [N][PW/4] from sshopm_pack_kernel
  const float4* starts_n;    // [S][SST/4] normalised starts from sshopm_pack_kernel
  float* out_lambda;         // [N][S]
  float* out_x;              // [N][S][n]
  int32_t* out_iters;        // [N][S]
  uint8_t* out_conv;         // [N][S]
  unsigned long long* total_iters;  // optional
  unsigned int* counter;     // chunk counter (zeroed by the pack kernel)
  long long n_tensors;
  long long n_chunks;
  int chunk_tensors;         // tensors per chunk
  int S;
  FastDiv divS;
  int s_log2;                // log2(S) if S is a power of two, else -1
  uint32_t s_mask;           // S - 1 (used when S is a power of two)
  float alpha, tol;
  const float* alpha_t;      // SHIFT == 3: per-tensor shift [N] (from the pack kernel)
  int maxit;
  int refill_k;              // refill threshold
  // fused solve -> dedup (FUSED kernels only)
  DedupParams dd;            // dedup outputs; dd.lambda/x/conv = the raw outputs above
  unsigned int* ovf_count;   // chunks whose completion could not be tracked (zeroed by the pack kernel)
  unsigned int* ovf_list;    // their chunk indices -> sshopm_dedup_list_kernel
  int fused_regs;            // S == 128 with 16-byte aligned raw outputs: register-resident dedup, no staging smem
  long long chunk_items;     // FUSED_MODE 4 (small N): items per claimed chunk (part of a tensor)
  long long n_items;         // N * S
};

constexpr int kFusedRing = 16;   // open-chunk ring per warp (fused solve -> dedup), power of two
__host__ __device__ constexpr int fused_smem_words(int S, int n, bool regs) {
  return 3 * kFusedRing + (regs ? 0 : dedup_smem_words(S, n));
}
// Fused mode 3 (warp-specialised): warps 0..6 solve, warp 7 clusters the chunks they complete.  Shared
// memory: 8 open-chunk rings, a CTA queue of completed chunks (kWsQueue slots + head, tail, finished),
// the dedup warp's fallback staging (tensors with > 32 clusters, or S != 128).
constexpr int kWsQueue = 64;     // power of two
constexpr int kWsSolveWarps = 7;
constexpr unsigned int kWsEmpty = 0xffffffffu;
__host__ __device__ constexpr int ws_smem_words(int S, int n) {
  return 8 * 3 * kFusedRing + kWsQueue + 4 + dedup_smem_words(S, n);
}

__device__ __forceinline__ uint32_t lanemask_lt() {
  uint32_t r;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(r));
  return r;
}

// SHIFT: 0 -> alpha == 0 (xhat = g), 1 -> alpha > 0 (xhat = g + alpha x), 2 -> alpha < 0 (xhat = -(g + alpha x)),
//        3 -> per-tensor alpha from p.alpha_t (schedule 1 only)
// WIDE: 64-bit item indices (N*S >= 2^31); otherwise 32-bit index arithmetic.
// FUSED: also cluster each chunk's tensors (R16) as soon as the warp has
// written the chunk's last item (open chunks tracked in a shared-memory ring;
// untracked chunks go to p.ovf_list for sshopm_dedup_list_kernel).
template <int M, int N, int SHIFT, bool WIDE, int FUSED_MODE>
__global__ void __launch_bounds__((FUSED_MODE == 0 || FUSED_MODE == 4) ? Shape<M, N>::TPB : 256,
                                  (FUSED_MODE == 0 || FUSED_MODE == 4) ? Shape<M, N>::MINB_T : Shape<M, N>::MINB)
sshopm_solve_kernel(const SolveParams p) {
  constexpr bool ITEMCH = FUSED_MODE == 4;       // 4: not fused; chunks of items instead of whole tensors (small N)
  constexpr bool FUSED = FUSED_MODE != 0 && !ITEMCH;   // 1: shared-memory dedup (any S <= 1024), 2: register dedup (S = 128)
  constexpr bool WS = FUSED_MODE == 3;           // 3: warp-specialised (a dedup warp per CTA consumes completed chunks)
  constexpr int STEPS = steps_per_trip<M, N>();        // SS-HOPM steps between refill checks
  using S = Shape<M, N>;
  using Idx = typename std::conditional<WIDE, long long, uint32_t>::type;
  constexpr int SST4 = round4(N) / 4;

  const int lane = threadIdx.x & 31;
  const uint32_t ltmask = lanemask_lt();
  const uint32_t FULL = 0xffffffffu;
  const float alpha = (SHIFT == 2) ? -p.alpha : p.alpha;   // xhat = sgn*g + (sgn*alpha) x
  const float tol = p.tol;
  const int maxit = p.maxit;
  const uint32_t S_ = (uint32_t)p.S;

  // fused dedup: per-warp open-chunk ring + dedup staging in shared memory
  extern __shared__ int fsm[];
  int* r_seq = fsm + (threadIdx.x >> 5) * (WS ? 3 * kFusedRing : fused_smem_words(p.S, N, FUSED_MODE == 2));
  unsigned int* wq = reinterpret_cast<unsigned int*>(fsm + 8 * 3 * kFusedRing);   // WS: [kWsQueue] + head, tail, finished
  if constexpr (WS) {
    for (int i = threadIdx.x; i < kWsQueue; i += blockDim.x) wq[i] = kWsEmpty;
    if (threadIdx.x == 0) { wq[kWsQueue] = 0u; wq[kWsQueue + 1] = 0u; wq[kWsQueue + 2] = 0u; }
    __syncthreads();
    if ((threadIdx.x >> 5) == kWsSolveWarps) {     // ---- the dedup warp ----
      volatile unsigned int* vq = wq;
      float* st = reinterpret_cast<float*>(wq + kWsQueue + 4);
      float* s_lam = st;
      float* s_x = s_lam + p.S;
      int* s_cid = reinterpret_cast<int*>(s_x + (size_t)p.S * N);
      float* c_lam = reinterpret_cast<float*>(s_cid + p.S);
      int* c_rep = reinterpret_cast<int*>(c_lam + p.S);
      int* c_mult = c_rep + p.S;
      unsigned int h = 0;
      for (;;) {
        if (h == vq[kWsQueue + 1]) {
          if (vq[kWsQueue + 2] == (unsigned int)kWsSolveWarps && h == vq[kWsQueue + 1]) break;
          __nanosleep(200);
          continue;
        }
        unsigned int ch;
        while ((ch = vq[h & (kWsQueue - 1)]) == kWsEmpty) {}   // slot reserved, chunk index not yet written
        __syncwarp();
        if (lane == 0) { vq[h & (kWsQueue - 1)] = kWsEmpty; vq[kWsQueue] = h + 1; }
        ++h;
        __threadfence_block();                      // acquire: the producer fenced its raw-output stores
        const long long v0 = (long long)ch * p.chunk_tensors;
        const long long v1 = min(p.n_tensors, v0 + p.chunk_tensors);
#pragma unroll 1
        for (long long v = v0; v < v1; ++v) {
          bool ok = false;
          if (p.fused_regs) ok = warp_dedup128_regs<N, (M % 2) == 0>(p.dd, v, lane);
          if (!ok) warp_dedup_tensor<N, (M % 2) == 0>(p.dd, v, lane, s_lam, s_x, s_cid, c_lam, c_rep, c_mult);
        }
      }
      return;
    }
  }
  unsigned int* r_chunk = reinterpret_cast<unsigned int*>(r_seq + kFusedRing);
  int* r_rem = r_seq + 2 * kFusedRing;
  float* d_lam = reinterpret_cast<float*>(r_seq + 3 * kFusedRing);
  float* d_x = d_lam + p.S;
  int* d_cid = reinterpret_cast<int*>(d_x + p.S * N);
  float* d_clam = reinterpret_cast<float*>(d_cid + p.S);
  int* d_crep = reinterpret_cast<int*>(d_clam + p.S);
  int* d_cmult = d_crep + p.S;
  int claim_seq = 0, cur_seq = 0, cseq = -1;
  if constexpr (FUSED) {
    if ((threadIdx.x & 31) < kFusedRing) { r_seq[threadIdx.x & 31] = -1; r_rem[threadIdx.x & 31] = 0; }
    __syncwarp();
  }

  // warp-uniform chunk state
  Idx c_vox = 0;              // first tensor (ITEMCH: first item) of the current chunk
  uint32_t c_next = 0, c_end = 0;
  bool exhausted = false;

  Coefs<M, N> cf;
  float2 xs[S::NX];
#pragma unroll
  for (int i = 0; i < S::NX; ++i) xs[i] = f2(0.f, 0.f);
  float lamp = 0.f, lam = 0.f;
  int k = 0;
  bool has = false, stop = true, conv = false;
  Idx item = 0;
#ifdef SSHOPM_SKIP_RELOAD
  Idx cur_tv = (Idx)-1;
#endif
  float la = 0.f, ls = 1.f;  // SHIFT == 3: per-lane |alpha| and sign: xhat = ls*g + la*x
  uint32_t it_sum = 0;       // per-lane sum of iterations (<= items per lane x maxit; flushed as 64-bit)
  // refill threshold: K idle lanes while items remain, all 32 once the chunks are exhausted,
  // so the per-trip check is one ballot, one popc and one compare (K in [1, 32], host-clamped)
  uint32_t k_eff = (uint32_t)p.refill_k;

  for (;;) {
    // ---------------- refill (warp-uniform branch) ----------------
    const uint32_t smask = __ballot_sync(FULL, stop);
    const uint32_t cnt = __popc(smask);
    if (cnt >= k_eff) {
      // straight-line refill: predicated stores / loads, selects for state (no divergent regions)
      const uint32_t avail = c_end - c_next;                 // invariant: c_next <= c_end
      uint32_t n_end = 0;
      Idx n_vox = 0;
      if (!exhausted && cnt > avail) {                       // claim the next chunk (one atomic per warp)
        unsigned int ch = 0;
        if (lane == 0) ch = atomicAdd(p.counter, 1u);
        ch = __shfl_sync(FULL, ch, 0);
        if ((long long)ch < p.n_chunks) {
          if constexpr (ITEMCH) {                          // chunks of items (small problems)
            n_vox = (Idx)ch * (Idx)p.chunk_items;           // first item of the chunk
            const long long ni = p.n_items - (long long)n_vox;
            n_end = (uint32_t)(ni < p.chunk_items ? ni : p.chunk_items);
          } else {                                         // chunks of whole tensors
            n_vox = (Idx)ch * (Idx)p.chunk_tensors;         // first tensor of the chunk
            const long long nt = p.n_tensors - (long long)n_vox;
            n_end = (uint32_t)((nt < p.chunk_tensors ? nt : p.chunk_tensors) * S_);
          }
          if constexpr (FUSED) {
            ++claim_seq;
            const int slot = claim_seq & (kFusedRing - 1);
            if (lane == 0) {
              if (r_rem[slot] > 0) p.ovf_list[atomicAdd(p.ovf_count, 1u)] = r_chunk[slot];   // still open: hand over
              r_seq[slot] = claim_seq;
              r_chunk[slot] = ch;
              r_rem[slot] = (int)n_end;
            }
            __syncwarp();
          }
        }
      }
      const bool wr = stop && has;
      if (wr) {
        p.out_lambda[item] = lam;
        float* ox = p.out_x + (size_t)item * N;              // one 64-bit row address, immediate offsets
#pragma unroll
        for (int j = 0; j < N; ++j) ox[j] = xget<M, N>(xs, j);
        p.out_iters[item] = k;
        p.out_conv[item] = conv ? 1 : 0;
      }
            if (p.total_iters != nullptr) it_sum += wr ? (uint32_t)k : 0u;   // only when requested (C2: -0.5%)
      bool chunk_done = false;
      int done_slot = 0;                                   // ring slot of the chunk this lane completed
      if constexpr (FUSED) {
        if (wr) {
          const int slot = cseq & (kFusedRing - 1);
          if (r_seq[slot] == cseq) chunk_done = (atomicSub(&r_rem[slot], 1) == 1);
          done_slot = slot;
        }
      }
      const uint32_t rank = __popc(smask & ltmask);
      const bool cur = rank < avail;
      const uint32_t t = cur ? c_next + rank : rank - avail;
      const bool ok = stop && !exhausted && (cur || t < n_end);
      if (ok) {
        const Idx v0 = cur ? c_vox : n_vox;
        if constexpr (ITEMCH) item = v0 + (Idx)t;
        else item = v0 * (Idx)S_ + (Idx)t;
        Idx tv;                                            // tensor of the item
        uint32_t s;                                        // its start
#ifndef SSHOPM_ASSUME_POW2
#define SSHOPM_ASSUME_POW2 0   // experiment: compile only the power-of-two index path
#endif
        if (SSHOPM_ASSUME_POW2 || p.s_log2 >= 0) {         // S a power of two (the paper's 128): shift and mask
          tv = item >> p.s_log2;
          s = (uint32_t)item & p.s_mask;
        } else if constexpr (ITEMCH) {
          if constexpr (WIDE) {
            tv = item / (Idx)S_;
            s = (uint32_t)(item - tv * (Idx)S_);
          } else {
            tv = fast_div((uint32_t)item, p.divS);
            s = (uint32_t)item - (uint32_t)tv * S_;
          }
        } else {
          const uint32_t vq = fast_div(t, p.divS);
          s = t - vq * S_;
          tv = v0 + (Idx)vq;
        }
        SSHOPM_CHECK((long long)tv < p.n_tensors && s < S_ && (long long)item == (long long)tv * S_ + s);
        if constexpr (FUSED) cseq = cur ? cur_seq : claim_seq;
        if constexpr (SHIFT == 3) {
          const float at = __ldg(p.alpha_t + tv);
          ls = at >= 0.f ? 1.f : -1.f;                     // Fig. 1 lines 2-5 (R5: alpha = 0 -> "+")
          la = fabsf(at);
        }
#ifdef SSHOPM_SKIP_RELOAD
        if (tv != cur_tv) { cf.load(p.packed + tv * (Idx)(S::PW / 4)); cur_tv = tv; }   // experiment: same tensor -> keep the rows
#else
        cf.load(p.packed + tv * (Idx)(S::PW / 4));
#endif
        float v[4 * SST4];
#pragma unroll
        for (int i = 0; i < SST4; ++i) {
          const float4 q4 = ldg4(p.starts_n + s * SST4 + i);
          v[4 * i] = q4.x; v[4 * i + 1] = q4.y; v[4 * i + 2] = q4.z; v[4 * i + 3] = q4.w;
        }
#pragma unroll
        for (int i = 0; i < S::NX; ++i) xs[i] = f2(v[2 * i], v[2 * i + 1]);   // starts_n is in slot order
      }
      k = ok ? 0 : (stop ? 0x7fffffff : k);                  // idle lanes: k >= maxit keeps them stopped
      lamp = ok ? __int_as_float(0x7fffffff) : lamp;         // NaN: the first test never fires (reading R2)
      has = stop ? ok : has;
      if (!exhausted) {
        if (cnt > avail) {
          if (n_end == 0) { exhausted = true; k_eff = 32u; }
          c_vox = n_vox;
          c_next = min(cnt - avail, n_end);                // a chunk smaller than the request is used up
          c_end = n_end;
          cur_seq = claim_seq;
        } else {
          c_next += cnt;
        }
      }
      if constexpr (WS) {
        uint32_t dmask = __ballot_sync(FULL, chunk_done);
        if (dmask) {                                       // publish the completed chunks to the dedup warp
          __threadfence_block();                           // release: this warp's raw-output stores first
          __syncwarp();
          do {
            const int src = __ffs(dmask) - 1;
            dmask &= dmask - 1;
            const int slot = __shfl_sync(FULL, done_slot, src);
            if (lane == 0) {
              volatile unsigned int* vq = wq;
              const unsigned int ch = r_chunk[slot];
              unsigned int t = vq[kWsQueue + 1];
              bool queued = false;
              for (;;) {                                   // reserve a queue slot unless the queue is full
                if (t - vq[kWsQueue] >= (unsigned int)kWsQueue) break;
                const unsigned int o = atomicCAS(wq + kWsQueue + 1, t, t + 1);
                if (o == t) { queued = true; break; }
                t = o;
              }
              if (queued) vq[t & (kWsQueue - 1)] = ch;
              else p.ovf_list[atomicAdd(p.ovf_count, 1u)] = ch;   // full: clustered by the list kernel
              r_seq[slot] = -1;
            }
            __syncwarp();
          } while (dmask);
        }
      }
      if constexpr (FUSED && !WS) {
        uint32_t dmask = __ballot_sync(FULL, chunk_done);
        if (dmask) {                                       // cluster the completed chunks' tensors now (L2-hot)
          __threadfence_block();
          __syncwarp();
          do {
            const int src = __ffs(dmask) - 1;
            dmask &= dmask - 1;
            const int slot = __shfl_sync(FULL, done_slot, src);
            const long long v0 = (long long)r_chunk[slot] * p.chunk_tensors;
            const long long v1 = min(p.n_tensors, v0 + p.chunk_tensors);
            if constexpr (FUSED_MODE == 2) {
              bool ok = true;
#pragma unroll 1
              for (long long v = v0; v < v1 && ok; ++v) ok = warp_dedup128_regs<N, (M % 2) == 0>(p.dd, v, lane);
              if (!ok && lane == 0) p.ovf_list[atomicAdd(p.ovf_count, 1u)] = r_chunk[slot];   // > 32 clusters
            } else {
#pragma unroll 1
              for (long long v = v0; v < v1; ++v)
                warp_dedup_tensor<N, (M % 2) == 0>(p.dd, v, lane, d_lam, d_x, d_cid, d_clam, d_crep, d_cmult);
            }
            if (lane == 0) r_seq[slot] = -1;
            __syncwarp();
          } while (dmask);
          // the coefficient registers were dead during the dedup: rematerialise them
          Idx tv;
          if constexpr (WIDE) tv = item / (Idx)S_;
          else tv = fast_div(item, p.divS);
          cf.load(p.packed + tv * (Idx)(S::PW / 4));
        }
      }
      if (exhausted && __ballot_sync(FULL, has) == 0u) break;
    }

    // ---------------- SS-HOPM steps (Fig. 1), STEPS per refill check ----------------
#pragma unroll
    for (int rep = 0; rep < STEPS; ++rep)
      sshopm_step<M, N, SHIFT, true>(cf, xs, lam, lamp, k, conv, stop, has, alpha, la, ls, tol, maxit);
    __syncwarp();
  }
  if constexpr (WS) {                                      // every chunk of this warp has been published
    __threadfence_block();
    if (lane == 0) atomicAdd(wq + kWsQueue + 2, 1u);
  }

  if (p.total_iters) {
    unsigned long long ws = it_sum;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) ws += __shfl_xor_sync(0xffffffffu, ws, o);
    if (lane == 0) atomicAdd(p.total_iters, ws);
  }
}


// ----------------------------------------- solve kernel, schedule 8 (records) --
// Lane-owned work units for the records path (solve -> dedup without the raw per-start arrays).  A lane
// claims a unit of `unit` consecutive starts of one tensor (warp-aggregated atomic on p.counter), keeps the
// tensor's coefficient rows in its registers for the whole unit and, when its item stops, takes the
// unit's next start: the refill is one record store, one start load and a few selects (no coefficient
// reload, no item -> (tensor, start) arithmetic).  Each item leaves one record of REC4 float4s,
// (x_0 .. x_{n-1}, lambda if converged else NaN, 0 pad), at rec[(t * S + s) * REC4]: every store is a
// whole 16-byte vector (one L2 transaction), and for n = 3 the record is the lane's x registers plus one
// select.  Item indices are 32-bit (N * S < 2^32).  The per-lane arithmetic is sshopm_step, so the
// records carry bit for bit the values of the other schedules.
template <int N>
constexpr int rec4() { return (N + 1 + 3) / 4; }

struct RecParams {
  const float4* packed;      // [N][PW/4] (sshopm_pack_kernel)
  const float4* starts_n;    // [S][SST/4]
  float4* rec;               // [N][S][REC4]
  unsigned long long* total_iters;   // optional
  unsigned int* counter;     // unit counter (zeroed by the pack kernel)
  uint32_t n_units;          // N * units_per_tensor
  uint32_t units_per_tensor, unit, S;
  FastDiv div_upt;           // unit -> tensor
  float alpha, tol;
  const float* alpha_t;      // SHIFT == 3
  int maxit, refill_k;
};

template <int M, int N, int SHIFT>
__global__ void __launch_bounds__(256, Shape<M, N>::MINB)
sshopm_solve_rec_kernel(const RecParams p) {
#ifdef SSHOPM_REC_STEPS
  constexpr int STEPS = SSHOPM_REC_STEPS;
#else
  constexpr int STEPS = steps_per_trip<M, N>();
#endif
  constexpr int SST4 = round4(N) / 4;
  constexpr int R4 = rec4<N>();
  constexpr int IDLE = 0x7fffffff;
  const int lane = threadIdx.x & 31;
  const uint32_t ltmask = lanemask_lt();
  const uint32_t FULL = 0xffffffffu;
  const float alpha = (SHIFT == 2) ? -p.alpha : p.alpha;
  const float tol = p.tol;
  const int maxit = p.maxit;

  Coefs<M, N> cf;
  float2 xs[Shape<M, N>::NX];
#pragma unroll
  for (int i = 0; i < Shape<M, N>::NX; ++i) xs[i] = f2(0.f, 0.f);
  float lamp = 0.f, lam = 0.f;
  int k = IDLE;
  bool has = false, stop = true, conv = false;
  uint32_t item = 0, item_end = 0;   // current item t * S + s, end of the lane's unit
  uint32_t s = 0;                    // current start
  float la = 0.f, ls = 1.f;
  uint32_t it_sum = 0;
  bool exhausted = false;
  uint32_t k_eff = (uint32_t)p.refill_k;

  for (;;) {
    const uint32_t smask = __ballot_sync(FULL, stop);
    if ((uint32_t)__popc(smask) >= k_eff) {
      const bool wr = stop && has;
      if (wr) {                                          // the finished item's record
        float v[4 * R4];
#pragma unroll
        for (int j = 0; j < N; ++j) v[j] = xget<M, N>(xs, j);
        v[N] = conv ? lam : __int_as_float(0x7fffffff);
#pragma unroll
        for (int j = N + 1; j < 4 * R4; ++j) v[j] = 0.f;
        SSHOPM_CHECK(item < p.n_units / p.units_per_tensor * p.S && s < p.S && item < item_end);
        float4* r = p.rec + (size_t)item * R4;
#pragma unroll
        for (int i = 0; i < R4; ++i) r[i] = make_float4(v[4 * i], v[4 * i + 1], v[4 * i + 2], v[4 * i + 3]);
      }
      if (p.total_iters != nullptr) it_sum += wr ? (uint32_t)k : 0u;
      bool ok = wr && item + 1 < item_end;               // next start of the lane's unit
      item += ok ? 1u : 0u;
      s += ok ? 1u : 0u;
      const bool need = stop && !ok;                     // unit used up (or never had one)
      const uint32_t nmask = __ballot_sync(FULL, need);
      if (nmask != 0u && !exhausted) {                   // claim units for those lanes (one atomic per warp)
        const uint32_t nn = __popc(nmask);
        uint32_t base = 0;
        if (lane == 0) base = atomicAdd(p.counter, nn);
        base = __shfl_sync(FULL, base, 0);
        if (base + nn >= p.n_units || base + nn < base) exhausted = true;
        const uint32_t u = base + __popc(nmask & ltmask);
        if (need && u >= base && u < p.n_units) {
          const uint32_t t = fast_div(u, p.div_upt);
          SSHOPM_CHECK(t == u / p.units_per_tensor && t < p.n_units / p.units_per_tensor);
          s = (u - t * p.units_per_tensor) * p.unit;
          item = t * p.S + s;
          item_end = item + min(p.unit, p.S - s);
          cf.load(p.packed + (size_t)t * (Shape<M, N>::PW / 4));
          if constexpr (SHIFT == 3) {
            const float at = __ldg(p.alpha_t + t);
            ls = at >= 0.f ? 1.f : -1.f;
            la = fabsf(at);
          }
          ok = true;
        }
      }
      if (ok) {
        float v[4 * SST4];
#pragma unroll
        for (int i = 0; i < SST4; ++i) {
          const float4 q4 = ldg4(p.starts_n + s * SST4 + i);
          v[4 * i] = q4.x; v[4 * i + 1] = q4.y; v[4 * i + 2] = q4.z; v[4 * i + 3] = q4.w;
        }
#pragma unroll
        for (int i = 0; i < Shape<M, N>::NX; ++i) xs[i] = f2(v[2 * i], v[2 * i + 1]);
      }
      k = ok ? 0 : (stop ? IDLE : k);
      lamp = ok ? __int_as_float(0x7fffffff) : lamp;
      has = stop ? ok : has;
      if (exhausted) {                                   // idle lanes stay idle: count K beyond them
        const uint32_t idle = __popc(__ballot_sync(FULL, !has));
        if (idle == 32u) break;
        k_eff = min(32u, idle + (uint32_t)p.refill_k);
      }
    }
#pragma unroll
    for (int rep = 0; rep < STEPS; ++rep)
      sshopm_step<M, N, SHIFT, true>(cf, xs, lam, lamp, k, conv, stop, has, alpha, la, ls, tol, maxit);
    __syncwarp();
  }
  if (p.total_iters) {
    unsigned long long ws = it_sum;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) ws += __shfl_xor_sync(0xffffffffu, ws, o);
    if (lane == 0) atomicAdd(p.total_iters, ws);
  }
}

// ------------------------------------------------- solve kernel, schedule 6 --
// Item per lane with a branch-free refill (opt-in; measured 1.5% slower than schedule 1 at C2 with the
// same step, profiles/r2/solve_variants.md).  Each warp owns one chunk of
// consecutive items [c_next, c_end) at a time (items are tensor-major: item =
// t * S + s) and claims the next chunk from the global counter only when the
// current one is used up; the claim for the following chunk is issued one
// chunk ahead, so the atomic's latency is off the critical path.  A refill
// (once >= K lanes are stopped at a trip boundary) is straight-line predicated
// code: stores of the stopped lanes' results, rank = popc of the stopped
// lanes below, item = c_next + rank, one LDG.128 row load per 4 coefficient
// words and one start load.  Lanes beyond the chunk's remaining items go idle
// (k = IDLE) until the next refill.  Results are bitwise those of the other
// schedules (same per-step arithmetic, sshopm_step).
template <int M, int N, int SHIFT, bool WIDE>
__global__ void __launch_bounds__(256, Shape<M, N>::MINB)
sshopm_solve_lean_kernel(const SolveParams p) {
  constexpr int STEPS = steps_per_trip<M, N>();
  using S = Shape<M, N>;
  using Idx = typename std::conditional<WIDE, unsigned long long, uint32_t>::type;
  constexpr int SST4 = round4(N) / 4;
  constexpr int IDLE = 0x7fffffff;                       // k of a lane without an item (>= any maxit)

  const int lane = threadIdx.x & 31;
  const uint32_t ltmask = lanemask_lt();
  const uint32_t FULL = 0xffffffffu;
  const float alpha = (SHIFT == 2) ? -p.alpha : p.alpha;
  const float tol = p.tol;
  const int maxit = p.maxit;
  const uint32_t S_ = (uint32_t)p.S;
  const Idx total = (Idx)p.n_tensors * (Idx)S_;
  const Idx chunk_items = (Idx)p.chunk_tensors * (Idx)S_;
  const unsigned int n_chunks = (unsigned int)p.n_chunks;

  Idx c_next = 0, c_end = 0;                             // warp-uniform current chunk
  unsigned int pref = 0;                                 // next chunk index (claimed one chunk ahead)
  if (lane == 0) pref = atom_add1(p.counter);
  bool exhausted = false;
  uint32_t k_eff = (uint32_t)p.refill_k;

  Coefs<M, N> cf;
  float2 xs[S::NX];
#pragma unroll
  for (int i = 0; i < S::NX; ++i) xs[i] = f2(0.f, 0.f);
  float lamp = 0.f, lam = 0.f;
  int k = IDLE;
  bool stop = true, conv = false;
  Idx item = 0;
  float la = 0.f, ls = 1.f;
  uint32_t it_sum = 0;

  for (;;) {
    const uint32_t smask = __ballot_sync(FULL, stop);
    const uint32_t cnt = __popc(smask);
    if (cnt >= k_eff) {
      if (c_next == c_end && !exhausted) {               // warp-uniform: take the prefetched chunk, prefetch the next
        const unsigned int ch = __shfl_sync(FULL, pref, 0);
        if (ch < n_chunks) {
          c_next = (Idx)ch * chunk_items;
          c_end = c_next + chunk_items < total ? c_next + chunk_items : total;
          if (lane == 0) pref = atom_add1(p.counter);
        } else {
          exhausted = true;
          k_eff = 32u;
        }
      }
      // results of the lanes that stopped (A7): predicated stores
      const bool wr = stop && (k != IDLE);
      pst(wr, p.out_lambda + item, lam);
#pragma unroll
      for (int j = 0; j < N; ++j) pst(wr, p.out_x + (size_t)item * N + j, xget<M, N>(xs, j));
      pst(wr, p.out_iters + item, (int32_t)k);
      pst(wr, p.out_conv + item, conv ? 1u : 0u);
      it_sum += wr ? (uint32_t)k : 0u;
      // next items: rank among the stopped lanes, within the chunk's remaining items
      const uint32_t rank = __popc(smask & ltmask);
      const Idx avail = c_end - c_next;
      const bool ok = stop && (Idx)rank < avail;
      item = ok ? c_next + (Idx)rank : item;
      Idx tv;
      uint32_t s;
      if (p.s_log2 >= 0) {                               // S a power of two (the paper's 128): shift and mask
        tv = item >> p.s_log2;
        s = (uint32_t)item & p.s_mask;
      } else if constexpr (WIDE) {
        tv = item / S_;
        s = (uint32_t)(item - tv * S_);
      } else {
        tv = fast_div(item, p.divS);
        s = item - tv * S_;
      }
      if constexpr (SHIFT == 3) {
        float at = 0.f;
        if (ok) at = __ldg(p.alpha_t + tv);
        ls = ok ? (at >= 0.f ? 1.f : -1.f) : ls;         // Fig. 1 lines 2-5 (R5: alpha = 0 -> "+")
        la = ok ? fabsf(at) : la;
      }
      cf.load_if(ok, p.packed + tv * (Idx)(S::PW / 4));
      {
        float4 v[SST4];
#pragma unroll
        for (int i = 0; i < SST4; ++i) {
          v[i] = make_float4(xs[2 * i].x, xs[2 * i].y, (2 * i + 1 < S::NX) ? xs[2 * i + 1].x : 0.f,
                             (2 * i + 1 < S::NX) ? xs[2 * i + 1].y : 0.f);
          pld4(ok, p.starts_n + s * SST4 + i, v[i]);     // starts_n is in slot order
        }
#pragma unroll
        for (int i = 0; i < S::NX; ++i)
          xs[i] = (i % 2 == 0) ? f2(v[i / 2].x, v[i / 2].y) : f2(v[i / 2].z, v[i / 2].w);
      }
      lamp = ok ? __int_as_float(0x7fffffff) : lamp;     // NaN: the first test never fires (reading R2)
      k = stop ? (ok ? 0 : IDLE) : k;
      c_next += (Idx)cnt < avail ? (Idx)cnt : avail;
      if (exhausted && __ballot_sync(FULL, k != IDLE) == 0u) break;
    }
#pragma unroll
    for (int rep = 0; rep < STEPS; ++rep)
      sshopm_step<M, N, SHIFT, true>(cf, xs, lam, lamp, k, conv, stop, true, alpha, la, ls, tol, maxit);
  }

  if (p.total_iters) {
    unsigned long long ws = it_sum;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) ws += __shfl_xor_sync(0xffffffffu, ws, o);
    if (lane == 0) atomicAdd(p.total_iters, ws);
  }
}


// ------------------------------------------- solve kernel, tensor-per-lane --
// Schedule 2: a lane owns one tensor at a time and
// walks its S starts in order, so its coefficient registers are loaded once
// per S items and a refill only writes the finished item and loads the next
// start vector.  Lanes claim tensors individually (warp-aggregated atomic on
// the same counter); the per-step arithmetic is identical to schedule 1, so
// results are bitwise identical.
template <int M, int N, int SHIFT, bool WIDE>
__global__ void __launch_bounds__(256, Shape<M, N>::MINB)
sshopm_solve_tpl_kernel(const SolveParams p) {
  constexpr int STEPS = steps_per_trip<M, N>();
  using S = Shape<M, N>;
  using Idx = typename std::conditional<WIDE, long long, uint32_t>::type;
  constexpr int SST4 = round4(N) / 4;

  const int lane = threadIdx.x & 31;
  const uint32_t ltmask = lanemask_lt();
  const uint32_t FULL = 0xffffffffu;
  const float alpha = (SHIFT == 2) ? -p.alpha : p.alpha;
  const float tol = p.tol;
  const int maxit = p.maxit;
  const uint32_t S_ = (uint32_t)p.S;
  const Idx NT = (Idx)p.n_tensors;

  bool exhausted = false;
  Coefs<M, N> cf;
  float2 xs[S::NX];
#pragma unroll
  for (int i = 0; i < S::NX; ++i) xs[i] = f2(0.f, 0.f);
  float lamp = 0.f, lam = 0.f;
  int k = 0;
  bool has = false, stop = true, conv = false;
  Idx t = 0;                 // current tensor
  uint32_t s = S_;           // current start (S_ = needs a tensor)
  unsigned long long it_sum = 0;

  for (;;) {
    const uint32_t smask = __ballot_sync(FULL, stop);
    const uint32_t cnt = __popc(smask);
    if (cnt >= (uint32_t)p.refill_k || smask == FULL) {     // tensors may be exhausted; starts are not
      if (stop) {
        if (has) {
          const Idx item = t * (Idx)S_ + (Idx)s;
          p.out_lambda[item] = lam;
          float* ox = p.out_x + (size_t)item * N;
#pragma unroll
          for (int j = 0; j < N; ++j) ox[j] = xget<M, N>(xs, j);
          p.out_iters[item] = k;
          p.out_conv[item] = conv ? 1 : 0;
          it_sum += (unsigned long long)k;
          ++s;
        }
        has = false;
      }
      // lanes whose tensor is done claim the next tensors (one atomic per warp)
      const bool need = stop && s >= S_;
      const uint32_t nmask = __ballot_sync(FULL, need && !exhausted);
      if (nmask) {
        unsigned int base = 0;
        if (lane == __ffs(nmask) - 1) base = atomicAdd(p.counter, (unsigned int)__popc(nmask));
        base = __shfl_sync(FULL, base, __ffs(nmask) - 1);
        if (need && !exhausted) {
          const Idx nt = (Idx)base + (Idx)__popc(nmask & ltmask);
          if (nt < NT) {
            t = nt;
            s = 0;
            cf.load(p.packed + t * (Idx)(S::PW / 4));
          }
        }
        if ((long long)base + __popc(nmask) >= (long long)p.n_tensors) exhausted = true;
      }
      if (stop && s < S_) {                                  // next start of the lane's tensor
        has = true;
        float v[4 * SST4];
#pragma unroll
        for (int i = 0; i < SST4; ++i) {
          const float4 q4 = ldg4(p.starts_n + s * SST4 + i);
          v[4 * i] = q4.x; v[4 * i + 1] = q4.y; v[4 * i + 2] = q4.z; v[4 * i + 3] = q4.w;
        }
#pragma unroll
        for (int i = 0; i < S::NX; ++i) xs[i] = f2(v[2 * i], v[2 * i + 1]);   // starts_n is in slot order
        k = 0;
        lamp = __int_as_float(0x7fffffff);
      }
      if (__ballot_sync(FULL, has) == 0u) break;
    }

#pragma unroll
    for (int rep = 0; rep < STEPS; ++rep)
      sshopm_step<M, N, SHIFT>(cf, xs, lam, lamp, k, conv, stop, has, alpha, 0.f, 1.f, tol, maxit);
  }

  if (p.total_iters) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) it_sum += __shfl_xor_sync(0xffffffffu, it_sum, o);
    if (lane == 0) atomicAdd(p.total_iters, it_sum);
  }
}


// ---------------------------------------------------------- classify kernel --
constexpr int pair_row(int pr, int n) { int i = 0; while (pr >= n - i) { pr -= n - i; ++i; } return i; }
constexpr int pair_col(int pr, int n) { int i = 0; while (pr >= n - i) { pr -= n - i; ++i; } return i + pr; }

// Eigenpair type of each dedup record (reading R18): projected Hessian
// C = U^T [(m-1) A x^{m-2} - lam I] U on x-perp (Kolda-Mayo second-order test;
// fibre directions = local maxima).  U = the Householder
// reflection mapping e_k to x, minus column k.  Eigenvalues of C by cyclic
// Jacobi.  Codes: +1 max, -1 min, 0 saddle, 2 degenerate (|mu| <= ctol*max(1,|lam|)), 3 empty slot.
template <int M, int N>
__global__ void __launch_bounds__(128)
sshopm_classify_kernel(long long n_tensors, int kmax, const float* __restrict__ entries, const int32_t* __restrict__ count,
                       const float* __restrict__ lam_in, const float* __restrict__ x_in, float ctol,
                       int8_t* __restrict__ out) {
  using T2 = Tables2<M, N>;
  constexpr T2 T{};
  constexpr int U = Tables<M, N>::U;
  for (long long idx = (long long)blockIdx.x * blockDim.x + threadIdx.x; idx < n_tensors * kmax;
       idx += (long long)gridDim.x * blockDim.x) {
    const long long v = idx / kmax;
    const int slot = (int)(idx - v * kmax);
    if (slot >= count[v]) { out[idx] = 3; continue; }
    float a[U];
#pragma unroll
    for (int c = 0; c < U; ++c) a[c] = __ldg(entries + v * U + c);
    float x[N];
    float nx = 0.f;
#pragma unroll
    for (int j = 0; j < N; ++j) { x[j] = x_in[idx * N + j]; nx = fmaf(x[j], x[j], nx); }
    const float rx = rsqrtf(nx);
#pragma unroll
    for (int j = 0; j < N; ++j) x[j] *= rx;
    const float lam = lam_in[idx];
    // H = (m-1) A x^{m-2} - lam I
    float H[N][N];
#pragma unroll
    for (int i = 0; i < N; ++i)
#pragma unroll
      for (int j = 0; j < N; ++j) H[i][j] = 0.f;
    static_for<T2::Q2>([&](auto qq) {
      constexpr int q = decltype(qq)::value;
      float mono = (float)T.r_coef[q];
      static_for<T2::D2>([&](auto tt) {
        constexpr int t = decltype(tt)::value;
        constexpr int var = T.r_idx[q][t];
        mono *= x[var];
      });
      static_for<T2::NPR>([&](auto pp) {
        constexpr int pr = decltype(pp)::value;
        constexpr int cls = T.r_cls[q][pr];
        constexpr int i = pair_row(pr, N), j = pair_col(pr, N);
        H[i][j] = fmaf(mono, a[cls], H[i][j]);
      });
    });
#pragma unroll
    for (int i = 0; i < N; ++i) {
#pragma unroll
      for (int j = i; j < N; ++j) {
        H[i][j] *= (float)(M - 1);
        H[j][i] = H[i][j];
      }
      H[i][i] -= lam;
    }
    // Householder P = I - 2 w w^T / (w^T w), w = x + s e_k (s = sign x_k, k = argmax |x_k|): P e_k = -s x
    int kk = 0;
#pragma unroll
    for (int j = 1; j < N; ++j) kk = fabsf(x[j]) > fabsf(x[kk]) ? j : kk;
    float w[N];
    float ww = 0.f;
#pragma unroll
    for (int j = 0; j < N; ++j) {
      w[j] = x[j] + ((j == kk) ? (x[kk] >= 0.f ? 1.f : -1.f) : 0.f);
      ww = fmaf(w[j], w[j], ww);
    }
    const float beta = 2.f / ww;
    // B = P H P = H - beta w (H w)^T - beta (H w) w^T + beta^2 (w^T H w) w w^T
    float hw[N];
    float whw = 0.f;
#pragma unroll
    for (int i = 0; i < N; ++i) {
      float t = 0.f;
#pragma unroll
      for (int j = 0; j < N; ++j) t = fmaf(H[i][j], w[j], t);
      hw[i] = t;
      whw = fmaf(w[i], t, whw);
    }
    constexpr int R = N - 1;
    float Cm[R > 0 ? R : 1][R > 0 ? R : 1];
#pragma unroll
    for (int i = 0; i < R; ++i)
#pragma unroll
      for (int j = 0; j < R; ++j) {
        const int ii = i + (i >= kk), jj = j + (j >= kk);
        float hij = 0.f, wi = 0.f, wj = 0.f, hwi = 0.f, hwj = 0.f;
#pragma unroll
        for (int r2 = 0; r2 < N; ++r2) {
          if (r2 == ii) { wi = w[r2]; hwi = hw[r2]; }
          if (r2 == jj) { wj = w[r2]; hwj = hw[r2]; }
#pragma unroll
          for (int c2 = 0; c2 < N; ++c2)
            if (r2 == ii && c2 == jj) hij = H[r2][c2];
        }
        Cm[i][j] = hij - beta * wi * hwj - beta * hwi * wj + beta * beta * whw * wi * wj;
      }
    // cyclic Jacobi
#pragma unroll 1
    for (int sweep = 0; sweep < 12; ++sweep) {
#pragma unroll
      for (int p_ = 0; p_ < R; ++p_)
#pragma unroll
        for (int q_ = p_ + 1; q_ < R; ++q_) {
          const float apq = Cm[p_][q_];
          if (fabsf(apq) < 1e-30f) continue;
          const float theta = (Cm[q_][q_] - Cm[p_][p_]) / (2.f * apq);
          const float t = copysignf(1.f, theta) / (fabsf(theta) + sqrtf(theta * theta + 1.f));
          const float c = rsqrtf(t * t + 1.f), sn = t * c;
#pragma unroll
          for (int r2 = 0; r2 < R; ++r2) {
            const float crp = Cm[r2][p_], crq = Cm[r2][q_];
            Cm[r2][p_] = c * crp - sn * crq;
            Cm[r2][q_] = sn * crp + c * crq;
          }
#pragma unroll
          for (int r2 = 0; r2 < R; ++r2) {
            const float cpr = Cm[p_][r2], cqr = Cm[q_][r2];
            Cm[p_][r2] = c * cpr - sn * cqr;
            Cm[q_][r2] = sn * cpr + c * cqr;
          }
        }
    }
    const float thr = ctol * fmaxf(1.f, fabsf(lam));
    int npos = 0, nneg = 0, nzero = 0;
#pragma unroll
    for (int i = 0; i < R; ++i) {
      const float mu = Cm[i][i];
      nzero += fabsf(mu) <= thr;
      npos += mu > thr;
      nneg += mu < -thr;
    }
    int8_t code = 0;
    if (nzero) code = 2;
    else if (nneg == R) code = 1;
    else if (npos == R) code = -1;
    out[idx] = code;
  }
}

// ------------------------------------------------------------ apply kernel --
template <int M, int N>
__global__ void __launch_bounds__(256)
sshopm_apply_kernel(long long n_items, const float4* __restrict__ packed, const float* __restrict__ x,
                    float* __restrict__ out_g, float* __restrict__ out_lam) {
  using S = Shape<M, N>;
  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n_items; i += (long long)gridDim.x * blockDim.x) {
    Coefs<M, N> cf;
    cf.load(packed + i * (S::PW / 4));
    float2 xs[S::NX];
#pragma unroll
    for (int t = 0; t < S::NX; ++t) xs[t] = f2(0.f, 0.f);
#pragma unroll
    for (int j = 0; j < N; ++j) {
      const int sl = xslot<M, N>(j);
      if (sl & 1) xs[sl >> 1].y = __ldg(x + i * N + j);
      else xs[sl >> 1].x = __ldg(x + i * N + j);
    }
    if constexpr (X21<M, N>::v) xs[1].y = xs[0].y;
    float lam;
    if constexpr (N == 3 && SSHOPM_HORNER3 && M >= 6) {     // the solver's Horner evaluation (raw rows: integer
      float g0, g1, g2;                                     // weights instead of divided powers, exact on integers)
      horner3<M, true>(cf, xs[0].x, xs[0].y, xs[1].x, g0, g1, g2);
      lam = fmaf(xs[1].x, g2, fmaf(xs[0].y, g1, xs[0].x * g0));
      out_g[i * N + 0] = g0;
      out_g[i * N + 1] = g1;
      out_g[i * N + 2] = g2;
    } else if constexpr (SSHOPM_HORNERN && !Shape<M, N>::BFORM && N >= SSHOPM_HORNERN_MIN_N && N >= 4) {   // hornerN, integer weights
      float xv[N], g[N];
#pragma unroll
      for (int j = 0; j < N; ++j) xv[j] = xget<M, N>(xs, j);
      hornerN<M, N, true>(cf, xv, g);
      lam = 0.f;
#pragma unroll
      for (int j = 0; j < N; ++j) { out_g[i * N + j] = g[j]; lam = fmaf(xv[j], g[j], lam); }
    } else if constexpr (H43<M, N>::v) {
      float g0, g1, g2;
      horner43(cf, xs, g0, g1, g2);
      lam = fmaf(xs[1].x, g2, fmaf(xs[0].y, g1, xs[0].x * g0));
      out_g[i * N + 0] = g0;
      out_g[i * N + 1] = g1;
      out_g[i * N + 2] = g2;
    } else if constexpr (S43<M, N>::v) {
      float g0, g1, g2;
      lam = eval43s(cf, xs[0].x, xs[0].y, xs[1].x, g0, g1, g2);
      out_g[i * N + 0] = g0;
      out_g[i * N + 1] = g1;
      out_g[i * N + 2] = g2;
    } else if constexpr (N43<M, N>::v) {
      float2 g01;
      float g2;
      lam = eval43n(cf, xs, g01, g2);
      out_g[i * N + 0] = g01.x;
      out_g[i * N + 1] = g01.y;
      out_g[i * N + 2] = g2;
    } else if constexpr (X02<M, N>::v) {
      float g0, g1, g2;
      lam = eval43(cf, xs, g0, g1, g2);
      out_g[i * N + 0] = g0;
      out_g[i * N + 1] = g1;
      out_g[i * N + 2] = g2;
    } else {
      float2 gp[S::NP > 0 ? S::NP : 1];
      float gs = 0.f;
      lam = evaluate<M, N>(cf, xs, gp, gs);
      static_for<S::NP>([&](auto pp) {
        constexpr int q = decltype(pp)::value;
        out_g[i * N + 2 * q] = gp[q].x;
        out_g[i * N + 2 * q + 1] = gp[q].y;
      });
      if constexpr (S::ODD) out_g[i * N + N - 1] = gs;
    }
    out_lam[i] = lam;
  }
}

#include "sshopm_wt.cuh"

}  // namespace sshopm
