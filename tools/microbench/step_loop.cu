// Throughput of the (4,3) SS-HOPM step body alone (no refill, every lane
// busy for a fixed number of steps): the ceiling the solve kernel's main loop
// can reach, and variants of it.  Uses the library's own evaluate<4,3>.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 --expt-relaxed-constexpr \
//        -I../../paper_conf_ipps_ballardkp11_b200/csrc step_loop.cu -o step_loop
#include <cstdio>
#include <cstdlib>
#include <vector>
#include "sshopm_kernels.cuh"

using namespace sshopm;
constexpr int M = 4, N = 3;
using SH = Shape<M, N>;

// One SS-HOPM step (alpha = 0) of the solve kernel's main loop for state (xs, lamp, k, stop).
template <bool RAW>
__device__ __forceinline__ void step(const Coefs<M, N, !RAW ? SH::BFORM : false>& cf, float2 (&xs)[SH::NX], float& lamp,
                                     float& lam, int& k, bool& stop, float tol, int maxit) {
  float2 gp[SH::NP];
  float gs = 0.f;
  {
    float mq[SH::Q];
    monomials<M, N>(xs, mq);
    cf.contract(mq, gp, gs);
    const float2 t = __fmul2_rn(xs[0], gp[0]);
    lam = fmaf(xs[1].x, gs, t.x + t.y);
  }
  const float2 q = __fmul2_rn(gp[0], gp[0]);
  const float nn = fmaf(gs, gs, q.x + q.y);
  const float r = rsqrt_ftz(nn);
  const bool conv = fabsf(lam - lamp) <= tol * fmaxf(1.0f, fabsf(lam));
  const bool deg = !(nn >= 1.17549435e-38f);
  stop = conv || k >= maxit || deg;
  const float2 n01 = __fmul2_rn(gp[0], bc(r));
  const float n2 = gs * r;
  xs[0].x = stop ? xs[0].x : n01.x;
  xs[0].y = stop ? xs[0].y : n01.y;
  xs[1].x = stop ? xs[1].x : n2;
  xs[1].y = xs[0].y;
  lamp = stop ? lamp : lam;
  k += stop ? 0 : 1;
}


// q-paired contraction: acc_j = sum_t (B[2t][j], B[2t+1][j]) * (m_2t, m_2t+1); g_j = acc_j.x + acc_j.y.
// Consecutive FFMA2s share the monomial pair (operand reuse), so each reads 4 registers instead of 5-6.
__device__ __forceinline__ void mono_pairs43(const float2 (&xs)[2], float2 (&mp)[5]) {
  const float2 x01 = xs[0], x21 = xs[1];
  const float2 x12 = f2(x21.y, x21.x);
  const float2 s0 = __fmul2_rn(bc(x01.x), x01);
  const float2 s1 = __fmul2_rn(x01, x21);
  const float2 s2 = __fmul2_rn(bc(x21.x), x12);
  mp[0] = __fmul2_rn(bc(x01.x), s0);
  mp[1] = __fmul2_rn(bc(x01.x), s1);
  mp[2] = __fmul2_rn(bc(x01.x), s2);
  mp[3] = __fmul2_rn(bc(s1.y), x12);
  mp[4] = __fmul2_rn(bc(s2.y), x12);
}
template <int LAMP_SEL>
__device__ __forceinline__ void step_q(const float4 (&w)[8], float2 (&xs)[SH::NX], float& lamp, float& lam, int& k,
                                       bool& stop, float tol, int maxit) {
  float2 mp[5];
  mono_pairs43(xs, mp);
  float2 acc[3];
  static_for<5>([&](auto tt) {
    constexpr int t = decltype(tt)::value;
    static_for<3>([&](auto jj) {
      constexpr int j = decltype(jj)::value;
      constexpr int i = t * 3 + j;   // pair index
      const float2 b = (i % 2 == 0) ? f2(w[i / 2].x, w[i / 2].y) : f2(w[i / 2].z, w[i / 2].w);
      if constexpr (t == 0) acc[j] = __fmul2_rn(b, mp[t]);
      else acc[j] = __ffma2_rn(b, mp[t], acc[j]);
    });
  });
  const float g0 = acc[0].x + acc[0].y, g1 = acc[1].x + acc[1].y, g2 = acc[2].x + acc[2].y;
  const float2 g01 = f2(g0, g1);
  const float2 t2 = __fmul2_rn(xs[0], g01);
  lam = fmaf(xs[1].x, g2, t2.x + t2.y);
  const float2 q = __fmul2_rn(g01, g01);
  const float nn = fmaf(g2, g2, q.x + q.y);
  const float r = rsqrt_ftz(nn);
  const bool conv = fabsf(lam - lamp) <= tol * fmaxf(1.0f, fabsf(lam));
  const bool deg = !(nn >= 1.17549435e-38f);
  stop = conv || k >= maxit || deg;
  const float2 n01 = __fmul2_rn(g01, bc(r));
  const float n2 = g2 * r;
  xs[0].x = stop ? xs[0].x : n01.x;
  xs[0].y = stop ? xs[0].y : n01.y;
  xs[1].x = stop ? xs[1].x : n2;
  xs[1].y = xs[0].y;
  if constexpr (LAMP_SEL) lamp = stop ? lamp : lam;
  else lamp = lam;
  k += stop ? 0 : 1;
}


// Contraction variants on the B-form row (same words as Coefs::contract):
//   MODE 0: scalar FFMA, q outer / j inner (the monomial is the reused operand)
//   MODE 1: (g0,g1) FFMA2 with broadcast monomial, then g2 scalar FFMA on the same monomial
template <int MODE>
__device__ __forceinline__ void step_v(const Coefs<M, N, true>& cf, float2 (&xs)[SH::NX], float& lamp, float& lam,
                                       int& k, bool& stop, float tol, int maxit) {
  float mq[SH::Q];
  monomials<M, N>(xs, mq);
  constexpr int base = SH::Q * SH::NP * 2;
  float g0, g1, g2;
  float2 g01;
  static_for<SH::Q>([&](auto qq) {
    constexpr int q = decltype(qq)::value;
    if constexpr (MODE == 0) {
      if constexpr (q == 0) {
        g0 = cf.template word<0>() * mq[0]; g1 = cf.template word<1>() * mq[0]; g2 = cf.template word<base>() * mq[0];
      } else {
        g0 = fmaf(cf.template word<2 * q>(), mq[q], g0);
        g1 = fmaf(cf.template word<2 * q + 1>(), mq[q], g1);
        g2 = fmaf(cf.template word<base + q>(), mq[q], g2);
      }
    } else {
      if constexpr (q == 0) {
        g01 = __fmul2_rn(cf.template pair<0>(), bc(mq[0]));
        g2 = cf.template word<base>() * mq[0];
      } else {
        g01 = __ffma2_rn(cf.template pair<2 * q>(), bc(mq[q]), g01);
        g2 = fmaf(cf.template word<base + q>(), mq[q], g2);
      }
    }
  });
  if constexpr (MODE == 0) g01 = f2(g0, g1);
  const float2 t2 = __fmul2_rn(xs[0], g01);
  lam = fmaf(xs[1].x, g2, t2.x + t2.y);
  const float2 q2 = __fmul2_rn(g01, g01);
  const float nn = fmaf(g2, g2, q2.x + q2.y);
  const float r = rsqrt_ftz(nn);
  const bool conv = fabsf(lam - lamp) <= tol * fmaxf(1.0f, fabsf(lam));
  const bool deg = !(nn >= 1.17549435e-38f);
  stop = conv || k >= maxit || deg;
  const float2 n01 = __fmul2_rn(g01, bc(r));
  const float n2 = g2 * r;
  xs[0].x = stop ? xs[0].x : n01.x;
  xs[0].y = stop ? xs[0].y : n01.y;
  xs[1].x = stop ? xs[1].x : n2;
  xs[1].y = xs[0].y;
  lamp = stop ? lamp : lam;
  k += stop ? 0 : 1;
}


// The kernel's step with the freeze written as a guarded update (if-converted to predicated instructions).
__device__ __forceinline__ void step_p(const Coefs<M, N, true>& cf, float2 (&xs)[SH::NX], float& lamp, float& lam,
                                       int& k, bool& stop, float tol, int maxit) {
  float2 gp[SH::NP];
  float gs = 0.f;
  lam = evaluate<M, N>(cf, xs, gp, gs);
  const float2 q = __fmul2_rn(gp[0], gp[0]);
  const float nn = fmaf(gs, gs, q.x + q.y);
  const float r = rsqrt_ftz(nn);
  const bool conv = fabsf(lam - lamp) <= tol * fmaxf(1.0f, fabsf(lam));
  const bool deg = !(nn >= 1.17549435e-38f);
  stop = conv || k >= maxit || deg;
  if (!stop) {
    xs[0] = __fmul2_rn(gp[0], bc(r));
    xs[1] = f2(gs * r, xs[0].y);
    lamp = lam;
    ++k;
  }
}

// V 0: the kernel's step (B-form, conv test, selects, k);  1: without the stop logic;
//   3: raw-form contraction (scalar FFMA on class entries);  4: two items per lane sharing the coefficients
//   5: q-paired contraction;  6: q-paired, lambda_prev unconditional;  7/8: step_v MODE 0/1
// Two starts per lane vectorised ACROSS starts: every FP op is an FFMA2/FMUL2 on
// (start A, start B) with the B-form coefficient broadcast; stop logic per start.
__device__ __forceinline__ void step_x2(const Coefs<M, N, true>& cf, float2 (&X)[3], float2& lamp, float2& lam,
                                        int& kA, int& kB, bool& sA, bool& sB, float tol, int maxit) {
  const float2 s00 = __fmul2_rn(X[0], X[0]), s01 = __fmul2_rn(X[0], X[1]), s02 = __fmul2_rn(X[0], X[2]);
  const float2 s11 = __fmul2_rn(X[1], X[1]), s12 = __fmul2_rn(X[1], X[2]), s22 = __fmul2_rn(X[2], X[2]);
  const float2 mq[10] = {__fmul2_rn(X[0], s00), __fmul2_rn(X[0], s01), __fmul2_rn(X[0], s02), __fmul2_rn(X[0], s11),
                         __fmul2_rn(X[0], s12), __fmul2_rn(X[0], s22), __fmul2_rn(X[1], s11), __fmul2_rn(X[1], s12),
                         __fmul2_rn(X[1], s22), __fmul2_rn(X[2], s22)};
  constexpr int base = SH::Q * SH::NP * 2;
  float2 g0, g1, g2;
  static_for<SH::Q>([&](auto qq) {
    constexpr int q = decltype(qq)::value;
    if constexpr (q == 0) {
      g0 = __fmul2_rn(bc(cf.template word<0>()), mq[0]);
      g1 = __fmul2_rn(bc(cf.template word<1>()), mq[0]);
      g2 = __fmul2_rn(bc(cf.template word<base>()), mq[0]);
    } else {
      g0 = __ffma2_rn(bc(cf.template word<2 * q>()), mq[q], g0);
      g1 = __ffma2_rn(bc(cf.template word<2 * q + 1>()), mq[q], g1);
      g2 = __ffma2_rn(bc(cf.template word<base + q>()), mq[q], g2);
    }
  });
  lam = __ffma2_rn(X[2], g2, __ffma2_rn(X[1], g1, __fmul2_rn(X[0], g0)));
  const float2 nn = __ffma2_rn(g2, g2, __ffma2_rn(g1, g1, __fmul2_rn(g0, g0)));
  const float2 r = f2(rsqrt_ftz(nn.x), rsqrt_ftz(nn.y));
  const bool cA = fabsf(lam.x - lamp.x) <= tol * fmaxf(1.0f, fabsf(lam.x));
  const bool cB = fabsf(lam.y - lamp.y) <= tol * fmaxf(1.0f, fabsf(lam.y));
  sA = cA | (kA >= maxit) | !(nn.x >= 1.17549435e-38f);
  sB = cB | (kB >= maxit) | !(nn.y >= 1.17549435e-38f);
  const float2 n0 = __fmul2_rn(g0, r), n1 = __fmul2_rn(g1, r), n2 = __fmul2_rn(g2, r);
  if (!sA) { X[0].x = n0.x; X[1].x = n1.x; X[2].x = n2.x; lamp.x = lam.x; ++kA; }
  if (!sB) { X[0].y = n0.y; X[1].y = n1.y; X[2].y = n2.y; lamp.y = lam.y; ++kB; }
}

template <int V, int MINB>
__global__ void __launch_bounds__(256, MINB) step_kernel(const float4* packed, float* out, int iters, int maxit) {
  const int t = blockIdx.x * blockDim.x + threadIdx.x;
  Coefs<M, N, V == 3 ? false : SH::BFORM> cf;   // V 5/6 reinterpret the 32 words in q-pair layout
  cf.load(packed + (t & 4095) * (SH::PW / 4));
  float2 xs[SH::NX], xs2[SH::NX];
  const float a = 0.3f + 1e-4f * (t & 63), b = 0.5f, c = 0.81f;
  const float r0 = rsqrtf(a * a + b * b + c * c);
  xs[0] = f2(a * r0, b * r0);
  xs[1] = f2(c * r0, b * r0);
  xs2[0] = f2(b * r0, a * r0);
  xs2[1] = f2(-c * r0, a * r0);
  float lamp = __int_as_float(0x7fffffff), lam = 0.f, lamp2 = lamp, lam2 = 0.f;
  int k = 0, k2 = 0;
  bool stop = false, stop2 = false;
  const float tol = 0.f;
  float2 X2[3] = {f2(xs[0].x, xs2[0].x), f2(xs[0].y, xs2[0].y), f2(xs[1].x, xs2[1].x)};
  float2 lamp_x2 = f2(lamp, lamp2), lam_x2 = f2(0.f, 0.f);
  for (int it = 0; it < iters; ++it) {
    if constexpr (V == 10) {
      step_x2(cf, X2, lamp_x2, lam_x2, k, k2, stop, stop2, tol, maxit);
    } else if constexpr (V == 1) {
      float2 gp[SH::NP];
      float gs = 0.f;
      lam = evaluate<M, N>(cf, xs, gp, gs);
      const float2 q = __fmul2_rn(gp[0], gp[0]);
      const float r = rsqrt_ftz(fmaf(gs, gs, q.x + q.y));
      const float2 n01 = __fmul2_rn(gp[0], bc(r));
      xs[0] = n01;
      xs[1].x = gs * r;
      xs[1].y = n01.y;
      lamp = lam;
    } else if constexpr (V == 4) {
      step<false>(cf, xs, lamp, lam, k, stop, tol, maxit);
      step<false>(cf, xs2, lamp2, lam2, k2, stop2, tol, maxit);
    } else if constexpr (V == 9) {
      step_p(cf, xs, lamp, lam, k, stop, tol, maxit);
    } else if constexpr (V == 7 || V == 8) {
      step_v<V - 7>(cf, xs, lamp, lam, k, stop, tol, maxit);
    } else if constexpr (V == 5 || V == 6) {
      step_q<V == 5>(cf.w, xs, lamp, lam, k, stop, tol, maxit);
    } else {
      step<V == 3>(cf, xs, lamp, lam, k, stop, tol, maxit);
    }
  }
  float o = lam + xs[0].x + (float)k + (stop ? 1.f : 0.f) + (V == 10 ? 0.f : lamp);
  if constexpr (V == 10) o += lam_x2.x + lam_x2.y + X2[0].x + X2[2].y + lamp_x2.x + lamp_x2.y + (float)k2 + (stop2 ? 1.f : 0.f);
  if constexpr (V == 4) o += lam2 + xs2[0].y + (float)k2 + lamp2 + (stop2 ? 1.f : 0.f);
  out[t] = o;
}

template <int V, int MINB>
void run(const char* name, const float4* packed, float* out, int sms, int ctas) {
  const int iters = 4000;
  const int grid = sms * ctas;
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0); cudaEventCreate(&e1);
  step_kernel<V, MINB><<<grid, 256>>>(packed, out, iters, 1 << 30);
  cudaEventRecord(e0);
  for (int r = 0; r < 5; ++r) step_kernel<V, MINB><<<grid, 256>>>(packed, out, iters, 1 << 30);
  cudaEventRecord(e1);
  cudaEventSynchronize(e1);
  float ms; cudaEventElapsedTime(&ms, e0, e1);
  ms /= 5;
  const double flops = (V == 4 || V == 10 ? 2 : 1) * 89.0 * iters * (double)grid * 256;
  cudaFuncAttributes fa; cudaFuncGetAttributes(&fa, step_kernel<V, MINB>);
  printf("{\"variant\":\"%s\",\"ctas_per_sm\":%d,\"regs\":%d,\"ms\":%.4f,\"tflops_alg\":%.2f,\"frac_of_74.4\":%.3f}\n",
         name, ctas, fa.numRegs, ms, flops / ms / 1e9, flops / ms / 1e9 / 74.4);
}

int main() {
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  std::vector<float> h(4096 * SH::PW);
  srand(1);
  for (auto& v : h) v = (rand() / (float)RAND_MAX - 0.5f);
  float4* packed; float* out;
  cudaMalloc(&packed, h.size() * 4);
  cudaMemcpy(packed, h.data(), h.size() * 4, cudaMemcpyHostToDevice);
  cudaMalloc(&out, sms * 8 * 256 * 4);
  run<0, 4>("kernel_step", packed, out, sms, 4);
  run<9, 4>("predicated_update", packed, out, sms, 4);
  run<10, 4>("two_starts_ffma2_across_starts", packed, out, sms, 4);
  run<10, 3>("two_starts_ffma2_across_starts", packed, out, sms, 3);
  run<10, 2>("two_starts_ffma2_across_starts", packed, out, sms, 2);
  run<0, 2>("kernel_step", packed, out, sms, 2);
  run<0, 4>("kernel_step", packed, out, sms, 3);
  run<1, 4>("no_stop_logic", packed, out, sms, 4);
  run<5, 4>("q_paired_contraction", packed, out, sms, 4);
  run<6, 4>("q_paired_lamp_uncond", packed, out, sms, 4);
  run<9, 4>("predicated_update", packed, out, sms, 4);
  run<7, 4>("bform_scalar_ffma_q_outer", packed, out, sms, 4);
  run<8, 4>("bform_ffma2_pair_plus_scalar_g2", packed, out, sms, 4);
  run<3, 4>("raw_form_scalar_ffma", packed, out, sms, 4);
  run<4, 4>("two_items_per_lane", packed, out, sms, 4);
  run<4, 2>("two_items_per_lane", packed, out, sms, 2);
  cudaError_t e = cudaDeviceSynchronize();
  printf("{\"status\":\"%s\"}\n", cudaGetErrorString(e));
  return 0;
}
