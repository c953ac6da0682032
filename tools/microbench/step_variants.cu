// Step-body variants for (4,3), alpha = 0, all with the solve kernel's
// predicated freeze: how the contraction's operand pattern and the
// dependency-chain shape move the refill-free step throughput on B200.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 --expt-relaxed-constexpr \
//        -I../../paper_conf_ipps_ballardkp11_b200/csrc step_variants.cu -o step_variants
#include <cstdio>
#include <cstdlib>
#include <vector>
#include "sshopm_kernels.cuh"

using namespace sshopm;
constexpr int M = 4, N = 3;
using SH = Shape<M, N>;

// common tail: lambda, ||g||, stop test, predicated update (as sshopm_step)
__device__ __forceinline__ void tail(float2 g01, float g2, float2 (&xs)[2], float& lamp, int& k, bool& stop,
                                     float tol, int maxit) {
  const float2 t = __fmul2_rn(xs[0], g01);
  const float lam = fmaf(xs[1].x, g2, t.x + t.y);
  const float2 q = __fmul2_rn(g01, g01);
  const float nn = fmaf(g2, g2, q.x + q.y);
  const bool conv = fabsf(lam - lamp) <= tol * fmaxf(1.0f, fabsf(lam));
  const bool deg = !(nn >= 1.17549435e-38f);
  stop = conv | (k >= maxit) | deg;
  const float r = rsqrt_ftz(nn);
  if (!stop) {
    xs[0] = __fmul2_rn(g01, bc(r));
    xs[1] = f2(g2 * r, xs[0].y);
    lamp = lam;
    ++k;
  }
}

// V0: the library step (sshopm_step<4,3,0>)
// V1: scalar FFMA, q outer (monomial reused by 3 consecutive FFMAs)
// V2: q-paired FFMA2 for all 3 outputs (monomial pair reused by 3 consecutive FFMA2s)
// V3: (g0,g1) FFMA2 in two interleaved chains (even/odd q) + g2 q-paired
// V4: (g0,g1) FFMA2 + g2 scalar FFMA on the same monomial, adjacent
template <int V>
__device__ __forceinline__ void step(const Coefs<M, N>& cf, float2 (&xs)[2], float& lamp, float& lam, int& k,
                                     bool& stop, float tol, int maxit) {
  constexpr int base = SH::Q * SH::NP * 2;   // 20: start of the g2 words
  if constexpr (V == 0) {
    bool conv;
    sshopm_step<M, N, 0>(cf, xs, lam, lamp, k, conv, stop, true, 0.f, 0.f, 1.f, tol, maxit);
    return;
  } else {
    float mq[10];
    monomials<M, N>(xs, mq);
    float2 g01;
    float g2;
    if constexpr (V == 1) {
      float g0, g1;
      static_for<10>([&](auto qq) {
        constexpr int q = decltype(qq)::value;
        const float2 b = cf.template pair<2 * q>();
        const float c = cf.template word<base + q>();
        if constexpr (q == 0) { g0 = b.x * mq[0]; g1 = b.y * mq[0]; g2 = c * mq[0]; }
        else { g0 = fmaf(b.x, mq[q], g0); g1 = fmaf(b.y, mq[q], g1); g2 = fmaf(c, mq[q], g2); }
      });
      g01 = f2(g0, g1);
    } else if constexpr (V == 2) {
      // words reinterpreted: pair index 3t + j holds (B_{2t,j}, B_{2t+1,j}) (throughput only)
      float2 a0, a1, a2;
      static_for<5>([&](auto tt) {
        constexpr int t = decltype(tt)::value;
        const float2 mp = f2(mq[2 * t], mq[2 * t + 1]);
        const float2 b0 = cf.template pair<2 * (3 * t + 0)>();
        const float2 b1 = cf.template pair<2 * (3 * t + 1)>();
        const float2 b2 = (3 * t + 2 < 15) ? cf.template pair<2 * ((3 * t + 2) % 15)>() : f2(0.f, 0.f);
        if constexpr (t == 0) { a0 = __fmul2_rn(b0, mp); a1 = __fmul2_rn(b1, mp); a2 = __fmul2_rn(b2, mp); }
        else { a0 = __ffma2_rn(b0, mp, a0); a1 = __ffma2_rn(b1, mp, a1); a2 = __ffma2_rn(b2, mp, a2); }
      });
      g01 = f2(a0.x + a0.y, a1.x + a1.y);
      g2 = a2.x + a2.y;
    } else if constexpr (V == 3) {
      float2 e = __fmul2_rn(cf.template pair<0>(), bc(mq[0]));
      float2 o = __fmul2_rn(cf.template pair<2>(), bc(mq[1]));
      static_for<4>([&](auto tt) {
        constexpr int t = decltype(tt)::value + 1;
        e = __ffma2_rn(cf.template pair<4 * t>(), bc(mq[2 * t]), e);
        o = __ffma2_rn(cf.template pair<4 * t + 2>(), bc(mq[2 * t + 1]), o);
      });
      g01 = __fadd2_rn(e, o);
      float2 h = __fmul2_rn(cf.template pair<base>(), f2(mq[0], mq[1]));
      static_for<4>([&](auto tt) {
        constexpr int t = decltype(tt)::value + 1;
        h = __ffma2_rn(cf.template pair<base + 2 * t>(), f2(mq[2 * t], mq[2 * t + 1]), h);
      });
      g2 = h.x + h.y;
    } else {
      static_for<10>([&](auto qq) {
        constexpr int q = decltype(qq)::value;
        if constexpr (q == 0) { g01 = __fmul2_rn(cf.template pair<0>(), bc(mq[0])); g2 = cf.template word<base>() * mq[0]; }
        else { g01 = __ffma2_rn(cf.template pair<2 * q>(), bc(mq[q]), g01); g2 = fmaf(cf.template word<base + q>(), mq[q], g2); }
      });
    }
    tail(g01, g2, xs, lamp, k, stop, tol, maxit);
  }
}


// V5: two items of the same tensor in the two halves of every float2 (item-pair SIMD):
// coefficients broadcast, monomials / accumulators / x as (item A, item B) pairs.
// Per-item operation order matches the library step (bitwise-identical results).
__device__ __forceinline__ void step_pair(const Coefs<M, N>& cf, float2 (&X)[3], float2& lamp, int& kA, int& kB,
                                          bool& stopA, bool& stopB, float tol, int maxit) {
  constexpr int base = SH::Q * SH::NP * 2;
  const float2 x0 = X[0], x1 = X[1], x2 = X[2];
  // monomials (lex order of Tables<4,3>): 000 001 002 011 012 022 111 112 122 222
  const float2 s00 = __fmul2_rn(x0, x0), s01 = __fmul2_rn(x0, x1), s02 = __fmul2_rn(x0, x2);
  const float2 s11 = __fmul2_rn(x1, x1), s12 = __fmul2_rn(x2, x1), s22 = __fmul2_rn(x2, x2);
  float2 mq[10];
  mq[0] = __fmul2_rn(x0, s00); mq[1] = __fmul2_rn(x0, s01); mq[2] = __fmul2_rn(x0, s02); mq[3] = __fmul2_rn(x0, s11);
  mq[4] = __fmul2_rn(x0, s12); mq[5] = __fmul2_rn(x0, s22); mq[6] = __fmul2_rn(s11, x1); mq[7] = __fmul2_rn(s11, x2);
  mq[8] = __fmul2_rn(s22, x1); mq[9] = __fmul2_rn(s22, x2);
  float2 g0, g1, hx, hy;
  static_for<10>([&](auto qq) {
    constexpr int q = decltype(qq)::value;
    const float2 b = cf.template pair<2 * q>();
    if constexpr (q == 0) { g0 = __fmul2_rn(bc(b.x), mq[0]); g1 = __fmul2_rn(bc(b.y), mq[0]); }
    else { g0 = __ffma2_rn(bc(b.x), mq[q], g0); g1 = __ffma2_rn(bc(b.y), mq[q], g1); }
  });
  static_for<5>([&](auto tt) {
    constexpr int t = decltype(tt)::value;
    const float2 b = cf.template pair<base + 2 * t>();
    if constexpr (t == 0) { hx = __fmul2_rn(bc(b.x), mq[0]); hy = __fmul2_rn(bc(b.y), mq[1]); }
    else { hx = __ffma2_rn(bc(b.x), mq[2 * t], hx); hy = __ffma2_rn(bc(b.y), mq[2 * t + 1], hy); }
  });
  const float2 g2 = __fadd2_rn(hx, hy);
  const float2 t0 = __fmul2_rn(x0, g0), t1 = __fmul2_rn(x1, g1);
  const float2 lam = __ffma2_rn(x2, g2, __fadd2_rn(t0, t1));
  const float2 q0 = __fmul2_rn(g0, g0), q1 = __fmul2_rn(g1, g1);
  const float2 nn = __ffma2_rn(g2, g2, __fadd2_rn(q0, q1));
  const float2 d = __fadd2_rn(lam, f2(-lamp.x, -lamp.y));
  const bool convA = fabsf(d.x) <= tol * fmaxf(1.0f, fabsf(lam.x));
  const bool convB = fabsf(d.y) <= tol * fmaxf(1.0f, fabsf(lam.y));
  stopA = convA | (kA >= maxit) | !(nn.x >= 1.17549435e-38f);
  stopB = convB | (kB >= maxit) | !(nn.y >= 1.17549435e-38f);
  const float2 r = f2(rsqrt_ftz(nn.x), rsqrt_ftz(nn.y));
  const float2 y0 = __fmul2_rn(g0, r), y1 = __fmul2_rn(g1, r), y2 = __fmul2_rn(g2, r);
  if (!stopA) { X[0].x = y0.x; X[1].x = y1.x; X[2].x = y2.x; lamp.x = lam.x; ++kA; }
  if (!stopB) { X[0].y = y0.y; X[1].y = y1.y; X[2].y = y2.y; lamp.y = lam.y; ++kB; }
}

template <int MINB>
__global__ void __launch_bounds__(256, MINB) pair_kernel(const float4* packed, float* out, int iters, int maxit) {
  const int t = blockIdx.x * blockDim.x + threadIdx.x;
  Coefs<M, N> cf;
  cf.load(packed + (t & 4095) * (SH::PW / 4));
  const float a = 0.3f + 1e-4f * (t & 63), b = 0.5f, c = 0.81f;
  const float r0 = rsqrtf(a * a + b * b + c * c);
  float2 X[3] = {f2(a * r0, b * r0), f2(b * r0, a * r0), f2(c * r0, -c * r0)};
  float2 lamp = f2(__int_as_float(0x7fffffff), __int_as_float(0x7fffffff));
  int kA = 0, kB = 0;
  bool sA = false, sB = false;
  for (int it = 0; it < iters; ++it) step_pair(cf, X, lamp, kA, kB, sA, sB, 0.f, maxit);
  out[t] = lamp.x + lamp.y + X[0].x + X[2].y + (float)(kA + kB) + (sA ? 1.f : 0.f) + (sB ? 1.f : 0.f);
}

template <int MINB>
void run_pair(const char* name, const float4* packed, float* out, int sms, int ctas) {
  const int iters = 2000;   // x 2 items per lane
  const int grid = sms * ctas;
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0); cudaEventCreate(&e1);
  pair_kernel<MINB><<<grid, 256>>>(packed, out, iters, 1 << 30);
  cudaEventRecord(e0);
  for (int r = 0; r < 5; ++r) pair_kernel<MINB><<<grid, 256>>>(packed, out, iters, 1 << 30);
  cudaEventRecord(e1);
  cudaEventSynchronize(e1);
  float ms; cudaEventElapsedTime(&ms, e0, e1);
  ms /= 5;
  const double lane_steps = 2.0 * iters * grid * 256;   // item-steps
  const double flops = 89.0 * lane_steps;
  cudaFuncAttributes fa; cudaFuncGetAttributes(&fa, pair_kernel<MINB>);
  const double cyc = 1.965e9 * ms * 1e-3 * sms * 4 / (lane_steps / 32);
  printf("{\"variant\":\"%s\",\"ctas_per_sm\":%d,\"regs\":%d,\"ms\":%.4f,\"frac_of_74.4\":%.3f,\"smsp_cycles_per_warp_step\":%.1f}\n",
         name, ctas, fa.numRegs, ms, flops / ms / 1e9 / 74.4, cyc);
}

template <int V, int MINB>
__global__ void __launch_bounds__(256, MINB) step_kernel(const float4* packed, float* out, int iters, int maxit) {
  const int t = blockIdx.x * blockDim.x + threadIdx.x;
  Coefs<M, N> cf;
  cf.load(packed + (t & 4095) * (SH::PW / 4));
  float2 xs[2];
  const float a = 0.3f + 1e-4f * (t & 63), b = 0.5f, c = 0.81f;
  const float r0 = rsqrtf(a * a + b * b + c * c);
  xs[0] = f2(a * r0, b * r0);
  xs[1] = f2(c * r0, b * r0);
  float lamp = __int_as_float(0x7fffffff), lam = 0.f;
  int k = 0;
  bool stop = false;
  const float tol = 0.f;
  for (int it = 0; it < iters; ++it) step<V>(cf, xs, lamp, lam, k, stop, tol, maxit);
  out[t] = lam + lamp + xs[0].x + xs[1].x + (float)k + (stop ? 1.f : 0.f);
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
  const double lane_steps = (double)iters * grid * 256;
  const double flops = 89.0 * lane_steps;
  cudaFuncAttributes fa; cudaFuncGetAttributes(&fa, step_kernel<V, MINB>);
  const double cyc = 1.965e9 * ms * 1e-3 * sms * 4 / (lane_steps / 32);   // SMSP cycles per warp-step
  printf("{\"variant\":\"%s\",\"ctas_per_sm\":%d,\"regs\":%d,\"ms\":%.4f,\"frac_of_74.4\":%.3f,\"smsp_cycles_per_warp_step\":%.1f}\n",
         name, ctas, fa.numRegs, ms, flops / ms / 1e9 / 74.4, cyc);
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
  run<0, 4>("library_step", packed, out, sms, 4);
  run<1, 4>("scalar_q_outer", packed, out, sms, 4);
  run<2, 4>("q_paired_all", packed, out, sms, 4);
  run<3, 4>("two_chain_g01_qpair_g2", packed, out, sms, 4);
  run<4, 4>("ffma2_g01_scalar_g2", packed, out, sms, 4);
  run<0, 2>("library_step", packed, out, sms, 2);
  run<1, 2>("scalar_q_outer", packed, out, sms, 2);
  run_pair<4>("item_pair_simd", packed, out, sms, 4);
  run_pair<3>("item_pair_simd", packed, out, sms, 3);
  run_pair<2>("item_pair_simd", packed, out, sms, 2);
  cudaError_t e = cudaDeviceSynchronize();
  printf("{\"status\":\"%s\"}\n", cudaGetErrorString(e));
  return 0;
}
