// Bare (4,3) step loop (the solve kernel's sshopm_step, 4 steps per trip, no refill): coefficient words
// in vector registers (per-lane rows, LDG) vs in uniform registers (constant bank, per-CTA row, LDCU).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 --expt-relaxed-constexpr \
//        -I../../paper_conf_ipps_ballardkp11_b200/csrc ur_step.cu -o ur_step
#include <cstdio>
#include <vector>
#include "sshopm_kernels.cuh"
using namespace sshopm;
constexpr int PW4 = Shape<4, 3>::PW / 4;
__constant__ float4 cb[512 * PW4];

template <bool UR>
__global__ void __launch_bounds__(128) loop(const float4* __restrict__ rows, const float4* __restrict__ st,
                                            float* out, int trips) {
  Coefs<4, 3> cf;
  const int r = UR ? (blockIdx.x & 511) : ((blockIdx.x * 128 + threadIdx.x) & 4095);
  if (UR) {
#pragma unroll
    for (int i = 0; i < PW4; ++i) cf.w[i] = cb[r * PW4 + i];
  } else {
    cf.load(rows + r * PW4);
  }
  const float4 s = st[threadIdx.x & 127];
  float2 xs[2] = {f2(s.x, s.y), f2(s.z, s.w)};
  float lam = 0.f, lamp = __int_as_float(0x7fffffff);
  int k = 0;
  bool conv = false, stop = false;
  for (int t = 0; t < trips; ++t) {
#pragma unroll
    for (int rep = 0; rep < 4; ++rep)
      sshopm_step<4, 3, 0, true>(cf, xs, lam, lamp, k, conv, stop, true, 0.f, 0.f, 1.f, -1.f, 0x7fffffff);
    __syncwarp();
  }
  out[blockIdx.x * 128 + threadIdx.x] = lam + xs[0].x + (float)k;
}

// two starts per lane on one coefficient set: contraction as scalar FFMA, start a then start b per
// (q, j), so the coefficient word is read once for both (operand reuse) and the two monomials alternate.
__device__ __forceinline__ void tail43(float g0, float g1, float g2, float2 (&xs)[2], float& lam, float& lamp, int& k,
                                       bool& stop, float tol, int maxit) {
  const float x0 = xs[0].x, x1 = xs[0].y, x2 = xs[1].x;
  lam = fmaf(x2, g2, fmaf(x1, g1, x0 * g0));
  const bool conv = fabsf(lam - lamp) <= tol * fmaxf(1.0f, fabsf(lam));
  const float nn = fmaf(g2, g2, fmaf(g1, g1, g0 * g0));
  const bool deg = !(nn >= 1.17549435e-38f);
  stop = conv | (k >= maxit) | deg;
  const float r = rsqrt_ftz(nn);
  if (!stop) {
    const float y1 = g1 * r;
    xs[0] = f2(g0 * r, y1);
    xs[1] = f2(g2 * r, y1);
    lamp = lam;
    ++k;
  }
}
template <int ORDER>
__device__ __forceinline__ void step2(const Coefs<4, 3>& cf, float2 (&xa)[2], float2 (&xb)[2], float& la, float& lb,
                                      float& lpa, float& lpb, int& ka, int& kb, bool& sa, bool& sb, float tol, int maxit) {
  float ma[10], mb[10];
  monomials<4, 3>(xa, ma);
  monomials<4, 3>(xb, mb);
  float a0, a1, a2, b0, b1, b2;
  a0 = cf.template word<0>() * ma[0]; b0 = cf.template word<0>() * mb[0];
  a1 = cf.template word<1>() * ma[0]; b1 = cf.template word<1>() * mb[0];
  a2 = cf.template word<20>() * ma[0]; b2 = cf.template word<20>() * mb[0];
  static_for<9>([&](auto qq) {
    constexpr int q = decltype(qq)::value + 1;
    a0 = fmaf(cf.template word<2 * q>(), ma[q], a0); b0 = fmaf(cf.template word<2 * q>(), mb[q], b0);
    a1 = fmaf(cf.template word<2 * q + 1>(), ma[q], a1); b1 = fmaf(cf.template word<2 * q + 1>(), mb[q], b1);
    a2 = fmaf(cf.template word<20 + q>(), ma[q], a2); b2 = fmaf(cf.template word<20 + q>(), mb[q], b2);
  });
  tail43(a0, a1, a2, xa, la, lpa, ka, sa, tol, maxit);
  tail43(b0, b1, b2, xb, lb, lpb, kb, sb, tol, maxit);
}

// Horner in x0 with shared (x1, x2) monomials: g_j = x0 (x0 (x0 B000 + B001 x1 + B002 x2) + Q_j) + C_j,
// Q_j = B011 x1^2 + B012 x1 x2 + B022 x2^2, C_j = B111 x1^3 + B112 x1^2 x2 + B122 x1 x2^2 + B222 x2^3:
// 36 FMA-type ops + 7 shared products per step (43 FP32 pipe ops) instead of 30 + 16.
template <int V>
__device__ __forceinline__ void steph(const Coefs<4, 3>& cf, float2 (&xs)[2], float& lam, float& lamp, int& k,
                                      bool& stop, float tol, int maxit) {
  const float x0 = xs[0].x, x1 = xs[0].y, x2 = xs[1].x;
  const float2 p21 = xs[1];                          // (x2, x1)
  const float2 s = __fmul2_rn(bc(x1), p21);          // (s12, s11)
  const float s22 = x2 * x2;
  const float2 c1 = __fmul2_rn(bc(s.y), p21);        // (c112, c111)
  const float2 c2 = __fmul2_rn(bc(s22), p21);        // (c222, c122)
  float g0, g1, g2;
  if constexpr (V == 0) {
    float gg[3];
    static_for<3>([&](auto jj) {
      constexpr int j = decltype(jj)::value;
      auto B = [&](auto qq) { constexpr int q = decltype(qq)::value; return j < 2 ? cf.template word<2 * q + (j < 2 ? j : 0)>() : cf.template word<20 + q>(); };
      float L = B(std::integral_constant<int, 1>{}) * x1;
      L = fmaf(B(std::integral_constant<int, 2>{}), x2, L);
      float t = fmaf(B(std::integral_constant<int, 0>{}), x0, L);
      float Q = B(std::integral_constant<int, 3>{}) * s.y;
      Q = fmaf(B(std::integral_constant<int, 4>{}), s.x, Q);
      Q = fmaf(B(std::integral_constant<int, 5>{}), s22, Q);
      t = fmaf(t, x0, Q);
      float C = B(std::integral_constant<int, 6>{}) * c1.y;
      C = fmaf(B(std::integral_constant<int, 7>{}), c1.x, C);
      C = fmaf(B(std::integral_constant<int, 8>{}), c2.y, C);
      C = fmaf(B(std::integral_constant<int, 9>{}), c2.x, C);
      gg[j] = fmaf(t, x0, C);
    });
    g0 = gg[0]; g1 = gg[1]; g2 = gg[2];
  } else {
    // (g0, g1) as FFMA2 on the B-form word pairs, g2 scalar
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
    g0 = g01.x; g1 = g01.y;
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
  lam = fmaf(x2, g2, fmaf(x1, g1, x0 * g0));
  const bool conv = fabsf(lam - lamp) <= tol * fmaxf(1.0f, fabsf(lam));
  const float nn = fmaf(g2, g2, fmaf(g1, g1, g0 * g0));
  const bool deg = !(nn >= 1.17549435e-38f);
  stop = conv | (k >= maxit) | deg;
  const float r = rsqrt_ftz(nn);
  if (!stop) {
    const float y1 = g1 * r;
    xs[0] = f2(g0 * r, y1);
    xs[1] = f2(g2 * r, y1);
    lamp = lam;
    ++k;
  }
}
template <int V>
__global__ void __launch_bounds__(128) looph(const float4* __restrict__ rows, const float4* __restrict__ st,
                                             float* out, int trips) {
  Coefs<4, 3> cf;
  const int r = (blockIdx.x * 128 + threadIdx.x) & 4095;
  cf.load(rows + r * PW4);
  const float4 s = st[threadIdx.x & 127];
  float2 xs[2] = {f2(s.x, s.y), f2(s.z, s.w)};
  float lam = 0.f, lamp = __int_as_float(0x7fffffff);
  int k = 0;
  bool stop = false;
  for (int t = 0; t < trips; ++t) {
#pragma unroll
    for (int rep = 0; rep < 4; ++rep) steph<V>(cf, xs, lam, lamp, k, stop, -1.f, 0x7fffffff);
    __syncwarp();
  }
  out[blockIdx.x * 128 + threadIdx.x] = lam + xs[0].x + (float)k;
}

__global__ void __launch_bounds__(128) loop2(const float4* __restrict__ rows, const float4* __restrict__ st,
                                             float* out, int trips) {
  Coefs<4, 3> cf;
  const int r = (blockIdx.x * 128 + threadIdx.x) & 4095;
  cf.load(rows + r * PW4);
  const float4 s = st[threadIdx.x & 127], s2 = st[(threadIdx.x + 1) & 127];
  float2 xa[2] = {f2(s.x, s.y), f2(s.z, s.w)}, xb[2] = {f2(s2.x, s2.y), f2(s2.z, s2.w)};
  float la = 0.f, lb = 0.f, lpa = __int_as_float(0x7fffffff), lpb = lpa;
  int ka = 0, kb = 0;
  bool sa = false, sb = false;
  for (int t = 0; t < trips; ++t) {
#pragma unroll
    for (int rep = 0; rep < 2; ++rep) step2<0>(cf, xa, xb, la, lb, lpa, lpb, ka, kb, sa, sb, -1.f, 0x7fffffff);
    __syncwarp();
  }
  out[blockIdx.x * 128 + threadIdx.x] = la + lb + xa[0].x + xb[0].x + (float)(ka + kb);
}

int main() {
  const int rowsN = 4096, trips = 2000;
  std::vector<float> h(rowsN * PW4 * 4), hs(128 * 4);
  unsigned s = 1;
  auto rnd = [&]() { s = s * 1664525u + 1013904223u; return (float)((s >> 8) & 0xffff) / 65536.f - 0.3f; };
  for (auto& v : h) v = rnd();
  for (int i = 0; i < 128; ++i) {
    float a = rnd(), b = rnd(), c = rnd(), n = sqrtf(a * a + b * b + c * c);
    hs[4 * i] = a / n; hs[4 * i + 1] = b / n; hs[4 * i + 2] = c / n; hs[4 * i + 3] = b / n;
  }
  float4 *rows, *st; float* out;
  cudaMalloc(&rows, h.size() * 4); cudaMalloc(&st, hs.size() * 4);
  cudaMemcpy(rows, h.data(), h.size() * 4, cudaMemcpyHostToDevice);
  cudaMemcpy(st, hs.data(), hs.size() * 4, cudaMemcpyHostToDevice);
  cudaMemcpyToSymbol(cb, h.data(), 512 * PW4 * 16);
  int sms = 0; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  for (int v = 0; v < 2; ++v) for (int bps : {8, 12, 16}) {
    const int grid = sms * bps;
    cudaMalloc(&out, grid * 128 * 4);
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    float best = 1e9;
    for (int rep = 0; rep < 5; ++rep) {
      cudaEventRecord(a);
      if (v == 0) looph<0><<<grid, 128>>>(rows, st, out, trips); else looph<1><<<grid, 128>>>(rows, st, out, trips);
      cudaEventRecord(b); cudaEventSynchronize(b);
      float ms; cudaEventElapsedTime(&ms, a, b); if (ms < best) best = ms;
    }
    const double steps = (double)grid * 128 * trips * 4;
    int occ = 0; if (v == 0) cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, looph<0>, 128, 0); else cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, looph<1>, 128, 0);
    printf("{\"variant\":\"horner_%s\",\"ctas_per_sm\":%d,\"max_ctas\":%d,\"ms\":%.4f,\"cycles_per_warp_step\":%.2f,\"frac_of_74.4\":%.4f,\"err\":\"%s\"}\n",
           v ? "ffma2_g01" : "scalar", bps, occ, best, best * 1e-3 * 1.965e9 * sms * 4 / (steps / 32), steps * 89.0 / (best * 1e-3) / 74.4e12,
           cudaGetErrorString(cudaGetLastError()));
    cudaFree(out);
  }
  for (int bps : {4, 6, 8, 12}) {
    const int grid = sms * bps;
    cudaMalloc(&out, grid * 128 * 4);
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    float best = 1e9;
    for (int rep = 0; rep < 5; ++rep) {
      cudaEventRecord(a);
      loop2<<<grid, 128>>>(rows, st, out, trips / 2);
      cudaEventRecord(b); cudaEventSynchronize(b);
      float ms; cudaEventElapsedTime(&ms, a, b); if (ms < best) best = ms;
    }
    const double steps = (double)grid * 128 * (trips / 2) * 2 * 2;
    int occ = 0; cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, loop2, 128, 0);
    printf("{\"variant\":\"two_starts_scalar\",\"ctas_per_sm\":%d,\"max_ctas\":%d,\"ms\":%.4f,\"cycles_per_warp_step\":%.2f,\"frac_of_74.4\":%.4f,\"err\":\"%s\"}\n",
           bps, occ, best, best * 1e-3 * 1.965e9 * sms * 4 / (steps / 32), steps * 89.0 / (best * 1e-3) / 74.4e12,
           cudaGetErrorString(cudaGetLastError()));
    cudaFree(out);
  }
  for (int ur = 0; ur < 2; ++ur) {
    for (int bps : {8, 12, 16}) {
      const int grid = sms * bps;
      cudaMalloc(&out, grid * 128 * 4);
      cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
      float best = 1e9;
      for (int rep = 0; rep < 5; ++rep) {
        cudaEventRecord(a);
        if (ur) loop<true><<<grid, 128>>>(rows, st, out, trips); else loop<false><<<grid, 128>>>(rows, st, out, trips);
        cudaEventRecord(b); cudaEventSynchronize(b);
        float ms; cudaEventElapsedTime(&ms, a, b); if (ms < best) best = ms;
      }
      const double steps = (double)grid * 128 * trips * 4;
      const double flops = steps * 89.0;
      int occ = 0;
      if (ur) cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, loop<true>, 128, 0);
      else cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, loop<false>, 128, 0);
      printf("{\"variant\":\"%s\",\"ctas_per_sm\":%d,\"max_ctas\":%d,\"ms\":%.4f,\"cycles_per_warp_step\":%.2f,\"frac_of_74.4\":%.4f,\"err\":\"%s\"}\n",
             ur ? "uniform_coef" : "vector_coef", bps, occ, best, best * 1e-3 * 1.965e9 * sms * 4 / (steps / 32), flops / (best * 1e-3) / 74.4e12,
             cudaGetErrorString(cudaGetLastError()));
      cudaFree(out);
    }
  }
  return 0;
}
