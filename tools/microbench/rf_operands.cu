// Register-file operand cost of FFMA2 / FFMA patterns on sm_100a: each
// pattern runs 8 independent accumulator chains; throughput relative to the
// FP32 peak tells how many cycles one instruction holds the issue port.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 rf_operands.cu -o rf_operands
#include <cstdio>
#include <cuda_runtime.h>

__constant__ float2 cB[16];

__device__ __forceinline__ float2 f2(float a, float b) { return make_float2(a, b); }
__device__ __forceinline__ float2 bc(float a) { return make_float2(a, a); }

// P 0: ffma2(B_i pair, bc(m) same m, acc_i)        1: ffma2(B_i, pair M same, acc_i)
//   2: ffma2(B_i, bc(m_i) distinct, acc_i)          3: ffma2(B_i, C_i pair distinct, acc_i)
//   4: ffma(b_i, m same, acc_i)                     5: ffma(b_i, m_i distinct, acc_i)
//   6: ffma2(constant-bank pair, bc(m_i), acc_i)    7: ffma(constant-bank, m_i, acc_i)
//   8: ffma2(acc_i, bc(m) same, B_i) (acc as A)     9: fmul2(B_i, bc(m_i))  (2 sources)
template <int P>
__global__ void __launch_bounds__(256, 4) k(float* out, const float* in, int iters) {
  const int t = blockIdx.x * blockDim.x + threadIdx.x;
  float2 B[8], C[8], acc[8];
  float m[8];
#pragma unroll
  for (int i = 0; i < 8; ++i) {
    B[i] = f2(in[(t + i) & 1023], in[(t + 3 * i + 1) & 1023]);
    C[i] = f2(in[(t + 5 * i + 2) & 1023], in[(t + 7 * i + 3) & 1023]);
    m[i] = in[(t + 11 * i + 4) & 1023];
    acc[i] = f2(0.f, 0.f);
  }
  float2 M = f2(m[0], m[1]);
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int r = 0; r < 4; ++r) {
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        if constexpr (P == 0) acc[i] = __ffma2_rn(B[i], bc(m[r]), acc[i]);
        else if constexpr (P == 1) acc[i] = __ffma2_rn(B[i], M, acc[i]);
        else if constexpr (P == 2) acc[i] = __ffma2_rn(B[i], bc(m[(i + r) & 7]), acc[i]);
        else if constexpr (P == 3) acc[i] = __ffma2_rn(B[i], C[(i + r) & 7], acc[i]);
        else if constexpr (P == 4) { acc[i].x = fmaf(B[i].x, m[r], acc[i].x); }
        else if constexpr (P == 5) { acc[i].x = fmaf(B[i].x, m[(i + r) & 7], acc[i].x); }
        else if constexpr (P == 6) acc[i] = __ffma2_rn(cB[(i + 8 * r) & 15], bc(m[(i + r) & 7]), acc[i]);
        else if constexpr (P == 7) { acc[i].x = fmaf(cB[(i + 8 * r) & 15].x, m[(i + r) & 7], acc[i].x); }
        else if constexpr (P == 8) acc[i] = __ffma2_rn(acc[i], bc(m[r]), B[i]);
        else if constexpr (P == 9) acc[i] = __fmul2_rn(acc[i], bc(m[(i + r) & 7]));
      }
    }
#pragma unroll
    for (int i = 0; i < 8; ++i) m[i] = m[i] * 0.999f;   // keep m live
  }
  float s = 0.f;
#pragma unroll
  for (int i = 0; i < 8; ++i) s += acc[i].x + acc[i].y;
  out[t] = s;
}

template <int P>
void run(const char* name, float* out, const float* in, int sms, bool packed) {
  const int iters = 20000, grid = sms * 4;
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0); cudaEventCreate(&e1);
  k<P><<<grid, 256>>>(out, in, 100);
  cudaEventRecord(e0);
  k<P><<<grid, 256>>>(out, in, iters);
  cudaEventRecord(e1);
  cudaEventSynchronize(e1);
  float ms; cudaEventElapsedTime(&ms, e0, e1);
  // lane-FMAs per instruction: 2 (packed) or 1
  const double lane_fma = (double)grid * 256 * iters * 32 * (packed ? 2 : 1);
  const double tflops = 2 * lane_fma / ms / 1e9;
  // cycles one warp instruction holds the SMSP at 1.965 GHz
  const double instr = (double)grid * 8 * iters * 32;   // warp instructions
  const double cyc = ms * 1e-3 * 1.965e9 * sms * 4 / instr;
  printf("{\"pattern\":\"%s\",\"ms\":%.3f,\"tflops\":%.2f,\"cycles_per_warp_instr\":%.2f}\n", name, ms, tflops, cyc);
}

int main() {
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  float *in, *out; cudaMalloc(&in, 4096 * 4); cudaMalloc(&out, sms * 8 * 256 * 4);
  cudaMemset(in, 0, 4096 * 4);
  float2 h[16];
  for (int i = 0; i < 16; ++i) h[i] = make_float2(0.5f + i * 0.01f, 0.25f);
  cudaMemcpyToSymbol(cB, h, sizeof(h));
  run<0>("ffma2_pair_bcast_same", out, in, sms, true);
  run<1>("ffma2_pair_pair_same", out, in, sms, true);
  run<2>("ffma2_pair_bcast_distinct", out, in, sms, true);
  run<3>("ffma2_pair_pair_distinct", out, in, sms, true);
  run<4>("ffma_same_m", out, in, sms, false);
  run<5>("ffma_distinct_m", out, in, sms, false);
  run<6>("ffma2_constbank_bcast_distinct", out, in, sms, true);
  run<7>("ffma_constbank_distinct", out, in, sms, false);
  run<8>("ffma2_acc_as_A_bcast_same", out, in, sms, true);
  run<9>("fmul2_acc_bcast_distinct", out, in, sms, true);
  printf("{\"status\":\"%s\"}\n", cudaGetErrorString(cudaDeviceSynchronize()));
  return 0;
}
