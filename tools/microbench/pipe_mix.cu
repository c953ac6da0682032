// FP32 pipe mix on sm_100a: cycles per loop iteration of independent-chain bodies, to tell how
// FFMA, FMUL2/FFMA2 and the ALU pipe share an SMSP.  One CTA of 256 threads per SM x MINB, 16 chains.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 pipe_mix.cu -o pipe_mix
#include <cstdio>
#include <cuda_runtime.h>
__device__ __forceinline__ float2 f2(float a, float b) { return make_float2(a, b); }
__device__ __forceinline__ float2 bc(float a) { return make_float2(a, a); }

template <int V>
__global__ void __launch_bounds__(256, 4) k(float* out, float s, int iters) {
  float a[16];
  float2 p[8];
  int q[8];
#pragma unroll
  for (int i = 0; i < 16; ++i) a[i] = threadIdx.x * 1e-3f + i;
#pragma unroll
  for (int i = 0; i < 8; ++i) { p[i] = f2(s + i, s - i); q[i] = threadIdx.x + i; }
  const float y = s * 0.999f, z = s * 0.5f;
  const float2 Y = f2(y, z);
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int r = 0; r < 4; ++r) {
      if constexpr (V == 0) {            // 16 FFMA, 1 fresh register each (y, z reused)
#pragma unroll
        for (int i = 0; i < 16; ++i) a[i] = fmaf(a[i], y, z);
      } else if constexpr (V == 1) {     // 8 FMUL2 pair x pair(shared)
#pragma unroll
        for (int i = 0; i < 8; ++i) p[i] = __fmul2_rn(p[i], Y);
      } else if constexpr (V == 2) {     // 8 FFMA + 4 FMUL2 interleaved (same flops as 16 FFMA)
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          a[2 * i] = fmaf(a[2 * i], y, z);
          p[i] = __fmul2_rn(p[i], Y);
          a[2 * i + 1] = fmaf(a[2 * i + 1], y, z);
        }
      } else if constexpr (V == 3) {     // 8 FFMA2 with a broadcast scalar (a pair x bcast + pair acc)
#pragma unroll
        for (int i = 0; i < 8; ++i) p[i] = __ffma2_rn(p[i], bc(y), Y);
      } else if constexpr (V == 4) {     // 16 FFMA + 8 IADD3 (ALU pipe)
#pragma unroll
        for (int i = 0; i < 16; ++i) a[i] = fmaf(a[i], y, z);
#pragma unroll
        for (int i = 0; i < 8; ++i) q[i] = q[i] + (q[(i + 1) & 7] ^ it);
      } else if constexpr (V == 5) {     // 16 FFMA + 8 IMAD (fmaheavy)
#pragma unroll
        for (int i = 0; i < 16; ++i) a[i] = fmaf(a[i], y, z);
#pragma unroll
        for (int i = 0; i < 8; ++i) q[i] = q[i] * 3 + it;
      } else if constexpr (V == 6) {     // 16 FFMA with 2 fresh registers (a[i], a[i+8] distinct banks?)
#pragma unroll
        for (int i = 0; i < 8; ++i) { a[i] = fmaf(a[i], a[i + 8], z); a[i + 8] = fmaf(a[i + 8], y, a[i]); }
      } else if constexpr (V == 7) {     // 16 FFMA + 2 MUFU.RSQ
#pragma unroll
        for (int i = 0; i < 16; ++i) a[i] = fmaf(a[i], y, z);
        a[0] = rsqrtf(a[0]); a[8] = rsqrtf(a[8]);
      } else if constexpr (V == 8) {     // 8 FMUL2 with a broadcast scalar operand
#pragma unroll
        for (int i = 0; i < 8; ++i) p[i] = __fmul2_rn(p[i], bc(y));
      } else if constexpr (V == 9) {     // 8 FFMA then 4 FMUL2 (grouped, asm volatile keeps the order)
#pragma unroll
        for (int i = 0; i < 8; ++i) asm volatile("fma.rn.f32 %0, %0, %1, %2;" : "+f"(a[i]) : "f"(y), "f"(z));
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          unsigned long long v, w;
          asm volatile("mov.b64 %0, {%1, %2};" : "=l"(v) : "f"(p[i].x), "f"(p[i].y));
          asm volatile("mov.b64 %0, {%1, %2};" : "=l"(w) : "f"(Y.x), "f"(Y.y));
          asm volatile("mul.rn.f32x2 %0, %0, %1;" : "+l"(v) : "l"(w));
          asm volatile("mov.b64 {%0, %1}, %2;" : "=f"(p[i].x), "=f"(p[i].y) : "l"(v));
        }
      } else if constexpr (V == 10) {    // 8 FFMA + 8 FMUL scalar interleaved
#pragma unroll
        for (int i = 0; i < 8; ++i) { a[i] = fmaf(a[i], y, z); a[i + 8] = a[i + 8] * y; }
      } else if constexpr (V == 11) {    // 8 FFMA + 4 FFMA2 interleaved
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          a[2 * i] = fmaf(a[2 * i], y, z);
          p[i] = __ffma2_rn(p[i], Y, Y);
          a[2 * i + 1] = fmaf(a[2 * i + 1], y, z);
        }
      } else if constexpr (V == 12) {    // 12 FFMA + 2 FMUL2 interleaved
#pragma unroll
        for (int i = 0; i < 2; ++i) {
#pragma unroll
          for (int j = 0; j < 6; ++j) a[6 * i + j] = fmaf(a[6 * i + j], y, z);
          p[i] = __fmul2_rn(p[i], Y);
        }
      } else if constexpr (V == 13) {    // 16 FFMA + 4 FSETP/SEL-free ALU: FMNMX
#pragma unroll
        for (int i = 0; i < 16; ++i) a[i] = fmaf(a[i], y, z);
#pragma unroll
        for (int i = 0; i < 4; ++i) a[i + 12] = fmaxf(a[i + 12], a[i]);
      }
    }
  }
  float acc = 0.f;
#pragma unroll
  for (int i = 0; i < 16; ++i) acc += a[i];
#pragma unroll
  for (int i = 0; i < 8; ++i) acc += p[i].x + p[i].y + (float)q[i];
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
}

template <int V>
void run(const char* name, float* out, int sms, int instr_per_rep) {
  const int iters = 20000, grid = sms * 4;
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0); cudaEventCreate(&e1);
  k<V><<<grid, 256>>>(out, 1.0f, 100);
  cudaEventRecord(e0);
  k<V><<<grid, 256>>>(out, 1.0f, iters);
  cudaEventRecord(e1);
  cudaEventSynchronize(e1);
  float ms; cudaEventElapsedTime(&ms, e0, e1);
  int clk; cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  // SMSP cycles per loop body (4 reps), per warp: 4 CTAs x 8 warps / 4 SMSP = 8 warps per SMSP
  const double cyc = ms * 1e-3 * 1.965e9 / ((double)iters * 8.0);
  printf("{\"variant\":\"%s\",\"ms\":%.3f,\"smsp_cycles_per_body\":%.2f,\"instr_per_body\":%d}\n", name, ms, cyc / 4.0,
         instr_per_rep);
}

int main() {
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  float* out; cudaMalloc(&out, sms * 4 * 256 * 4);
  run<0>("16_ffma_reuse", out, sms, 16);
  run<1>("8_fmul2_pairxpair", out, sms, 8);
  run<2>("8_ffma_4_fmul2", out, sms, 12);
  run<3>("8_ffma2_bcast", out, sms, 8);
  run<4>("16_ffma_8_iadd3", out, sms, 24);
  run<5>("16_ffma_8_imad", out, sms, 24);
  run<6>("16_ffma_2fresh", out, sms, 16);
  run<7>("16_ffma_2_mufu", out, sms, 18);
  run<8>("8_fmul2_bcast", out, sms, 8);
  run<9>("8_ffma_then_4_fmul2_grouped", out, sms, 12);
  run<10>("8_ffma_8_fmul_interleaved", out, sms, 16);
  run<11>("8_ffma_4_ffma2_interleaved", out, sms, 12);
  run<12>("12_ffma_2_fmul2", out, sms, 14);
  run<13>("16_ffma_4_fmnmx", out, sms, 20);
  printf("{\"status\":\"%s\"}\n", cudaGetErrorString(cudaDeviceSynchronize()));
  return 0;
}
