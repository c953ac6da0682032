// FP32 pipe microbenchmark for B200 (sm_100a): measures warp-instruction and
// lane-FMA throughput per SM per cycle for FFMA (3-reg), FFMA (imm), FFMA2.
// Used once to fix the ALU roofline denominator and the kernel design.
#include <cstdio>
#include <cuda_runtime.h>
#define CK(x) do{cudaError_t e=(x); if(e!=cudaSuccess){printf("err %s line %d\n",cudaGetErrorString(e),__LINE__);return 1;}}while(0)
__device__ __forceinline__ unsigned long long pk(float a, float b){unsigned long long r; asm("mov.b64 %0, {%1,%2};" : "=l"(r) : "f"(a), "f"(b)); return r;}
__device__ __forceinline__ float2 upk(unsigned long long v){float a,b; asm("mov.b64 {%0,%1}, %2;" : "=f"(a), "=f"(b) : "l"(v)); return make_float2(a,b);}

template<int MODE>
__global__ void __launch_bounds__(256) kern(float* out, float s, int iters, long long* cyc){
  float x = threadIdx.x * 1e-3f, y = s + threadIdx.x*1e-7f, z = s*0.5f - threadIdx.x*1e-7f;
  float a[16];
  #pragma unroll
  for (int i=0;i<16;i++) a[i] = x + i;
  unsigned long long p[8]; unsigned long long Y = pk(y, z);
  #pragma unroll
  for (int i=0;i<8;i++) p[i] = pk(x+i, x-i);
  long long t0 = clock64();
  for (int it=0; it<iters; it++){
    #pragma unroll
    for (int r=0;r<8;r++){
      if (MODE==0){
        #pragma unroll
        for (int i=0;i<16;i++) a[i] = fmaf(a[i], y, z);          // 3-reg FFMA
      } else if (MODE==1){
        #pragma unroll
        for (int i=0;i<16;i++) a[i] = fmaf(a[i], 0.999f, 0.5f);  // imm FFMA
      } else if (MODE==2){
        #pragma unroll
        for (int i=0;i<8;i++) asm volatile("fma.rn.f32x2 %0, %0, %1, %1;" : "+l"(p[i]) : "l"(Y));
      } else {
        #pragma unroll
        for (int i=0;i<8;i++) asm volatile("fma.rn.f32x2 %0, %0, %1, %0;" : "+l"(p[i]) : "l"(pk(y,y)));
      }
    }
  }
  long long t1 = clock64();
  float acc = 0;
  #pragma unroll
  for (int i=0;i<16;i++) acc += a[i];
  #pragma unroll
  for (int i=0;i<8;i++){ float2 f = upk(p[i]); acc += f.x + f.y; }
  out[blockIdx.x*blockDim.x+threadIdx.x] = acc;
  if (threadIdx.x==0) cyc[blockIdx.x] = t1 - t0;
}

int main(){
  int dev=0; cudaDeviceProp pr; CK(cudaGetDeviceProperties(&pr, dev));
  int clk=0; cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, dev);
  printf("{\"device\":\"%s\",\"sms\":%d,\"clock_khz\":%d}\n", pr.name, pr.multiProcessorCount, clk);
  int sms = pr.multiProcessorCount;
  float* out; long long* cyc; CK(cudaMalloc(&out, sizeof(float)*sms*8*256)); CK(cudaMalloc(&cyc, sizeof(long long)*sms*8));
  cudaEvent_t e0,e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  const char* names[4] = {"ffma_3reg","ffma_imm","ffma2","ffma2_bcast"};
  for (int mode=0; mode<4; mode++){
    for (int bps : {4, 8}){
      int iters = 20000;
      int grid = sms*bps;
      for (int rep=0; rep<2; rep++){
        cudaEventRecord(e0);
        if (mode==0) kern<0><<<grid,256>>>(out, 1.0001f, iters, cyc);
        if (mode==1) kern<1><<<grid,256>>>(out, 1.0001f, iters, cyc);
        if (mode==2) kern<2><<<grid,256>>>(out, 1.0001f, iters, cyc);
        if (mode==3) kern<3><<<grid,256>>>(out, 1.0001f, iters, cyc);
        cudaEventRecord(e1); CK(cudaEventSynchronize(e1));
      }
      float ms; cudaEventElapsedTime(&ms, e0, e1);
      long long hc[4096]; CK(cudaMemcpy(hc, cyc, sizeof(long long)*grid, cudaMemcpyDeviceToHost));
      double avgc=0; for(int i=0;i<grid;i++) avgc+=hc[i]; avgc/=grid;
      double lane_fma = (double)grid*256*iters*8*16;  // every mode does 16 lane-FMAs per r per thread
      double warp_instr = (mode<2) ? lane_fma/32 : lane_fma/64;
      double tflops = 2*lane_fma/(ms*1e-3)/1e12;
      // per-SM per-cycle rates using in-kernel clock64 (cycles of one CTA; all CTAs co-resident)
      double fma_per_sm_cyc = lane_fma/sms/avgc;
      printf("{\"mode\":\"%s\",\"ctas_per_sm\":%d,\"ms\":%.3f,\"tflops\":%.2f,\"lane_fma_per_sm_per_cycle\":%.1f,\"warp_instr_per_sm_per_cycle\":%.2f,\"implied_mhz\":%.0f}\n",
        names[mode], bps, ms, tflops, fma_per_sm_cyc, warp_instr/sms/avgc, avgc/(ms*1e-3)/1e6);
    }
  }
  return 0;
}
