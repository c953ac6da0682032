// Prototype host for uc_kern.cu: NMOD module instances (one constant bank each), one stream per module,
// batches of SLOTS tensors round-robin over the modules, then the resume kernel for parked lanes.
#include <cuda.h>
#include <cuda_runtime.h>
#include <vector>
#include <cstdio>
#include <cstdlib>
#include "sshopm_kernels.cuh"
using namespace sshopm;

namespace {
constexpr int PW4 = Shape<4, 3>::PW / 4;
constexpr int SLOTS = 65536 / (16 * PW4);
struct UcParams {
  float4* bank; const float4* packed; const float4* starts_n;
  float* out_lambda; float* out_x; int32_t* out_iters; uint8_t* out_conv;
  float4* park; unsigned int* park_count;
  long long t0; int nt; long long t_next; int nt_next;
  int S, maxit, refill_k, park_max; float tol;
};
struct Mod { CUmodule m; CUfunction solve, resume; CUdeviceptr bank; cudaStream_t st; cudaEvent_t ev; };
std::vector<Mod> g_mods;
cudaEvent_t g_fork;
}

extern "C" int uc_init(const char* cubin, int nmod) {
  cudaFree(0);
  for (int i = 0; i < nmod; ++i) {
    Mod md;
    if (cuModuleLoad(&md.m, cubin) != CUDA_SUCCESS) return 1;
    if (cuModuleGetFunction(&md.solve, md.m, "uc_solve43") != CUDA_SUCCESS) return 2;
    if (cuModuleGetFunction(&md.resume, md.m, "uc_resume43") != CUDA_SUCCESS) return 3;
    size_t bytes = 0;
    if (cuModuleGetGlobal(&md.bank, &bytes, md.m, "uc_bank") != CUDA_SUCCESS) return 4;
    if (bytes != (size_t)SLOTS * PW4 * 16) return 5;
    md.st = nullptr; md.ev = nullptr;
    if (i < 64) {
      cudaStreamCreateWithFlags(&md.st, cudaStreamNonBlocking);
      cudaEventCreateWithFlags(&md.ev, cudaEventDisableTiming);
    }
    g_mods.push_back(md);
  }
  cudaEventCreateWithFlags(&g_fork, cudaEventDisableTiming);
  return 0;
}

extern "C" size_t uc_ws_bytes(long long N, int S) {
  return 256 + (size_t)S * 16 + (size_t)N * PW4 * 16 + (size_t)N * 8 * 32;
}

// pack (library pack kernel) + batches + resume, all enqueued on `st`
extern "C" int uc_solve(long long N, const float* entries, int S, const float* starts, float tol, int maxit,
                        int refill_k, int park_max, float* olam, float* ox, int32_t* oit, uint8_t* ocv,
                        void* ws, int nmod_use, cudaStream_t st) {
  char* b = (char*)ws;
  unsigned int* park_count = (unsigned int*)b;
  float* starts_n = (float*)(b + 256);
  float4* packed = (float4*)(b + 256 + (size_t)S * 16);
  float4* park = packed + (size_t)N * PW4;
  const int phases = getenv("UC_PHASES") ? atoi(getenv("UC_PHASES")) : 3;
  if (phases == 2) {   // resume only (park list of the previous call)
    UcParams p{};
    p.packed = (float4*)(b + 256 + (size_t)S * 16); p.out_lambda = olam; p.out_x = ox; p.out_iters = oit; p.out_conv = ocv;
    p.park = (float4*)(b + 256 + (size_t)S * 16) + (size_t)N * PW4; p.park_count = park_count; p.S = S; p.maxit = maxit; p.tol = tol;
    void* args[] = {&p};
    return cuLaunchKernel(g_mods[0].resume, 148 * 4, 1, 1, 256, 1, 1, 0, st, args, nullptr) != CUDA_SUCCESS ? 11 : 0;
  }
  if (phases == 4) {   // timing mode: one launch, all tensors, rows reused from module 0's bank
    cudaMemsetAsync(park_count, 0, 4, st);
    UcParams p{};
    p.bank = (float4*)g_mods[0].bank; p.packed = (float4*)(b + 256 + (size_t)S * 16); p.starts_n = (const float4*)(b + 256);
    p.out_lambda = olam; p.out_x = ox; p.out_iters = oit; p.out_conv = ocv;
    p.park = (float4*)(b + 256 + (size_t)S * 16) + (size_t)N * PW4; p.park_count = park_count; p.t0 = 0; p.nt = (int)N; p.t_next = 0; p.nt_next = 0;
    p.S = S; p.maxit = maxit; p.refill_k = refill_k; p.park_max = -park_max - 1; p.tol = tol;
    void* args[] = {&p};
    return cuLaunchKernel(g_mods[0].solve, (unsigned)((N + 3) / 4), 1, 1, 128, 1, 1, 0, st, args, nullptr) != CUDA_SUCCESS ? 13 : 0;
  }
  cudaMemsetAsync(park_count, 0, 4, st);
  sshopm_pack_kernel<4, 3><<<148 * 8, 256, 0, st>>>(N, entries, packed, nullptr, S, starts, starts_n, 0, nullptr, nullptr);
  const int nmod = nmod_use < (int)g_mods.size() ? nmod_use : (int)g_mods.size();
  const long long nb = (N + SLOTS - 1) / SLOTS;
  cudaEventRecord(g_fork, st);
  for (int j = 0; j < nmod; ++j) {
    cudaStreamWaitEvent(g_mods[j].st, g_fork, 0);
    if (j < nb) {
      const long long t0 = (long long)j * SLOTS;
      const long long nt = (N - t0) < SLOTS ? (N - t0) : SLOTS;
      cudaMemcpyAsync((void*)g_mods[j].bank, packed + t0 * PW4, nt * PW4 * 16, cudaMemcpyDeviceToDevice, g_mods[j].st);
    }
  }
  for (long long bi = 0; bi < nb; ++bi) {
    Mod& md = g_mods[bi % nmod];
    UcParams p;
    p.bank = (float4*)md.bank; p.packed = packed; p.starts_n = (const float4*)starts_n;
    p.out_lambda = olam; p.out_x = ox; p.out_iters = oit; p.out_conv = ocv; p.park = park; p.park_count = park_count;
    p.t0 = bi * SLOTS; p.nt = (int)((N - p.t0) < SLOTS ? (N - p.t0) : SLOTS);
    p.t_next = (bi + nmod) * SLOTS;
    p.nt_next = p.t_next < N ? (int)((N - p.t_next) < SLOTS ? (N - p.t_next) : SLOTS) : 0;
    p.S = S; p.maxit = maxit; p.refill_k = refill_k; p.park_max = park_max; p.tol = tol;
    void* args[] = {&p};
    if (cuLaunchKernel(md.solve, (p.nt + 3) / 4, 1, 1, 128, 1, 1, 0, md.st, args, nullptr) != CUDA_SUCCESS) return 10;
  }
  for (int j = 0; j < nmod; ++j) {
    cudaEventRecord(g_mods[j].ev, g_mods[j].st);
    cudaStreamWaitEvent(st, g_mods[j].ev, 0);
  }
  if (!(phases & 2)) return 0;
  UcParams p{};
  p.packed = packed; p.out_lambda = olam; p.out_x = ox; p.out_iters = oit; p.out_conv = ocv;
  p.park = park; p.park_count = park_count; p.S = S; p.maxit = maxit; p.tol = tol;
  void* args[] = {&p};
  if (cuLaunchKernel(g_mods[0].resume, 148 * 4, 1, 1, 256, 1, 1, 0, st, args, nullptr) != CUDA_SUCCESS) return 11;
  return cudaGetLastError() == cudaSuccess ? 0 : 12;
}

// wide graph: one module per batch (banks filled by one kernel through a pointer table), every solve
// launch independent of the others, then the resume kernel
__global__ void fill_banks(const float4* __restrict__ packed, float4* const* __restrict__ banks, long long N) {
  const long long nw = N * PW4;
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < nw; i += (long long)gridDim.x * blockDim.x) {
    const long long t = i / PW4;
    banks[t / SLOTS][(t % SLOTS) * PW4 + (i % PW4)] = packed[i];
  }
}
static cudaGraphExec_t g_wexec = nullptr;
extern "C" int uc_wide(long long N, const float* entries, int S, const float* starts, float tol, int maxit,
                       int refill_k, int park_max, float* olam, float* ox, int32_t* oit, uint8_t* ocv, void* ws,
                       cudaStream_t st) {
  char* b = (char*)ws;
  unsigned int* park_count = (unsigned int*)b;
  float* starts_n = (float*)(b + 256);
  float4* packed = (float4*)(b + 256 + (size_t)S * 16);
  float4* park = packed + (size_t)N * PW4;
  const long long nb = (N + SLOTS - 1) / SLOTS;
  if ((long long)g_mods.size() < nb) return 40;
  static float4** d_banks = nullptr;
  if (!d_banks) {
    std::vector<float4*> hb(nb);
    for (long long i = 0; i < nb; ++i) hb[i] = (float4*)g_mods[i].bank;
    cudaMalloc(&d_banks, nb * sizeof(float4*));
    cudaMemcpy(d_banks, hb.data(), nb * sizeof(float4*), cudaMemcpyHostToDevice);
  }
  cudaStream_t cs;
  cudaStreamCreateWithFlags(&cs, cudaStreamNonBlocking);
  cudaGraph_t g;
  cudaStreamBeginCapture(cs, cudaStreamCaptureModeThreadLocal);
  cudaMemsetAsync(park_count, 0, 4, cs);
  sshopm_pack_kernel<4, 3><<<148 * 8, 256, 0, cs>>>(N, entries, packed, nullptr, S, starts, starts_n, 0, nullptr, nullptr);
  fill_banks<<<148 * 8, 256, 0, cs>>>(packed, d_banks, N);
  cudaStreamEndCapture(cs, &g);
  // add the solve nodes after the last captured node, then the resume node after all of them
  size_t nn = 0;
  cudaGraphGetNodes(g, nullptr, &nn);
  std::vector<cudaGraphNode_t> nodes(nn);
  cudaGraphGetNodes(g, nodes.data(), &nn);
  cudaGraphNode_t last = nodes[nn - 1];
  {   // find the sink (the node with no dependents)
    for (auto n : nodes) { size_t d = 0; cudaGraphNodeGetDependentNodes(n, nullptr, &d); if (d == 0) last = n; }
  }
  std::vector<UcParams> ps(nb);
  std::vector<CUgraphNode> solves(nb);
  for (long long bi = 0; bi < nb; ++bi) {
    UcParams& p = ps[bi];
    p = UcParams{};
    p.bank = (float4*)g_mods[bi].bank; p.packed = packed; p.starts_n = (const float4*)starts_n;
    p.out_lambda = olam; p.out_x = ox; p.out_iters = oit; p.out_conv = ocv; p.park = park; p.park_count = park_count;
    p.t0 = bi * SLOTS; p.nt = (int)((N - p.t0) < SLOTS ? (N - p.t0) : SLOTS);
    p.t_next = 0; p.nt_next = 0;
    p.S = S; p.maxit = maxit; p.refill_k = refill_k; p.park_max = park_max; p.tol = tol;
    void* args[] = {&p};
    CUDA_KERNEL_NODE_PARAMS kp{};
    kp.func = g_mods[bi].solve; kp.gridDimX = (p.nt + 3) / 4; kp.gridDimY = kp.gridDimZ = 1;
    kp.blockDimX = 128; kp.blockDimY = kp.blockDimZ = 1; kp.sharedMemBytes = 0; kp.kernelParams = args;
    CUgraphNode dep = (CUgraphNode)last;
    if (cuGraphAddKernelNode(&solves[bi], (CUgraph)g, &dep, 1, &kp) != CUDA_SUCCESS) return 41;
  }
  UcParams p{};
  p.packed = packed; p.out_lambda = olam; p.out_x = ox; p.out_iters = oit; p.out_conv = ocv;
  p.park = park; p.park_count = park_count; p.S = S; p.maxit = maxit; p.tol = tol;
  void* args[] = {&p};
  CUDA_KERNEL_NODE_PARAMS kp{};
  kp.func = g_mods[0].resume; kp.gridDimX = 148 * 4; kp.gridDimY = kp.gridDimZ = 1;
  kp.blockDimX = 256; kp.blockDimY = kp.blockDimZ = 1; kp.kernelParams = args;
  CUgraphNode rn;
  if (cuGraphAddKernelNode(&rn, (CUgraph)g, solves.data(), solves.size(), &kp) != CUDA_SUCCESS) return 42;
  if (g_wexec) cudaGraphExecDestroy(g_wexec);
  if (cudaGraphInstantiate(&g_wexec, g, 0) != cudaSuccess) return 43;
  cudaGraphDestroy(g);
  cudaStreamDestroy(cs);
  return 0;
}
extern "C" int uc_wide_replay(cudaStream_t st) { return cudaGraphLaunch(g_wexec, st) == cudaSuccess ? 0 : 44; }

// capture uc_solve into a graph once; replay
static cudaGraphExec_t g_exec = nullptr;
extern "C" int uc_capture(long long N, const float* entries, int S, const float* starts, float tol, int maxit,
                          int refill_k, int park_max, float* olam, float* ox, int32_t* oit, uint8_t* ocv,
                          void* ws, int nmod_use, cudaStream_t st) {
  cudaGraph_t g;
  if (cudaStreamBeginCapture(st, cudaStreamCaptureModeThreadLocal) != cudaSuccess) return 20;
  int rc = uc_solve(N, entries, S, starts, tol, maxit, refill_k, park_max, olam, ox, oit, ocv, ws, nmod_use, st);
  if (cudaStreamEndCapture(st, &g) != cudaSuccess) return 21;
  if (rc) return rc;
  if (g_exec) cudaGraphExecDestroy(g_exec);
  if (cudaGraphInstantiate(&g_exec, g, 0) != cudaSuccess) return 22;
  cudaGraphDestroy(g);
  return 0;
}
extern "C" int uc_replay(cudaStream_t st) { return cudaGraphLaunch(g_exec, st) == cudaSuccess ? 0 : 30; }
