// Prototype: (4,3) SS-HOPM solve with the tensor's coefficient words in the constant bank (uniform
// operands), one warp per tensor, stragglers parked for a resume kernel.  Loaded NMOD times by uc_host.cu
// (each module instance has its own 64 KB bank).
#include "sshopm_kernels.cuh"
using namespace sshopm;

constexpr int PW4 = Shape<4, 3>::PW / 4;          // 8 float4 per tensor row
constexpr int SLOTS = 65536 / (16 * PW4);         // 512 rows per bank
__constant__ float4 uc_bank[SLOTS * PW4];

struct UcParams {
  float4* bank;              // this module's bank (global address) — the next batch's rows are written here
  const float4* packed;      // [N][PW4]
  const float4* starts_n;    // [S][1]
  float* out_lambda; float* out_x; int32_t* out_iters; uint8_t* out_conv;
  float4* park;              // [cap][2]: (x0, x1, x2, x1) | (lamp, k, item, -)
  unsigned int* park_count;
  long long t0;              // first tensor of this launch
  int nt;                    // tensors in this launch
  long long t_next;          // first tensor of the next launch on this module
  int nt_next;
  int S, maxit, refill_k, park_max;
  float tol;
};

extern "C" __global__ void __launch_bounds__(128) uc_solve43(const UcParams p) {
  const int lane = threadIdx.x & 31;
  const uint32_t FULL = 0xffffffffu;
  const int wib = __reduce_or_sync(FULL, threadIdx.x >> 5);
  int slot = blockIdx.x * 4 + wib;
  if (slot >= p.nt) return;
  long long tvv = p.t0 + slot;
  if (p.park_max < 0) { slot &= SLOTS - 1; }   // timing mode: one launch over all tensors, rows reused
  const int park_max = p.park_max < 0 ? -p.park_max - 1 : p.park_max;
  Coefs<4, 3> cf;
#pragma unroll
  for (int i = 0; i < PW4; ++i) cf.w[i] = uc_bank[slot * PW4 + i];
  const uint32_t ltmask = lanemask_lt();
  const long long tv = tvv;
  const uint32_t S = (uint32_t)p.S;
  const float tol = p.tol;
  const int maxit = p.maxit;
  float2 xs[2] = {f2(0.f, 0.f), f2(0.f, 0.f)};
  float lam = 0.f, lamp = 0.f;
  int k = 0x7fffffff;
  bool has = false, stop = true, conv = false;
  uint32_t s = 0;           // this lane's start
  uint32_t qi = 0;          // next start of the tensor (warp-uniform)
  uint32_t k_eff = (uint32_t)p.refill_k;
  float* const olam = p.out_lambda + tv * S;
  for (;;) {
    const uint32_t smask = __ballot_sync(FULL, stop);
    const uint32_t cnt = __popc(smask);
    if (qi >= S) {                                   // starts exhausted: finish or park
      const uint32_t nact = 32u - cnt;
      if (nact <= (uint32_t)park_max) {
        const bool wr = stop && has;
        const size_t item = (size_t)tv * S + s;
        if (wr) {
          olam[s] = lam;
          float* ox = p.out_x + item * 3;
          ox[0] = xs[0].x; ox[1] = xs[0].y; ox[2] = xs[1].x;
          p.out_iters[item] = k;
          p.out_conv[item] = conv ? 1 : 0;
        }
        if (nact) {
          const bool pk = !stop;
          const uint32_t pm = __ballot_sync(FULL, pk);
          unsigned int base = 0;
          if (lane == 0) base = atomicAdd(p.park_count, (unsigned)__popc(pm));
          base = __shfl_sync(FULL, base, 0);
          if (pk) {
            const unsigned r = base + __popc(pm & ltmask);
            p.park[2 * (size_t)r] = make_float4(xs[0].x, xs[0].y, xs[1].x, xs[1].y);
            p.park[2 * (size_t)r + 1] = make_float4(lamp, __int_as_float(k), __int_as_float((int)(uint32_t)item),
                                                    __int_as_float((int)(uint32_t)(item >> 32)));
          }
        }
        break;
      }
    } else if (cnt >= k_eff) {
      const bool wr = stop && has;
      if (wr) {
        const size_t item = (size_t)tv * S + s;
        olam[s] = lam;
        float* ox = p.out_x + item * 3;
        ox[0] = xs[0].x; ox[1] = xs[0].y; ox[2] = xs[1].x;
        p.out_iters[item] = k;
        p.out_conv[item] = conv ? 1 : 0;
      }
      const uint32_t ns = qi + __popc(smask & ltmask);
      const bool ok = stop && ns < S;
      if (ok) {
        s = ns;
        const float4 q4 = ldg4(p.starts_n + ns);
        xs[0] = f2(q4.x, q4.y);
        xs[1] = f2(q4.z, q4.w);
      }
      k = ok ? 0 : (stop ? 0x7fffffff : k);
      lamp = ok ? __int_as_float(0x7fffffff) : lamp;
      has = stop ? ok : has;
      qi += cnt;
    }
#pragma unroll
    for (int rep = 0; rep < 4; ++rep)
      sshopm_step<4, 3, 0, true>(cf, xs, lam, lamp, k, conv, stop, has, 0.f, 0.f, 1.f, tol, maxit);
    __syncwarp();
  }
  // rows of the next batch for this slot (read by the next launch on this module)
  if (p.park_max >= 0 && slot < p.nt_next && lane < PW4) p.bank[slot * PW4 + lane] = ldg4(p.packed + (p.t_next + slot) * PW4 + lane);
}

// Parked lanes: thread per record, per-lane coefficients from the packed rows; the same step.
extern "C" __global__ void __launch_bounds__(256) uc_resume43(const UcParams p) {
  const unsigned int n = *p.park_count;
  for (unsigned int r = blockIdx.x * blockDim.x + threadIdx.x; r < n; r += gridDim.x * blockDim.x) {
    const float4 a = p.park[2 * (size_t)r], b = p.park[2 * (size_t)r + 1];
    float2 xs[2] = {f2(a.x, a.y), f2(a.z, a.w)};
    float lamp = b.x, lam = 0.f;
    int k = __float_as_int(b.y);
    const size_t item = (size_t)(uint32_t)__float_as_int(b.z) | ((size_t)(uint32_t)__float_as_int(b.w) << 32);
    const size_t tv = item / (uint32_t)p.S;
    Coefs<4, 3> cf;
    cf.load(p.packed + tv * PW4);
    bool stop = false, conv = false;
    while (!stop) sshopm_step<4, 3, 0, true>(cf, xs, lam, lamp, k, conv, stop, true, 0.f, 0.f, 1.f, p.tol, p.maxit);
    p.out_lambda[item] = lam;
    float* ox = p.out_x + item * 3;
    ox[0] = xs[0].x; ox[1] = xs[0].y; ox[2] = xs[1].x;
    p.out_iters[item] = k;
    p.out_conv[item] = conv ? 1 : 0;
  }
}
