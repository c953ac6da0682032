// sshopm_dedup.cuh — per-tensor eigenpair dedup (reading R16).
//
// The paper runs SS-HOPM from many starts "to find multiple eigenpairs"
// and keeps the local maxima as fibre directions
// but states no merge rule.  Reading R16 is a greedy pass over converged starts
// in start order: a start joins the first existing cluster whose
// representative matches (lambda within lam_tol*max(1,|lam_r|), angle within
// ang_tol, sign-free for even m), else it founds a new cluster.
//
// Parallel form (one warp per tensor, results staged in shared memory):
// round r picks rep_r = the first still-unassigned converged start, then
// every lane tests its unassigned starts against rep_r in parallel.  This is
// exactly the sequential greedy: rep_r matches none of rep_0..rep_{r-1} (else
// it would be assigned), reps increase in start order, and a start assigned
// in round r matches rep_r and none of the earlier reps — the first match in
// creation order.  Rounds = number of clusters (typically 1-5).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>
#ifdef SSHOPM_BOUNDS_CHECK
#include <cassert>
#endif

namespace sshopm {

struct DedupParams {
  const float* lambda;     // [N][S]
  const float* x;          // [N][S][n]
  const uint8_t* conv;     // [N][S]
  int32_t* out_count;      // [N]
  float* out_lambda;       // [N][kmax]
  float* out_x;            // [N][kmax][n]
  int32_t* out_mult;       // [N][kmax]
  int32_t* out_rep;        // [N][kmax] or null
  long long n_tensors;
  int S, kmax;
  float lam_tol, cos_tol;  // cos(ang_tol) (may be negative)
  const float4* rec;       // records path (sshopm_solve_rec_kernel): [N][S][rec4(n)] float4 per start,
                           // (x_0 .. x_{n-1}, lambda if converged else NaN, 0 pad); null = the raw arrays above
};
// float4s per start record of the records path: lambda + n components, padded to a multiple of 4 words
__host__ __device__ constexpr int dd_rec4(int n) { return (n + 1 + 3) / 4; }

// shared-memory words per warp for S starts, dimension n
__host__ __device__ constexpr int dedup_smem_words(int S, int n) { return S * (n + 2) + 3 * S; }

// R16 membership test of a start (ls, xs, squared norm n2s) against the round's
// representative (rl, rx, squared norm rn), ltol = lam_tol * max(1, |rl|),
// lim2 = cos_tol^2 * rn.  angle(xs, rx) <= ang_tol is cos >= cos_tol; for
// ang_tol <= pi/2 (cos_tol >= 0) it is evaluated squared, dot^2 >= lim2 * n2s,
// with the sign of dot chosen by the R15 rules (no square root); for larger
// ang_tol as |dot| >= cos_tol * sqrt(n2s * rn).  Every dedup path (standalone,
// list, fused) calls this one function, so they agree bit for bit.
template <int N, bool EVEN>
__device__ __forceinline__ bool dd_same(float ls, const float (&xs)[N], float n2s, float rl, const float (&rx)[N],
                                        float rn, float lim2, float ltol, float cos_tol) {
  float dot = 0.f;
#pragma unroll
  for (int j = 0; j < N; ++j) dot = fmaf(xs[j], rx[j], dot);
  if (cos_tol >= 0.f) {   // branch-free (bitwise & / |): predicate logic, no per-start branches
    const bool ang = dot * dot >= lim2 * n2s;
    if (EVEN) return ang & (fabsf(ls - rl) <= ltol);
    return ang & (((dot >= 0.f) & (fabsf(ls - rl) <= ltol)) | ((dot <= 0.f) & (fabsf(-ls - rl) <= ltol)));
  }
  const float lim = cos_tol * sqrtf(n2s * rn);
  if (EVEN) return fabsf(ls - rl) <= ltol && fabsf(dot) >= lim;
  return (fabsf(ls - rl) <= ltol && dot >= lim) || (fabsf(-ls - rl) <= ltol && -dot >= lim);
}

template <int N>
__device__ __forceinline__ float dd_norm2(const float (&x)[N]) {
  float n2 = 0.f;
#pragma unroll
  for (int j = 0; j < N; ++j) n2 = fmaf(x[j], x[j], n2);
  return n2;
}

// One warp clusters tensor v (R16), any S.  Staging arrays (per warp, shared
// memory): s_lam[S], s_x[S*N], s_cid[S], c_lam[S], c_rep[S], c_mult[S].  Inputs
// are read with ld.global.cg (L2), so the routine is also safe right after
// other lanes of the same warp wrote them (fused solve -> dedup; caller fences).
template <int N, bool EVEN, bool REC = false>
__device__ __forceinline__ void warp_dedup_tensor(const DedupParams& p, long long v, int lane, float* s_lam,
                                                  float* s_x, int* s_cid, float* c_lam, int* c_rep, int* c_mult) {
  const int S = p.S;
  const long long b = v * S;
  if constexpr (REC) {     // records: converged <=> lambda is not NaN (a converged lambda is finite)
    constexpr int R4 = dd_rec4(N);
    for (int s = lane; s < S; s += 32) {
      const float4* r = p.rec + (b + s) * R4;
      float w[4 * R4];
#pragma unroll
      for (int i = 0; i < R4; ++i) {
        const float4 q = __ldcg(r + i);
        w[4 * i] = q.x; w[4 * i + 1] = q.y; w[4 * i + 2] = q.z; w[4 * i + 3] = q.w;
      }
      s_lam[s] = w[N];
      s_cid[s] = (w[N] == w[N]) ? -1 : -2;
#pragma unroll
      for (int j = 0; j < N; ++j) s_x[s * N + j] = w[j];
    }
  } else {
    for (int s = lane; s < S; s += 32) {
      s_lam[s] = __ldcg(p.lambda + b + s);
      s_cid[s] = __ldcg(p.conv + b + s) ? -1 : -2;
    }
    for (int t = lane; t < S * N; t += 32) s_x[t] = __ldcg(p.x + b * N + t);
  }
  __syncwarp();

  const float ct2 = p.cos_tol * p.cos_tol;
  int ncl = 0;
  for (;;) {
    int first = 0x7fffffff;
    for (int s = lane; s < S; s += 32)
      if (s_cid[s] == -1) { first = s; break; }
    first = __reduce_min_sync(0xffffffffu, first);
    if (first == 0x7fffffff) break;
    const float rl = s_lam[first];
    float rx[N];
#pragma unroll
    for (int j = 0; j < N; ++j) rx[j] = s_x[first * N + j];
    const float rn = dd_norm2<N>(rx);
    const float ltol = p.lam_tol * fmaxf(1.0f, fabsf(rl));
    const float lim2 = ct2 * rn;
    int cnt = 0;
    for (int s = lane; s < S; s += 32) {
      if (s_cid[s] != -1) continue;
      float xs[N];
#pragma unroll
      for (int j = 0; j < N; ++j) xs[j] = s_x[s * N + j];
      const bool same = (s == first) || dd_same<N, EVEN>(s_lam[s], xs, dd_norm2<N>(xs), rl, rx, rn, lim2, ltol, p.cos_tol);
      if (same) { s_cid[s] = ncl; ++cnt; }
    }
    cnt = __reduce_add_sync(0xffffffffu, cnt);
    if (lane == 0) { c_lam[ncl] = rl; c_rep[ncl] = first; c_mult[ncl] = cnt; }
    ++ncl;
    __syncwarp();
  }

  if (lane == 0) p.out_count[v] = ncl;
  const long long ob = v * p.kmax;
  for (int c = lane; c < ncl; c += 32) {
    const float lc = c_lam[c];
    int rank = 0;
    for (int d = 0; d < ncl; ++d) {
      const float ld = c_lam[d];
      rank += (ld > lc) || (ld == lc && d < c);   // reps increase with cluster index
    }
    if (rank < p.kmax) {
      const int r = c_rep[c];
      p.out_lambda[ob + rank] = lc;
#pragma unroll
      for (int j = 0; j < N; ++j) p.out_x[(ob + rank) * N + j] = s_x[r * N + j];
      p.out_mult[ob + rank] = c_mult[c];
      if (p.out_rep) p.out_rep[ob + rank] = r;
    }
  }
  for (int slot = ncl + lane; slot < p.kmax; slot += 32) {
    p.out_lambda[ob + slot] = 0.f;
#pragma unroll
    for (int j = 0; j < N; ++j) p.out_x[(ob + slot) * N + j] = 0.f;
    p.out_mult[ob + slot] = 0;
    if (p.out_rep) p.out_rep[ob + slot] = -1;
  }
  __syncwarp();
}

template <int N, bool EVEN, bool REC = false>
__global__ void __launch_bounds__(256) sshopm_dedup_kernel(const DedupParams p) {
  extern __shared__ float smem[];
  const int lane = threadIdx.x & 31;
  const int wib = threadIdx.x >> 5;
  const int S = p.S;
  float* s_lam = smem + (size_t)wib * dedup_smem_words(S, N);
  float* s_x = s_lam + S;
  int* s_cid = reinterpret_cast<int*>(s_x + (size_t)S * N);
  float* c_lam = reinterpret_cast<float*>(s_cid + S);
  int* c_rep = reinterpret_cast<int*>(c_lam + S);
  int* c_mult = c_rep + S;
  const long long warps = (long long)gridDim.x * (blockDim.x >> 5);
  for (long long v = (long long)blockIdx.x * (blockDim.x >> 5) + wib; v < p.n_tensors; v += warps)
    warp_dedup_tensor<N, EVEN, REC>(p, v, lane, s_lam, s_x, s_cid, c_lam, c_rep, c_mult);
}

// Dedup of the tensors of listed chunks (fused solve: chunks whose completion
// could not be tracked).  list[i] = chunk index; chunk c = tensors
// [c*chunk_tensors, min(N, (c+1)*chunk_tensors)).  *count read on the device.
template <int N, bool EVEN>
__global__ void __launch_bounds__(256) sshopm_dedup_list_kernel(const DedupParams p, const unsigned int* count,
                                                                const unsigned int* list, int chunk_tensors) {
  extern __shared__ float smem[];
  const int lane = threadIdx.x & 31;
  const int wib = threadIdx.x >> 5;
  const int S = p.S;
  float* s_lam = smem + (size_t)wib * dedup_smem_words(S, N);
  float* s_x = s_lam + S;
  int* s_cid = reinterpret_cast<int*>(s_x + (size_t)S * N);
  float* c_lam = reinterpret_cast<float*>(s_cid + S);
  int* c_rep = reinterpret_cast<int*>(c_lam + S);
  int* c_mult = c_rep + S;
  const long long total = (long long)(*count) * chunk_tensors;
  const long long warps = (long long)gridDim.x * (blockDim.x >> 5);
  for (long long i = (long long)blockIdx.x * (blockDim.x >> 5) + wib; i < total; i += warps) {
    const long long v = (long long)list[i / chunk_tensors] * chunk_tensors + i % chunk_tensors;
    if (v < p.n_tensors) warp_dedup_tensor<N, EVEN>(p, v, lane, s_lam, s_x, s_cid, c_lam, c_rep, c_mult);
  }
}

// ----------------------------------------------------------------------------
// S = 128: lane l owns starts 4l..4l+3 in registers (float4 loads: lambda 1, x N,
// converged one u32); the unassigned converged starts of a lane are a 4-bit
// mask; cluster c's record lives in lane c's registers (up to 32 clusters).
// Same rounds as warp_dedup_tensor.  STAGE: the round representative is read
// back from a per-warp shared-memory copy of the tensor's results (4 LDS)
// instead of selected and shuffled out of the owning lane's registers.
template <int N>
struct DedupRegs {
  float4 lam;
  float4 x[N];      // 4 starts x N components, start-major
  uint32_t conv;    // 4 bytes
};

template <int N>
__device__ __forceinline__ void dedup_load(DedupRegs<N>& r, const DedupParams& p, long long v, int lane, bool stream) {
  const long long b = v * 128;
  const float4* pl = reinterpret_cast<const float4*>(p.lambda + b) + lane;
  const float4* px = reinterpret_cast<const float4*>(p.x + b * N) + lane * N;
  const unsigned int* pc = reinterpret_cast<const unsigned int*>(p.conv + b) + lane;
  if (stream) {                    // standalone kernel: read once, evict first
    r.lam = __ldcs(pl);
#pragma unroll
    for (int i = 0; i < N; ++i) r.x[i] = __ldcs(px + i);
    r.conv = __ldcs(pc);
  } else {                         // fused: just written by this warp's lanes, read through L2
    r.lam = __ldcg(pl);
#pragma unroll
    for (int i = 0; i < N; ++i) r.x[i] = __ldcg(px + i);
    r.conv = __ldcg(pc);
  }
}

// records path: lane l holds starts l, l + 32, l + 64, l + 96 (coalesced record loads; start index of
// register slot c = l + 32 c, the LANEMAJ form of dedup128_regs), one (x, lambda | NaN) record each
template <int N>
__device__ __forceinline__ void dedup_load_rec(DedupRegs<N>& r, const DedupParams& p, long long v, int lane) {
  constexpr int R4 = dd_rec4(N);
  const float4* pr = p.rec + (v * 128) * R4;
#ifdef SSHOPM_BOUNDS_CHECK
  assert(v < p.n_tensors && p.S == 128);
#endif
  float w[4][4 * R4];
#pragma unroll
  for (int c = 0; c < 4; ++c)
#pragma unroll
    for (int i = 0; i < R4; ++i) {
      const float4 q = __ldcs(pr + (size_t)(lane + 32 * c) * R4 + i);
      w[c][4 * i] = q.x; w[c][4 * i + 1] = q.y; w[c][4 * i + 2] = q.z; w[c][4 * i + 3] = q.w;
    }
  r.lam = make_float4(w[0][N], w[1][N], w[2][N], w[3][N]);
  float xf[4 * N];
#pragma unroll
  for (int c = 0; c < 4; ++c)
#pragma unroll
    for (int j = 0; j < N; ++j) xf[c * N + j] = w[c][j];
#pragma unroll
  for (int i = 0; i < N; ++i) r.x[i] = make_float4(xf[4 * i], xf[4 * i + 1], xf[4 * i + 2], xf[4 * i + 3]);
  r.conv = (w[0][N] == w[0][N] ? 0x1u : 0u) | (w[1][N] == w[1][N] ? 0x100u : 0u) | (w[2][N] == w[2][N] ? 0x10000u : 0u) |
           (w[3][N] == w[3][N] ? 0x1000000u : 0u);
}

// Returns false (nothing written) if the tensor has more than 32 clusters.
// stage: per-warp 128 * (N + 1) floats of shared memory when STAGE.
// LANEMAJ: register slot c of lane l holds start l + 32 c (records path) instead of 4 l + c; the shared-
// memory stage then keeps x component-major (stage[128 + j * 128 + start]).
template <int N, bool EVEN, bool STAGE, bool LANEMAJ = false>
__device__ __forceinline__ bool dedup128_regs(const DedupParams& p, long long v, int lane, const DedupRegs<N>& r,
                                              float* stage) {
  constexpr int SPL = 4;
  const uint32_t FULL = 0xffffffffu;
  const float lam[SPL] = {r.lam.x, r.lam.y, r.lam.z, r.lam.w};
  float xs[SPL][N];
#pragma unroll
  for (int c = 0; c < SPL; ++c)
#pragma unroll
    for (int j = 0; j < N; ++j) {
      const int w = c * N + j;
      const float4 q = r.x[w / 4];
      xs[c][j] = (w % 4 == 0) ? q.x : (w % 4 == 1) ? q.y : (w % 4 == 2) ? q.z : q.w;
    }
  float n2[SPL];
#pragma unroll
  for (int c = 0; c < SPL; ++c) n2[c] = dd_norm2<N>(xs[c]);
#ifndef SSHOPM_DD_MASK
#define SSHOPM_DD_MASK 1   // byte-mask unpack of the converged flags (C2: 0.422 -> 0.420 ms)
#endif
#if SSHOPM_DD_MASK
  // unassigned converged starts (bit c = start 4*lane + c): byte c nonzero -> bit c
  const uint32_t nz = __vcmpne4(r.conv, 0u) & 0x08040201u;
  uint32_t un = (nz | (nz >> 8) | (nz >> 16) | (nz >> 24)) & 0xfu;
#else
  uint32_t un = 0;                                   // unassigned converged starts (bit c = start 4*lane + c)
#pragma unroll
  for (int c = 0; c < SPL; ++c) un |= ((r.conv >> (8 * c)) & 0xffu) ? (1u << c) : 0u;
#endif
  if constexpr (STAGE && LANEMAJ) {
#pragma unroll
    for (int c = 0; c < SPL; ++c) {
      stage[32 * c + lane] = lam[c];
#pragma unroll
      for (int j = 0; j < N; ++j) stage[128 + 128 * j + 32 * c + lane] = xs[c][j];
    }
    __syncwarp();
  } else if constexpr (STAGE) {
    reinterpret_cast<float4*>(stage)[lane] = r.lam;
#pragma unroll
    for (int i = 0; i < N; ++i) reinterpret_cast<float4*>(stage + 128)[lane * N + i] = r.x[i];
    __syncwarp();
  }
  const float ct2 = p.cos_tol * p.cos_tol;
  float my_lam = 0.f, my_x[N];
  int my_rep = -1, my_mult = 0;
#pragma unroll
  for (int j = 0; j < N; ++j) my_x[j] = 0.f;
  int ncl = 0;
#pragma unroll 1
  for (;;) {
    const int fl = __ffs(un) - 1;                    // lowest unassigned local start (-1: none)
    const int first = __reduce_min_sync(FULL, fl >= 0 ? (LANEMAJ ? lane + 32 * fl : SPL * lane + fl) : 0x7fffffff);
    if (first == 0x7fffffff) break;
    if (ncl == 32) return false;                     // too many clusters for the register form
    float rl, rx[N];
    if constexpr (STAGE) {
      rl = stage[first];
#pragma unroll
      for (int j = 0; j < N; ++j) rx[j] = LANEMAJ ? stage[128 + 128 * j + first] : stage[128 + first * N + j];
    } else {
      const int src = LANEMAJ ? (first & 31) : first / SPL, fc = LANEMAJ ? (first >> 5) : first % SPL;
      rl = __shfl_sync(FULL, (fc == 0) ? lam[0] : (fc == 1) ? lam[1] : (fc == 2) ? lam[2] : lam[3], src);
#pragma unroll
      for (int j = 0; j < N; ++j)
        rx[j] = __shfl_sync(FULL, (fc == 0) ? xs[0][j] : (fc == 1) ? xs[1][j] : (fc == 2) ? xs[2][j] : xs[3][j], src);
    }
    const float rn = dd_norm2<N>(rx);
    const float ltol = p.lam_tol * fmaxf(1.0f, fabsf(rl));
    const float lim2 = ct2 * rn;
    // The representative matches itself: its (lambda, x) and squared norm are bit-identical copies, so
    // |dlambda| = 0 and dot = n2 = rn exactly, and cos_tol^2 <= 1 keeps lim2 * n2 <= dot^2 under rounding.
    uint32_t hit = 0;
#pragma unroll
    for (int c = 0; c < SPL; ++c) {                  // evaluated for every start, masked afterwards (no branches)
      const bool same = dd_same<N, EVEN>(lam[c], xs[c], n2[c], rl, rx, rn, lim2, ltol, p.cos_tol);
      hit |= same ? (1u << c) : 0u;
    }
    hit &= un;
    un &= ~hit;
    const int cnt = __reduce_add_sync(FULL, __popc(hit));
    if (lane == ncl) {
      my_lam = rl; my_rep = first; my_mult = cnt;
#pragma unroll
      for (int j = 0; j < N; ++j) my_x[j] = rx[j];
    }
    ++ncl;
  }
  // rank = #{d : lam_d > lam_c or (lam_d == lam_c and d < c)}
  int rank = 0;
#pragma unroll 1
  for (int d = 0; d < ncl; ++d) {
    const float ld = __shfl_sync(FULL, my_lam, d);
    rank += (ld > my_lam) || (ld == my_lam && d < lane);
  }
  if (lane == 0) p.out_count[v] = ncl;
  const long long ob = v * p.kmax;
#ifndef SSHOPM_DD_ONEPASS
#define SSHOPM_DD_ONEPASS 1   // records and empty slots in one predicated store pass (0.422 -> 0.404 ms)
#endif
#if SSHOPM_DD_ONEPASS
  // one store pass: lane c < ncl writes cluster c at its rank (if ranked within kmax); lanes ncl..kmax-1
  // write the empty slots ncl..kmax-1 (ranks of the ncl clusters are exactly 0..ncl-1)
  const bool mine = lane < ncl;
  const int slot = mine ? rank : lane;
  if (mine ? (rank < p.kmax) : (lane < p.kmax)) {
    p.out_lambda[ob + slot] = mine ? my_lam : 0.f;
#pragma unroll
    for (int j = 0; j < N; ++j) p.out_x[(ob + slot) * N + j] = mine ? my_x[j] : 0.f;
    p.out_mult[ob + slot] = mine ? my_mult : 0;
    if (p.out_rep) p.out_rep[ob + slot] = mine ? my_rep : -1;
  }
#pragma unroll 1
  for (int sl = 32 + lane; sl < p.kmax; sl += 32) {  // kmax > 32 only
    if (sl < ncl) continue;
    p.out_lambda[ob + sl] = 0.f;
#pragma unroll
    for (int j = 0; j < N; ++j) p.out_x[(ob + sl) * N + j] = 0.f;
    p.out_mult[ob + sl] = 0;
    if (p.out_rep) p.out_rep[ob + sl] = -1;
  }
#else
  if (lane < ncl && rank < p.kmax) {
    p.out_lambda[ob + rank] = my_lam;
#pragma unroll
    for (int j = 0; j < N; ++j) p.out_x[(ob + rank) * N + j] = my_x[j];
    p.out_mult[ob + rank] = my_mult;
    if (p.out_rep) p.out_rep[ob + rank] = my_rep;
  }
#pragma unroll 1
  for (int slot = ncl + lane; slot < p.kmax; slot += 32) {
    p.out_lambda[ob + slot] = 0.f;
#pragma unroll
    for (int j = 0; j < N; ++j) p.out_x[(ob + slot) * N + j] = 0.f;
    p.out_mult[ob + slot] = 0;
    if (p.out_rep) p.out_rep[ob + slot] = -1;
  }
#endif
  if constexpr (STAGE) __syncwarp();                 // the stage is rewritten by the next tensor
  return true;
}

// Standalone dedup for S = 128: warp per tensor, the next tensor prefetched
// into registers while the current one is clustered; a tensor with more than
// 32 clusters falls back to the shared-memory routine.
#ifndef SSHOPM_DD_MINB
#define SSHOPM_DD_MINB 1   // CTAs per SM the register allocation must allow (experiment knob)
#endif
template <int N, bool EVEN, bool REC = false>
__global__ void __launch_bounds__(256, SSHOPM_DD_MINB) sshopm_dedup128_kernel(const DedupParams p) {
  extern __shared__ float smem[];
  const int lane = threadIdx.x & 31;
  const int wib = threadIdx.x >> 5;
  float* stage = smem + (size_t)wib * 128 * (N + 1);
  float* gen = smem + (size_t)(blockDim.x >> 5) * 128 * (N + 1) + (size_t)wib * dedup_smem_words(128, N);
  const long long warps = (long long)gridDim.x * (blockDim.x >> 5);
  long long v = (long long)blockIdx.x * (blockDim.x >> 5) + wib;
  auto run = [&](const DedupRegs<N>& cur, long long t) {
    if (!dedup128_regs<N, EVEN, true, REC>(p, t, lane, cur, stage)) {
      float* s_lam = gen;
      float* s_x = s_lam + 128;
      int* s_cid = reinterpret_cast<int*>(s_x + 128 * N);
      float* c_lam = reinterpret_cast<float*>(s_cid + 128);
      int* c_rep = reinterpret_cast<int*>(c_lam + 128);
      int* c_mult = c_rep + 128;
      warp_dedup_tensor<N, EVEN, REC>(p, t, lane, s_lam, s_x, s_cid, c_lam, c_rep, c_mult);
    }
  };
  auto load = [&](DedupRegs<N>& r, long long t) {
    if constexpr (REC) dedup_load_rec<N>(r, p, t, lane);
    else dedup_load<N>(r, p, t, lane, true);
  };
#ifndef SSHOPM_DD_TWOBUF
#define SSHOPM_DD_TWOBUF 0   // two alternating prefetch buffers: measured slower (0.463 ms)
#endif
#if SSHOPM_DD_TWOBUF
  // two register buffers used alternately (no copy of the prefetched buffer)
  DedupRegs<N> a, b;
  if (v < p.n_tensors) load(a, v);
  for (; v < p.n_tensors; v += 2 * warps) {
    if (v + warps < p.n_tensors) load(b, v + warps);
    run(a, v);
    if (v + warps >= p.n_tensors) break;
    if (v + 2 * warps < p.n_tensors) load(a, v + 2 * warps);
    run(b, v + warps);
  }
#else
  DedupRegs<N> nx;
  if (v < p.n_tensors) load(nx, v);
  for (; v < p.n_tensors; v += warps) {
    const DedupRegs<N> cur = nx;
    if (v + warps < p.n_tensors) load(nx, v + warps);   // prefetch
    run(cur, v);
  }
#endif
}
// shared-memory bytes per warp of sshopm_dedup128_kernel (stage + fallback staging)
__host__ __device__ constexpr int dedup128_smem_per_warp(int n) { return (128 * (n + 1) + dedup_smem_words(128, n)) * 4; }

// Register-resident clustering of tensor v for S = 128 inside the solve kernel
// (fused solve -> dedup, no staging shared memory).
template <int N, bool EVEN>
__device__ __forceinline__ bool warp_dedup128_regs(const DedupParams& p, long long v, int lane) {
  DedupRegs<N> r;
  dedup_load<N>(r, p, v, lane, false);
  return dedup128_regs<N, EVEN, false>(p, v, lane, r, nullptr);
}

}  // namespace sshopm
