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
};

// shared-memory words per warp for S starts, dimension n
__host__ __device__ constexpr int dedup_smem_words(int S, int n) { return S * (n + 2) + 3 * S; }

// One warp clusters tensor v (R16).  Staging arrays (per warp, shared memory):
// s_lam[S], s_x[S*N], s_cid[S], c_lam[S], c_rep[S], c_mult[S].  Inputs are read
// with ld.global.cg (L2), so the routine is also safe right after other lanes
// of the same warp wrote them (fused solve -> dedup; caller fences).
template <int N, bool EVEN>
__device__ __forceinline__ void warp_dedup_tensor(const DedupParams& p, long long v, int lane, float* s_lam,
                                                  float* s_x, int* s_cid, float* c_lam, int* c_rep, int* c_mult) {
  const int S = p.S;
  const long long b = v * S;
  for (int s = lane; s < S; s += 32) {
    s_lam[s] = __ldcg(p.lambda + b + s);
    s_cid[s] = __ldcg(p.conv + b + s) ? -1 : -2;
  }
  for (int t = lane; t < S * N; t += 32) s_x[t] = __ldcg(p.x + b * N + t);
  __syncwarp();

  int ncl = 0;
  for (;;) {
    int first = 0x7fffffff;
    for (int s = lane; s < S; s += 32)
      if (s_cid[s] == -1) { first = s; break; }
    first = __reduce_min_sync(0xffffffffu, first);
    if (first == 0x7fffffff) break;
    const float rl = s_lam[first];
    float rx[N];
    float rn = 0.f;
#pragma unroll
    for (int j = 0; j < N; ++j) { rx[j] = s_x[first * N + j]; rn = fmaf(rx[j], rx[j], rn); }
    const float ltol = p.lam_tol * fmaxf(1.0f, fabsf(rl));
    int cnt = 0;
    for (int s = lane; s < S; s += 32) {
      if (s_cid[s] != -1) continue;
      bool same = (s == first);
      if (!same) {
        const float ls = s_lam[s];
        float dot = 0.f, n2 = 0.f;
#pragma unroll
        for (int j = 0; j < N; ++j) { const float xv = s_x[s * N + j]; dot = fmaf(xv, rx[j], dot); n2 = fmaf(xv, xv, n2); }
        const float lim = p.cos_tol * sqrtf(n2 * rn);
        if (EVEN) same = fabsf(ls - rl) <= ltol && fabsf(dot) >= lim;
        else same = (fabsf(ls - rl) <= ltol && dot >= lim) || (fabsf(-ls - rl) <= ltol && -dot >= lim);
      }
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

template <int N, bool EVEN>
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
    warp_dedup_tensor<N, EVEN>(p, v, lane, s_lam, s_x, s_cid, c_lam, c_rep, c_mult);
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
// Fast path for S = 128: lane l owns starts 4l..4l+3 in registers, loaded as
// float4 (lambda: 1, x: N, converged: one u32), and the next tensor is
// prefetched while the current one is clustered.  Same rounds as above (round
// representative = first unassigned converged start in start order).
template <int N>
struct DedupRegs {
  float4 lam;
  float4 x[N];      // 4 starts x N components, start-major
  uint32_t conv;    // 4 bytes
};

template <int N>
__device__ __forceinline__ void dedup_load(DedupRegs<N>& r, const DedupParams& p, long long v, int lane) {
  const long long b = v * 128;
  r.lam = __ldcs(reinterpret_cast<const float4*>(p.lambda + b) + lane);
#pragma unroll
  for (int i = 0; i < N; ++i) r.x[i] = __ldcs(reinterpret_cast<const float4*>(p.x + b * N) + lane * N + i);
  r.conv = __ldcs(reinterpret_cast<const unsigned int*>(p.conv + b) + lane);
}

template <int N>
__device__ __forceinline__ float xcomp(const DedupRegs<N>& r, int c, int j) {   // component j of local start c (c, j compile-time)
  const int w = c * N + j;
  const float4 q = r.x[w / 4];
  return (w % 4 == 0) ? q.x : (w % 4 == 1) ? q.y : (w % 4 == 2) ? q.z : q.w;
}

template <int N, bool EVEN>
__global__ void __launch_bounds__(256) sshopm_dedup128_kernel(const DedupParams p) {
  constexpr int S = 128, SPL = 4;
  extern __shared__ float smem[];
  const int lane = threadIdx.x & 31;
  const int wib = threadIdx.x >> 5;
  // per-warp cluster records: lam[S], rep[S], mult[S], x[S][N]
  float* c_lam = smem + (size_t)wib * S * (N + 3);
  int* c_rep = reinterpret_cast<int*>(c_lam + S);
  int* c_mult = c_rep + S;
  float* c_x = reinterpret_cast<float*>(c_mult + S);

  const long long warps = (long long)gridDim.x * (blockDim.x >> 5);
  long long v = (long long)blockIdx.x * (blockDim.x >> 5) + wib;
  DedupRegs<N> nx;
  if (v < p.n_tensors) dedup_load<N>(nx, p, v, lane);
  for (; v < p.n_tensors; v += warps) {
    const DedupRegs<N> cur = nx;
    if (v + warps < p.n_tensors) dedup_load<N>(nx, p, v + warps, lane);   // prefetch
    const float lam[SPL] = {cur.lam.x, cur.lam.y, cur.lam.z, cur.lam.w};
    // cid: -1 unassigned converged, -2 not converged, >= 0 cluster
    int cid[SPL];
#pragma unroll
    for (int c = 0; c < SPL; ++c) cid[c] = ((cur.conv >> (8 * c)) & 0xffu) ? -1 : -2;
    int ncl = 0;
    for (;;) {
      int first = 0x7fffffff;
#pragma unroll
      for (int c = SPL - 1; c >= 0; --c)
        if (cid[c] == -1) first = SPL * lane + c;
      first = __reduce_min_sync(0xffffffffu, first);
      if (first == 0x7fffffff) break;
      const int src = first / SPL, fc = first % SPL;
      float rl = (fc == 0) ? lam[0] : (fc == 1) ? lam[1] : (fc == 2) ? lam[2] : lam[3];
      rl = __shfl_sync(0xffffffffu, rl, src);
      float rx[N];
      float rn = 0.f;
#pragma unroll
      for (int j = 0; j < N; ++j) {
        float t = (fc == 0) ? xcomp<N>(cur, 0, j) : (fc == 1) ? xcomp<N>(cur, 1, j) : (fc == 2) ? xcomp<N>(cur, 2, j) : xcomp<N>(cur, 3, j);
        rx[j] = __shfl_sync(0xffffffffu, t, src);
        rn = fmaf(rx[j], rx[j], rn);
      }
      const float ltol = p.lam_tol * fmaxf(1.0f, fabsf(rl));
      int cnt = 0;
#pragma unroll
      for (int c = 0; c < SPL; ++c) {
        if (cid[c] != -1) continue;
        bool same = (SPL * lane + c == first);
        if (!same) {
          float dot = 0.f, n2 = 0.f;
#pragma unroll
          for (int j = 0; j < N; ++j) { const float xv = xcomp<N>(cur, c, j); dot = fmaf(xv, rx[j], dot); n2 = fmaf(xv, xv, n2); }
          const float lim = p.cos_tol * sqrtf(n2 * rn);
          if (EVEN) same = fabsf(lam[c] - rl) <= ltol && fabsf(dot) >= lim;
          else same = (fabsf(lam[c] - rl) <= ltol && dot >= lim) || (fabsf(-lam[c] - rl) <= ltol && -dot >= lim);
        }
        if (same) { cid[c] = ncl; ++cnt; }
      }
      cnt = __reduce_add_sync(0xffffffffu, cnt);
      if (lane == 0) {
        c_lam[ncl] = rl; c_rep[ncl] = first; c_mult[ncl] = cnt;
#pragma unroll
        for (int j = 0; j < N; ++j) c_x[ncl * N + j] = rx[j];
      }
      ++ncl;
    }
    __syncwarp();
    if (lane == 0) p.out_count[v] = ncl;
    const long long ob = v * p.kmax;
    for (int c = lane; c < ncl; c += 32) {
      const float lc = c_lam[c];
      int rank = 0;
      for (int d = 0; d < ncl; ++d) {
        const float ld = c_lam[d];
        rank += (ld > lc) || (ld == lc && d < c);
      }
      if (rank < p.kmax) {
        p.out_lambda[ob + rank] = lc;
#pragma unroll
        for (int j = 0; j < N; ++j) p.out_x[(ob + rank) * N + j] = c_x[c * N + j];
        p.out_mult[ob + rank] = c_mult[c];
        if (p.out_rep) p.out_rep[ob + rank] = c_rep[c];
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
}

// Register-resident clustering of tensor v for S = 128 (fused solve -> dedup):
// lane l owns starts 4l..4l+3 (float4 loads through L2), cluster c's record
// lives in lane c's registers.  Returns false (nothing written) if the tensor
// has more than 32 clusters; the caller then hands it to the list kernel.
template <int N, bool EVEN>
__device__ __forceinline__ bool warp_dedup128_regs(const DedupParams& p, long long v, int lane) {
  constexpr int SPL = 4;
  const long long b = v * 128;
  const float4 l4 = __ldcg(reinterpret_cast<const float4*>(p.lambda + b) + lane);
  float4 x4[N];
#pragma unroll
  for (int i = 0; i < N; ++i) x4[i] = __ldcg(reinterpret_cast<const float4*>(p.x + b * N) + lane * N + i);
  const uint32_t cv4 = __ldcg(reinterpret_cast<const unsigned int*>(p.conv + b) + lane);
  const float lam[SPL] = {l4.x, l4.y, l4.z, l4.w};
  auto xc = [&](int c, int j) -> float {
    const int w = c * N + j;
    const float4 q = x4[w / 4];
    return (w % 4 == 0) ? q.x : (w % 4 == 1) ? q.y : (w % 4 == 2) ? q.z : q.w;
  };
  int cid[SPL];
#pragma unroll
  for (int c = 0; c < SPL; ++c) cid[c] = ((cv4 >> (8 * c)) & 0xffu) ? -1 : -2;
  float my_lam = 0.f, my_x[N];
  int my_rep = -1, my_mult = 0;
#pragma unroll
  for (int j = 0; j < N; ++j) my_x[j] = 0.f;
  int ncl = 0;
#pragma unroll 1
  for (;;) {
    int first = 0x7fffffff;
#pragma unroll
    for (int c = SPL - 1; c >= 0; --c)
      if (cid[c] == -1) first = SPL * lane + c;
    first = __reduce_min_sync(0xffffffffu, first);
    if (first == 0x7fffffff) break;
    if (ncl == 32) return false;                      // too many clusters for the register form
    const int src = first / SPL, fc = first % SPL;
    float rl = (fc == 0) ? lam[0] : (fc == 1) ? lam[1] : (fc == 2) ? lam[2] : lam[3];
    rl = __shfl_sync(0xffffffffu, rl, src);
    float rx[N];
    float rn = 0.f;
#pragma unroll
    for (int j = 0; j < N; ++j) {
      const float t = (fc == 0) ? xc(0, j) : (fc == 1) ? xc(1, j) : (fc == 2) ? xc(2, j) : xc(3, j);
      rx[j] = __shfl_sync(0xffffffffu, t, src);
      rn = fmaf(rx[j], rx[j], rn);
    }
    const float ltol = p.lam_tol * fmaxf(1.0f, fabsf(rl));
    int cnt = 0;
#pragma unroll
    for (int c = 0; c < SPL; ++c) {
      if (cid[c] != -1) continue;
      bool same = (SPL * lane + c == first);
      if (!same) {
        float dot = 0.f, n2 = 0.f;
#pragma unroll
        for (int j = 0; j < N; ++j) { const float xv = xc(c, j); dot = fmaf(xv, rx[j], dot); n2 = fmaf(xv, xv, n2); }
        const float lim = p.cos_tol * sqrtf(n2 * rn);
        if (EVEN) same = fabsf(lam[c] - rl) <= ltol && fabsf(dot) >= lim;
        else same = (fabsf(lam[c] - rl) <= ltol && dot >= lim) || (fabsf(-lam[c] - rl) <= ltol && -dot >= lim);
      }
      if (same) { cid[c] = ncl; ++cnt; }
    }
    cnt = __reduce_add_sync(0xffffffffu, cnt);
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
    const float ld = __shfl_sync(0xffffffffu, my_lam, d);
    rank += (ld > my_lam) || (ld == my_lam && d < lane);
  }
  if (lane == 0) p.out_count[v] = ncl;
  const long long ob = v * p.kmax;
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
  return true;
}

}  // namespace sshopm
