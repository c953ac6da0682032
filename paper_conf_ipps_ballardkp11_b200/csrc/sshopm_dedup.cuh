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
  for (long long v = (long long)blockIdx.x * (blockDim.x >> 5) + wib; v < p.n_tensors; v += warps) {
    const long long b = v * S;
    for (int s = lane; s < S; s += 32) {
      s_lam[s] = p.lambda[b + s];
      s_cid[s] = p.conv[b + s] ? -1 : -2;
    }
    for (int t = lane; t < S * N; t += 32) s_x[t] = p.x[b * N + t];
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
}

}  // namespace sshopm
