// general.h — table-driven kernel for any (m, n) (general.cu).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>
#include "sshopm.h"

namespace sshopm {

constexpr int kGenMaxM = 16;     // order limit of the general kernel
constexpr int kGenMaxN = 16;     // dimension limit
constexpr long long kGenMaxU = 1 << 16;

constexpr long long kGen2MaxWords = 1500;   // item-per-lane kernel: per-lane shared words U + L (32 lanes per warp)
constexpr long long kBlkMaxT1 = 1 << 16;    // blocked kernel / tables: at most this many (q, j) terms

struct GeneralTables {           // host copies; uploaded per call (handles own no device memory)
  int m = 0, n = 0, U = 0;
  uint8_t* idx = nullptr;        // [U][m] index representations, lexicographic (Fig. 4 walk)
  int* mult = nullptr;           // [U] m!/k! (Property 2)
  long long paper_flops = 0, exec_flops = 0;
  // item-per-lane kernel (null when U + L > kGen2MaxWords: the block-per-tensor kernel is used)
  int L = 0, Q = 0;              // monomials of degree 1..m-1; those of degree m-1
  uint32_t* recipe = nullptr;    // [L] parent | var << 16 (degree >= 2)
  float* coef = nullptr;         // [Q] (m-1)!/q!
  uint32_t* cls = nullptr;       // [Q][n] 128 * class(q + e_j)
  bool gen2 = false;             // the item-per-lane kernel's per-lane arrays fit (U + L <= kGen2MaxWords)
  // blocked kernel (blocked.cu): classes unscaled and the degree-(m-2) prefixes' last indices
  uint32_t* cls_idx = nullptr;   // [Q][n] class(q + e_j)
  int P = 0;                     // degree-(m-2) monomials (1 for m = 2: the empty prefix)
  uint32_t* plast = nullptr;     // [P] their last (largest) index, lexicographic order
  uint32_t* porder = nullptr;    // [P] prefixes grouped by last index (stable)
  uint32_t* ppar = nullptr;      // [P] for porder[k]: recipe index of its own prefix p - e_last (m >= 4; else 0)
  uint32_t* gcnt = nullptr;      // [n] prefixes per last index
  uint32_t* qperm = nullptr;     // [Q] B-row order: for p in porder, q = p + e_i for i = last(p)..n-1
};

GeneralTables* general_create(int m, int n);
void general_destroy(GeneralTables* t);
int general_solve(const GeneralTables* t, int64_t N, const float* d_entries, int S, const float* d_starts, float alpha,
                  float tol, int maxit, float* d_lambda, float* d_x, int32_t* d_iters, uint8_t* d_conv,
                  const sshopm_solve_opts* opts, cudaStream_t st);
int blocked_solve(const GeneralTables* t, int64_t N, const float* d_entries, int S, const float* d_starts, float alpha,
                  float tol, int maxit, float* d_lambda, float* d_x, int32_t* d_iters, uint8_t* d_conv,
                  const sshopm_solve_opts* opts, cudaStream_t st);
bool blocked_fits(const GeneralTables* t);
int general_apply(const GeneralTables* t, int64_t N, const float* d_entries, const float* d_x, float* d_g, float* d_lam,
                  cudaStream_t st);

}  // namespace sshopm
