// symm_tables.cuh — compile-time index-class tables for R^[M,N] (device side).
//
// The paper computes index representations with UPDATEINDEX (Fig. 4,
// P:L223-253) and multinomials with MULTINOMIAL0/1
// at run time in its "general" kernel, and folds them into straight-line code
// in its unrolled (4,3) kernel (Sec. V-D: "indices and
// coefficients ... computed during the code generation at compile time").
// We do the latter for every compiled (M, N): all tables below are constexpr,
// so after full unrolling every index, class position and coefficient is an
// immediate in the SASS.
//
// Regrouping used by the kernels: Eq. 6
//   (A x^{M-1})_j = sum_{classes, k_j>0} sigma_c(j) a_c x^{k-e_j}
// is re-indexed by the degree-(M-1) monomial q = k - e_j:
//   (A x^{M-1})_j = sum_{|q| = M-1} [(M-1)!/q!] * a_{class(q + e_j)} * x^q,
// since sigma_{q+e_j}(j) = (M-1)!/prod_i (q_i)!.  The Q = C(M+N-2, M-1)
// scaled monomials are shared by all N outputs.  A x^M is then x . (A x^{M-1})
// (Definition 2 / Euler's identity), so the U-term Eq. 4 kernel is not needed.
#pragma once
#include <utility>

namespace sshopm {

constexpr int binom(int n, int k) {
  if (k < 0 || k > n) return 0;
  long long r = 1;
  for (int i = 1; i <= k; ++i) r = r * (n - k + i) / i;
  return (int)r;
}
constexpr long long fact(int n) { long long r = 1; for (int i = 2; i <= n; ++i) r *= i; return r; }

// Successor of a nondecreasing 0-based index tuple of length d over {0..n-1}
// (the Fig. 4 rule).  Returns false after the last tuple.
constexpr bool next_tuple(int* I, int d, int n) {
  int j = d - 1;
  while (j >= 0 && I[j] == n - 1) --j;
  if (j < 0) return false;
  I[j] += 1;
  for (int k = j + 1; k < d; ++k) I[k] = I[j];
  return true;
}

// Lexicographic rank of a nondecreasing tuple of length d (0-based) among all
// such tuples: count tuples that precede it.
constexpr int tuple_rank(const int* I, int d, int n) {
  int r = 0, lo = 0;
  for (int p = 0; p < d; ++p) {
    for (int v = lo; v < I[p]; ++v) r += binom((d - p - 1) + (n - v) - 1, d - p - 1);  // tuples with prefix..v at p
    lo = I[p];
  }
  return r;
}

template <int M, int N>
struct Tables {
  static constexpr int U = binom(M + N - 1, M);        // unique entries (Property 1)
  static constexpr int D = M - 1;                      // degree of the monomials in A x^{M-1}
  static constexpr int Q = binom(D + N - 1, D);        // number of degree-D monomials
  static constexpr int H = (D + 1) / 2;                // lower monomials computed up to degree H
  static constexpr int DL = D - H;                     // target q = (degree DL part) x (degree H part)
  static constexpr int T1 = N * Q;                     // terms of A x^{M-1}
  // lower monomial list: degrees 1..H, each degree block in lex order
  static constexpr int NL = []() { int s = 0; for (int d = 1; d <= H; ++d) s += binom(d + N - 1, d); return s; }();

  int cls_idx[U][M > 0 ? M : 1];  // index representation of class c (0-based)
  int deg_off[H + 2];             // offset of degree-d block in the lower list (deg_off[1] = 0)
  int low_parent[NL > 0 ? NL : 1];// degree >= 2: parent (degree d-1) lower-list index
  int low_var[NL > 0 ? NL : 1];   // variable multiplied onto the parent (degree 1: the variable itself)
  int q_left[Q];                  // lower-list index of the degree-DL prefix (-1 if DL == 0)
  int q_right[Q];                 // lower-list index of the degree-H suffix (-1 if H == 0)
  int q_cls[Q][N];                // class position of q + e_j
  long long q_coef[Q];            // (M-1)! / q!
  long long cls_mult[U];          // M! / k! : tensor indices in class c (Property 2)
  int n_products;                 // FP32 multiplies to form the Q monomials (no coefficient)

  constexpr Tables() : cls_idx(), deg_off(), low_parent(), low_var(), q_left(), q_right(), q_cls(), q_coef(), cls_mult(), n_products(0) {
    // classes of degree M in lex order
    {
      int I[M > 0 ? M : 1] = {};
      for (int c = 0; c < U; ++c) {
        long long den = 1;
        int run = 1;
        for (int t = 0; t < M; ++t) {
          cls_idx[c][t] = I[t];
          if (t > 0 && I[t] == I[t - 1]) { ++run; den *= run; } else run = 1;
        }
        cls_mult[c] = fact(M) / den;
        next_tuple(I, M, N);
      }
    }
    // lower monomials, degree 1..H
    int off = 0;
    for (int d = 1; d <= H; ++d) {
      deg_off[d] = off;
      int I[M > 0 ? M : 1] = {};
      int cnt = binom(d + N - 1, d);
      for (int t = 0; t < cnt; ++t) {
        if (d == 1) { low_parent[off + t] = -1; low_var[off + t] = I[0]; }
        else {
          low_parent[off + t] = deg_off[d - 1] + tuple_rank(I, d - 1, N);
          low_var[off + t] = I[d - 1];
          n_products += 1;
        }
        next_tuple(I, d, N);
      }
      off += cnt;
    }
    deg_off[H + 1] = off;
    // degree-D targets
    int I[M > 0 ? M : 1] = {};
    for (int q = 0; q < Q; ++q) {
      q_left[q] = DL > 0 ? deg_off[DL] + tuple_rank(I, DL, N) : -1;
      q_right[q] = H > 0 ? deg_off[H] + tuple_rank(I + DL, H, N) : -1;
      if (DL > 0 && H > 0) n_products += 1;
      long long den = 1; int run = 1;
      for (int t = 1; t < D; ++t) { if (I[t] == I[t - 1]) { ++run; den *= run; } else run = 1; }
      q_coef[q] = fact(D) / den;
      for (int j = 0; j < N; ++j) {
        // insert j into the sorted tuple I (length D) -> class of degree M
        int K[M > 0 ? M : 1] = {};
        int a = 0, b = 0; bool ins = false;
        while (b < M) {
          if (!ins && (a >= D || j <= I[a])) { K[b++] = j; ins = true; }
          else K[b++] = I[a++];
        }
        q_cls[q][j] = tuple_rank(K, M, N);
      }
      next_tuple(I, D, N);
    }
  }
};

// Degree-(M-2) tables for A x^{M-2} (Definition 2 with p = 2, used by the
// eigenpair classification): (A x^{M-2})_{ij} = sum_{|r| = M-2} [(M-2)!/r!] a_{class(r + e_i + e_j)} x^r.
template <int M, int N>
struct Tables2 {
  static constexpr int D2 = M - 2;
  static constexpr int Q2 = binom(D2 + N - 1, D2);     // 1 when M = 2 (the empty monomial)
  static constexpr int NPR = N * (N + 1) / 2;          // pairs i <= j
  int r_idx[Q2][D2 > 0 ? D2 : 1];
  long long r_coef[Q2];
  int r_cls[Q2][NPR];
  constexpr Tables2() : r_idx(), r_coef(), r_cls() {
    int I[M > 2 ? M - 2 : 1] = {};
    for (int q = 0; q < Q2; ++q) {
      long long den = 1; int run = 1;
      for (int t = 0; t < D2; ++t) {
        r_idx[q][t] = I[t];
        if (t > 0 && I[t] == I[t - 1]) { ++run; den *= run; } else run = 1;
      }
      r_coef[q] = fact(D2) / den;
      int pr = 0;
      for (int i = 0; i < N; ++i)
        for (int j = i; j < N; ++j) {
          int K[M] = {};
          int a = 0, b = 0, ins = 0;
          const int add[2] = {i, j};
          while (b < M) {                                  // merge the sorted tuple I with (i, j)
            if (ins < 2 && (a >= D2 || add[ins] <= I[a])) K[b++] = add[ins++];
            else K[b++] = I[a++];
          }
          r_cls[q][pr++] = tuple_rank(K, M, N);
        }
      if (D2 > 0) next_tuple(I, D2, N);
    }
  }
};

// Flop counts.
template <int M, int N>
constexpr long long paper_flops_per_iter() {
  // Reading R12: (M+2) U + (M+1) T1 + 5N
  return (long long)(M + 2) * Tables<M, N>::U + (long long)(M + 1) * Tables<M, N>::T1 + 5LL * N;
}

template <int M, int N>
constexpr long long executed_flops_per_iter() {
  // monomials (FMUL) + T1 terms (FMA = 2) + lambda = x.g (2N-1) + shift (2N) + ||.||^2 (2N-1) + scale (N)
  constexpr Tables<M, N> T{};
  return (long long)T.n_products + 2LL * T.T1 + (2LL * N - 1) + 2LL * N + (2LL * N - 1) + N;
}

// compile-time loop: f(std::integral_constant<int, I>{}) for I in [0, Count)
template <int Count, typename F, int... Is>
__host__ __device__ __forceinline__ constexpr void static_for_impl(F&& f, std::integer_sequence<int, Is...>) {
  (f(std::integral_constant<int, Is>{}), ...);
}
template <int Count, typename F>
__host__ __device__ __forceinline__ constexpr void static_for(F&& f) {
  static_for_impl<Count>(f, std::make_integer_sequence<int, Count>{});
}

}  // namespace sshopm
