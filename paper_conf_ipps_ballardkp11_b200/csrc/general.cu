// general.cu — table-driven SS-HOPM for any (m, n) (the paper's "general"
// implementation).
//
// Mapping as in the paper: one block per tensor (grid-stride),
// its U entries and the shared index/multinomial tables in shared memory
// ("the index information is stored as an array of size m x U and can
// be shared by all threads ... We store the multinomial coefficient for each
// unique tensor value"), one thread per start.  Per evaluation each thread
// walks the U classes (Fig. 2/3 order); for the first occurrence t of each
// index i in the class it adds sigma(i) a_c x^{k - e_i} with
// sigma(i) = c * k_i / m and x^{k - e_i} = prefix(t) * suffix(t) (the
// product without one occurrence of i — never a division, reading R10).
// lambda = x . g (Euler identity).  Stopping rule, shift and outputs are
// exactly those of the specialised kernels (readings R1-R7).
#include <cstdio>
#include <cstring>
#include <new>

#include "api_internal.h"
#include "general.h"
#include "sshopm.h"

namespace sshopm {

struct GenParams {
  const float* entries;      // [N][U]
  const float* starts;       // [S][n] raw
  const uint8_t* cls_idx;    // [U][m] 0-based
  const int* cls_mult;       // [U]  m!/k!
  float* out_lambda;
  float* out_x;
  int32_t* out_iters;
  uint8_t* out_conv;
  unsigned long long* total_iters;
  const float* alpha_in;     // alpha_mode 1
  long long N;
  int m, n, U, S;
  float alpha, tol;
  int alpha_mode, maxit;
};

// g = A x^{m-1} (Eq. 6 by classes) for this thread; x, g in the thread's shared slots
__device__ __forceinline__ void gen_eval(const GenParams& p, const float* __restrict__ ent, const uint8_t* __restrict__ idx,
                                         const int* __restrict__ mult, const float* x, float* g) {
  const int m = p.m, n = p.n;
  for (int j = 0; j < n; ++j) g[j] = 0.f;
  float suf[kGenMaxM + 1];
  for (int c = 0; c < p.U; ++c) {
    const uint8_t* I = idx + c * m;
    suf[m] = 1.f;
    for (int t = m - 1; t >= 0; --t) suf[t] = suf[t + 1] * x[I[t]];
    const float ca = (float)mult[c] * ent[c] / (float)m;        // c * a_c / m
    float pre = 1.f;
    int t = 0;
    while (t < m) {
      const int i = I[t];
      int k = 1;
      while (t + k < m && I[t + k] == i) ++k;
      g[i] = fmaf(ca * (float)k, pre * suf[t + 1], g[i]);      // sigma(i) a_c x^{k - e_i}
      for (int r = 0; r < k; ++r) pre *= x[i];
      t += k;
    }
  }
}

__global__ void __launch_bounds__(128) sshopm_general_kernel(const GenParams p) {
  extern __shared__ float gsm[];
  const int m = p.m, n = p.n, U = p.U;
  float* ent = gsm;                                                   // [U]
  int* mult = reinterpret_cast<int*>(ent + U);                        // [U]
  float* xs = reinterpret_cast<float*>(mult + U) + threadIdx.x * (2 * n + 1);
  float* g = xs + n;
  uint8_t* idx = reinterpret_cast<uint8_t*>(reinterpret_cast<float*>(mult + U) + blockDim.x * (2 * n + 1));
  for (int i = threadIdx.x; i < U * m; i += blockDim.x) idx[i] = p.cls_idx[i];
  for (int i = threadIdx.x; i < U; i += blockDim.x) mult[i] = p.cls_mult[i];
  unsigned long long it_sum = 0;
  for (long long v = blockIdx.x; v < p.N; v += gridDim.x) {
    __syncthreads();
    for (int i = threadIdx.x; i < U; i += blockDim.x) ent[i] = p.entries[v * U + i];
    __syncthreads();
    float alpha = p.alpha;
    if (p.alpha_mode == 1) {
      alpha = p.alpha_in[v];
    } else if (p.alpha_mode >= 2) {
      float b = 0.f;
      for (int c = 0; c < U; ++c) b = fmaf((float)mult[c], fabsf(ent[c]), b);
      alpha = (p.alpha_mode == 2 ? 1.f : -1.f) * (float)(m - 1) * b;
    }
    const float sg = alpha >= 0.f ? 1.f : -1.f;                      // Fig. 1 lines 2-5 (R5)
    for (int s = threadIdx.x; s < p.S; s += blockDim.x) {
      float nn = 0.f;
      for (int j = 0; j < n; ++j) { xs[j] = p.starts[(size_t)s * n + j]; nn = fmaf(xs[j], xs[j], nn); }
      const float r0 = nn > 0.f ? rsqrtf(nn) : 0.f;                  // R7
      for (int j = 0; j < n; ++j) xs[j] *= r0;
      float lamp = __int_as_float(0x7fffffff), lam = 0.f;
      int k = 0;
      bool conv = false;
      for (;;) {
        gen_eval(p, ent, idx, mult, xs, g);
        lam = 0.f;
        for (int j = 0; j < n; ++j) lam = fmaf(xs[j], g[j], lam);   // lambda_k = x_k . g
        conv = fabsf(lam - lamp) <= p.tol * fmaxf(1.0f, fabsf(lam)); // R2
        if (conv || k >= p.maxit) break;
        float h2 = 0.f;
        for (int j = 0; j < n; ++j) { g[j] = sg * fmaf(alpha, xs[j], g[j]); h2 = fmaf(g[j], g[j], h2); }
        if (!(h2 >= 1.17549435e-38f)) break;                         // R6
        const float r = rsqrtf(h2);
        for (int j = 0; j < n; ++j) xs[j] = g[j] * r;
        lamp = lam;
        ++k;
      }
      const long long item = v * p.S + s;
      p.out_lambda[item] = lam;
      for (int j = 0; j < n; ++j) p.out_x[item * n + j] = xs[j];
      p.out_iters[item] = k;
      p.out_conv[item] = conv ? 1 : 0;
      it_sum += (unsigned long long)k;
    }
  }
  if (p.total_iters && it_sum) atomicAdd(p.total_iters, it_sum);
}

// test hook: g = A x^{m-1}, lambda = x . g for N (tensor, x) pairs (thread per pair)
__global__ void __launch_bounds__(128) sshopm_general_apply_kernel(const GenParams p, const float* __restrict__ x,
                                                                   float* __restrict__ out_g, float* __restrict__ out_lam) {
  extern __shared__ float gsm[];
  const int m = p.m, n = p.n, U = p.U;
  int* mult = reinterpret_cast<int*>(gsm);
  float* xs = reinterpret_cast<float*>(mult + U) + threadIdx.x * (2 * n + 1);
  float* g = xs + n;
  uint8_t* idx = reinterpret_cast<uint8_t*>(reinterpret_cast<float*>(mult + U) + blockDim.x * (2 * n + 1));
  for (int i = threadIdx.x; i < U * m; i += blockDim.x) idx[i] = p.cls_idx[i];
  for (int i = threadIdx.x; i < U; i += blockDim.x) mult[i] = p.cls_mult[i];
  __syncthreads();
  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < p.N; i += (long long)gridDim.x * blockDim.x) {
    for (int j = 0; j < n; ++j) xs[j] = x[i * n + j];
    gen_eval(p, p.entries + i * U, idx, mult, xs, g);
    float lam = 0.f;
    for (int j = 0; j < n; ++j) { out_g[i * n + j] = g[j]; lam = fmaf(xs[j], g[j], lam); }
    out_lam[i] = lam;
  }
}

// ------------------------------------------------------------------ host --
static long long binom_ll(int a, int b) {
  if (b < 0 || b > a) return 0;
  long long r = 1;
  for (int i = 1; i <= b; ++i) r = r * (a - b + i) / i;
  return r;
}

GeneralTables* general_create(int m, int n) {
  if (m < 2 || n < 1 || m > kGenMaxM || n > kGenMaxN) return nullptr;
  const long long U = binom_ll(m + n - 1, m);
  if (U > kGenMaxU) return nullptr;
  GeneralTables* t = new (std::nothrow) GeneralTables;
  if (!t) return nullptr;
  t->m = m;
  t->n = n;
  t->U = (int)U;
  t->idx = new (std::nothrow) uint8_t[U * m];
  t->mult = new (std::nothrow) int[U];
  if (!t->idx || !t->mult) { general_destroy(t); return nullptr; }
  // Fig. 4 UPDATEINDEX walk from [0..0]; multinomial by one pass
  int I[kGenMaxM] = {};
  long long fm = 1;
  for (int i = 2; i <= m; ++i) fm *= i;
  for (long long c = 0; c < U; ++c) {
    long long den = 1;
    int run = 1;
    for (int k = 0; k < m; ++k) {
      t->idx[c * m + k] = (uint8_t)I[k];
      if (k > 0 && I[k] == I[k - 1]) { ++run; den *= run; } else run = 1;
    }
    t->mult[c] = (int)(fm / den);
    int j = m - 1;
    while (j >= 0 && I[j] == n - 1) --j;
    if (j < 0) break;
    I[j] += 1;
    for (int k = j + 1; k < m; ++k) I[k] = I[j];
  }
  const long long Q = binom_ll(m + n - 2, m - 1);
  t->paper_flops = (long long)(m + 2) * U + (long long)(m + 1) * n * Q + 5LL * n;
  // executed per update: per class ~ (m suffix + m prefix + 3 per unique index) + lambda/shift/normalise
  t->exec_flops = U * (2LL * m + 3LL * n / 2) + 7LL * n;
  return t;
}

void general_destroy(GeneralTables* t) {
  if (!t) return;
  delete[] t->idx;
  delete[] t->mult;
  delete t;
}

size_t general_table_bytes(const GeneralTables* t) { return ((size_t)t->U * t->m + 255) / 256 * 256 + (size_t)t->U * 4; }

static int general_smem(const GeneralTables* t, int block, bool with_entries) {
  return (with_entries ? t->U * 4 : 0) + t->U * 4 + block * (2 * t->n + 1) * 4 + t->U * t->m;
}

int general_upload(const GeneralTables* t, void* dev, cudaStream_t st, const uint8_t** d_idx, const int** d_mult) {
  uint8_t* di = reinterpret_cast<uint8_t*>(dev);
  int* dm = reinterpret_cast<int*>(di + ((size_t)t->U * t->m + 255) / 256 * 256);
  cudaError_t e = cudaMemcpyAsync(di, t->idx, (size_t)t->U * t->m, cudaMemcpyHostToDevice, st);
  if (e == cudaSuccess) e = cudaMemcpyAsync(dm, t->mult, (size_t)t->U * 4, cudaMemcpyHostToDevice, st);
  if (e != cudaSuccess) return cuda_fail(e, "general: table upload");
  *d_idx = di;
  *d_mult = dm;
  return SSHOPM_OK;
}

int general_solve(const GeneralTables* t, int64_t N, const float* d_entries, int S, const float* d_starts, float alpha,
                  float tol, int maxit, float* d_lambda, float* d_x, int32_t* d_iters, uint8_t* d_conv,
                  const sshopm_solve_opts* opts, cudaStream_t st) {
  const int block = 128;
  const int smem = general_smem(t, block, true);
  if (smem > 200 * 1024) return SSHOPM_EUNSUPPORTED;
  const int alpha_mode = opts ? opts->alpha_mode : 0;
  if (alpha_mode < 0 || alpha_mode > 3 || (alpha_mode == 1 && !opts->d_alpha)) return SSHOPM_EINVAL;
  void* tab = nullptr;
  cudaError_t e = cudaMallocAsync(&tab, general_table_bytes(t), st);
  if (e != cudaSuccess) return e == cudaErrorMemoryAllocation ? SSHOPM_ENOMEM : cuda_fail(e, "general: malloc");
  GenParams p;
  int rc = general_upload(t, tab, st, &p.cls_idx, &p.cls_mult);
  if (rc != SSHOPM_OK) { cudaFreeAsync(tab, st); return rc; }
  p.entries = d_entries;
  p.starts = d_starts;
  p.out_lambda = d_lambda;
  p.out_x = d_x;
  p.out_iters = d_iters;
  p.out_conv = d_conv;
  p.total_iters = opts ? opts->d_total_iters : nullptr;
  p.alpha_in = alpha_mode == 1 ? opts->d_alpha : nullptr;
  p.N = N;
  p.m = t->m;
  p.n = t->n;
  p.U = t->U;
  p.S = S;
  p.alpha = alpha;
  p.tol = tol;
  p.alpha_mode = alpha_mode;
  p.maxit = maxit;
  if (smem > 48 * 1024) cudaFuncSetAttribute(sshopm_general_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  const int sms = device_sms();
  long long grid = N < (long long)sms * 16 ? N : (long long)sms * 16;
  sshopm_general_kernel<<<(int)grid, block, smem, st>>>(p);
  e = cudaGetLastError();
  cudaFreeAsync(tab, st);
  if (e != cudaSuccess) return cuda_fail(e, "general: launch");
  return SSHOPM_OK;
}

int general_apply(const GeneralTables* t, int64_t N, const float* d_entries, const float* d_x, float* d_g, float* d_lam,
                  cudaStream_t st) {
  const int block = 128;
  const int smem = general_smem(t, block, false);
  if (smem > 200 * 1024) return SSHOPM_EUNSUPPORTED;
  void* tab = nullptr;
  cudaError_t e = cudaMallocAsync(&tab, general_table_bytes(t), st);
  if (e != cudaSuccess) return e == cudaErrorMemoryAllocation ? SSHOPM_ENOMEM : cuda_fail(e, "general: malloc");
  GenParams p;
  memset(&p, 0, sizeof(p));
  int rc = general_upload(t, tab, st, &p.cls_idx, &p.cls_mult);
  if (rc != SSHOPM_OK) { cudaFreeAsync(tab, st); return rc; }
  p.entries = d_entries;
  p.N = N;
  p.m = t->m;
  p.n = t->n;
  p.U = t->U;
  if (smem > 48 * 1024) cudaFuncSetAttribute(sshopm_general_apply_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  const int sms = device_sms();
  long long grid = (N + block - 1) / block;
  if (grid > (long long)sms * 16) grid = (long long)sms * 16;
  sshopm_general_apply_kernel<<<(int)grid, block, smem, st>>>(p, d_x, d_g, d_lam);
  e = cudaGetLastError();
  cudaFreeAsync(tab, st);
  if (e != cudaSuccess) return cuda_fail(e, "general: apply launch");
  return SSHOPM_OK;
}

}  // namespace sshopm
