// sshopm_wt.cuh — schedule 7: warp-tensor pipeline (included by sshopm_kernels.cuh).
//
// Same per-lane arithmetic as schedules 1/2/6 (sshopm_step; results bitwise
// identical), different work assignment:
//   * a warp works on the S starts of one tensor at a time, with a second
//     tensor opened as soon as the first one's starts are handed out, so lanes
//     never wait for the first tensor's slow starts (two staging slots);
//   * a lane that stops takes the next start of the warp's current tensor:
//     one start load, and a coefficient-row load only when the lane moves to
//     the other tensor (the refill of schedule 1 reloads 8 LDG.128 per item);
//   * per-start results go to the slot's shared-memory staging (two STS per
//     item: (x, lambda) and iters|converged) instead of six scattered global
//     stores; when all S starts of a tensor are done the warp flushes its
//     staging to the raw outputs as coalesced warp stores (MODE 0, 2) and/or
//     clusters it in registers right there (R16 dedup, MODE 1, 2), so the
//     records-only path (MODE 1) never writes or re-reads per-start results.
// P:L321-325 (Sec. V-C): "fit all the data for each thread block in the
// memory on the multiprocessor and minimize the accesses to device memory".
#pragma once

// staging bytes per warp: two slots x S x (record of round4(N+1) floats + one int)
template <int N>
__host__ __device__ constexpr int wt_smem_per_warp(int S) {
  return 2 * S * (((N + 1 + 3) / 4) * 16 + 4);
}

template <int M, int N, int SHIFT, int MODE>
__global__ void __launch_bounds__(256, Shape<M, N>::MINB)
sshopm_solve_wt_kernel(const SolveParams p) {
  constexpr int STEPS = steps_per_trip<M, N>();
  using Sh = Shape<M, N>;
  constexpr int SST4 = round4(N) / 4;
  constexpr int REC4 = (N + 1 + 3) / 4;                 // float4 per staged record: x[0..N), lambda at word N
  constexpr int IDLE = 0x7fffffff;
  constexpr bool EVEN = (M % 2) == 0;

  const int lane = threadIdx.x & 31;
  const int wib = threadIdx.x >> 5;
  const uint32_t ltmask = lanemask_lt();
  const uint32_t FULL = 0xffffffffu;
  const float alpha = (SHIFT == 2) ? -p.alpha : p.alpha;
  const float tol = p.tol;
  const int maxit = p.maxit;
  const int S = p.S;
  const unsigned int NT = (unsigned int)p.n_tensors;

  extern __shared__ float4 wt_smem[];
  float4* rec = wt_smem + (size_t)wib * (2 * S * REC4 + (2 * S + 3) / 4);   // [2][S][REC4]
  int* its = reinterpret_cast<int*>(rec + 2 * S * REC4);                       // [2][S]: iters | converged << 31

  // warp-uniform pipeline state (every lane holds the same values)
  unsigned int T0 = 0xffffffffu, T1 = 0xffffffffu;   // tensor in slot 0 / 1 (none = ~0)
  int rem0 = 0, rem1 = 0;                              // starts of the slot's tensor not yet finished
  int cur = 0, nxt = S;                                // slot handing out starts, next start index
  bool exhausted = false;
  unsigned int pref = 0;                               // next tensor index (claimed one tensor ahead)
  if (lane == 0) pref = atomicAdd(p.counter, 1u);
  uint32_t k_eff = (uint32_t)p.refill_k;

  // per-lane state
  Coefs<M, N> cf;
  float2 xs[Sh::NX];
#pragma unroll
  for (int i = 0; i < Sh::NX; ++i) xs[i] = f2(0.f, 0.f);
  float lamp = 0.f, lam = 0.f;
  int k = IDLE;
  bool stop = true, conv = false;
  int sidx = 0, slot = -1;                             // start index and staging slot of the lane's item
  float la = 0.f, ls = 1.f;
  uint32_t it_sum = 0;

  for (;;) {
    const uint32_t smask = __ballot_sync(FULL, stop);
    const uint32_t cnt = __popc(smask);
    if (cnt >= k_eff) {
      // ---- retire: stopped lanes stage their result (A7) ----
      const bool wr = stop && (k != IDLE);
      if (wr) {
        float4* r = rec + (slot * S + sidx) * REC4;
        float w[4 * REC4];
#pragma unroll
        for (int j = 0; j < 4 * REC4; ++j) w[j] = 0.f;
#pragma unroll
        for (int j = 0; j < N; ++j) w[j] = xget<M, N>(xs, j);
        w[N] = lam;
#pragma unroll
        for (int i = 0; i < REC4; ++i) r[i] = make_float4(w[4 * i], w[4 * i + 1], w[4 * i + 2], w[4 * i + 3]);
        its[slot * S + sidx] = k | (conv ? (int)0x80000000 : 0);
        it_sum += (uint32_t)k;
        k = IDLE;
      }
      const uint32_t dmask = __ballot_sync(FULL, wr);
      if (dmask) {
        const uint32_t d1 = __popc(dmask & __ballot_sync(FULL, slot == 1));
        rem1 -= (int)d1;
        rem0 -= (int)(__popc(dmask) - d1);
        // ---- flush the tensors whose S starts are all done ----
#pragma unroll 1
        for (int b = 0; b < 2; ++b) {
          const unsigned int T = b ? T1 : T0;
          if (T == 0xffffffffu || (b ? rem1 : rem0) != 0) continue;
          __syncwarp();
          const float4* rb = rec + b * S * REC4;
          const int* ib = its + b * S;
          const size_t base = (size_t)T * (size_t)S;
          bool raw = MODE != 1;
          if constexpr (MODE != 0) {                     // R16 clustering straight from the staging (S = 128)
            DedupRegs<N> dr;
            float lm[4], xx[4][N];
            uint32_t cv4 = 0;
#pragma unroll
            for (int c = 0; c < 4; ++c) {
              const int i = 4 * lane + c;
              float w[4 * REC4];
#pragma unroll
              for (int q = 0; q < REC4; ++q) {
                const float4 v = rb[i * REC4 + q];
                w[4 * q] = v.x; w[4 * q + 1] = v.y; w[4 * q + 2] = v.z; w[4 * q + 3] = v.w;
              }
#pragma unroll
              for (int j = 0; j < N; ++j) xx[c][j] = w[j];
              lm[c] = w[N];
              cv4 |= (ib[i] < 0 ? 1u : 0u) << (8 * c);
            }
            dr.lam = make_float4(lm[0], lm[1], lm[2], lm[3]);
#pragma unroll
            for (int q = 0; q < N; ++q) {
              float v4[4];
#pragma unroll
              for (int e = 0; e < 4; ++e) { const int w = 4 * q + e; v4[e] = xx[w / N][w % N]; }
              dr.x[q] = make_float4(v4[0], v4[1], v4[2], v4[3]);
            }
            dr.conv = cv4;
            if (!dedup128_regs<N, EVEN, false>(p.dd, (long long)T, lane, dr, nullptr)) {
              raw = true;                                // > 32 clusters: raw outputs + list kernel
              if (MODE == 1 && lane == 0) p.ovf_list[atomicAdd(p.ovf_count, 1u)] = T;
            }
          }
          if (raw) {                                     // coalesced: lane l writes items l, l + 32, ...
            for (int i = lane; i < S; i += 32) {
              const float4* r = rb + i * REC4;
              float w[4 * REC4];
#pragma unroll
              for (int q = 0; q < REC4; ++q) {
                const float4 v = r[q];
                w[4 * q] = v.x; w[4 * q + 1] = v.y; w[4 * q + 2] = v.z; w[4 * q + 3] = v.w;
              }
              const int iv = ib[i];
              p.out_lambda[base + i] = w[N];
#pragma unroll
              for (int j = 0; j < N; ++j) p.out_x[(base + i) * N + j] = w[j];
              p.out_iters[base + i] = iv & 0x7fffffff;
              p.out_conv[base + i] = iv < 0 ? 1 : 0;
            }
          }
          __syncwarp();
          if (b) T1 = 0xffffffffu; else T0 = 0xffffffffu;
        }
      }
      // ---- open the next tensor when the current one's starts are all handed out ----
      if (nxt >= S && !exhausted) {
        const int o = cur ^ 1;
        if ((o ? T1 : T0) == 0xffffffffu) {
          const unsigned int t = __shfl_sync(FULL, pref, 0);
          if (t < NT) {
            if (o) { T1 = t; rem1 = S; } else { T0 = t; rem0 = S; }
            cur = o;
            nxt = 0;
            if (lane == 0) pref = atomicAdd(p.counter, 1u);
          } else {
            exhausted = true;
            k_eff = 32u;
          }
        }
      }
      // ---- hand the current tensor's next starts to the free lanes ----
      const uint32_t fmask = __ballot_sync(FULL, k == IDLE);
      const int avail = (nxt < S) ? S - nxt : 0;
      const int rank = __popc(fmask & ltmask);
      const bool ok = (k == IDLE) && rank < avail;
      const unsigned int Tc = cur ? T1 : T0;
      const bool sw = ok && (slot != cur);
      if (__ballot_sync(FULL, sw)) {                     // lanes moving to the current tensor load its row
        if (sw) {
          cf.load(p.packed + (size_t)Tc * (Sh::PW / 4));
          if constexpr (SHIFT == 3) {
            const float at = __ldg(p.alpha_t + Tc);
            ls = at >= 0.f ? 1.f : -1.f;                 // Fig. 1 lines 2-5 (R5: alpha = 0 -> "+")
            la = fabsf(at);
          }
        }
      }
      if (ok) {
        sidx = nxt + rank;
        slot = cur;
        float v[4 * SST4];
#pragma unroll
        for (int i = 0; i < SST4; ++i) {
          const float4 q4 = ldg4(p.starts_n + sidx * SST4 + i);
          v[4 * i] = q4.x; v[4 * i + 1] = q4.y; v[4 * i + 2] = q4.z; v[4 * i + 3] = q4.w;
        }
#pragma unroll
        for (int i = 0; i < Sh::NX; ++i) xs[i] = f2(v[2 * i], v[2 * i + 1]);   // starts_n is in slot order
        lamp = __int_as_float(0x7fffffff);               // NaN: the first test never fires (reading R2)
        k = 0;
      }
      const int taken = (int)__popc(fmask) < avail ? (int)__popc(fmask) : avail;
      nxt += taken;
      if (exhausted && __ballot_sync(FULL, k != IDLE) == 0u && T0 == 0xffffffffu && T1 == 0xffffffffu) break;
    }
#pragma unroll
    for (int rep = 0; rep < STEPS; ++rep)
      sshopm_step<M, N, SHIFT, true>(cf, xs, lam, lamp, k, conv, stop, true, alpha, la, ls, tol, maxit);
  }

  if (p.total_iters) {
    unsigned long long ws = it_sum;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) ws += __shfl_xor_sync(0xffffffffu, ws, o);
    if (lane == 0) atomicAdd(p.total_iters, ws);
  }
}
