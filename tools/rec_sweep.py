"""Records path (sshopm_solve_dedup fuse_dedup = 4, schedule 8) vs the two-pass step (solve + dedup) on one GPU:
dedup outputs compared bit for bit, step times (CUDA events, L2 flushed, median of reps) and per-kernel times
(torch.profiler / CUPTI) for each (refill K, unit) setting.

    python tools/rec_sweep.py --config C2 --sets "4:32,2:32,4:16,6:32" [--reps 7]
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C2")
    ap.add_argument("--voxels", type=int, default=0)
    ap.add_argument("--sets", default="4:32")
    ap.add_argument("--reps", type=int, default=7)
    a = ap.parse_args()
    import numpy as np
    import torch
    import synthetic as syn
    import paper_conf_ipps_ballardkp11_b200 as sh
    cfg = dict(syn.CONFIGS[a.config])
    N = a.voxels or cfg["N"]
    m, n, S = cfg["m"], cfg["n"], cfg["S"]
    dev = torch.device("cuda:0")
    ent = torch.from_numpy(syn.gen_voxels(m, n, 0, N, seed=0)).to(dev)
    st = torch.from_numpy(syn.gen_starts(S, n, seed=0)).to(dev)
    solver = sh.Solver(m, n)
    flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)
    kw = dict(alpha=cfg["alpha"], tol=cfg["tol"], maxit=cfg["maxit"], lam_tol=1e-2, ang_tol=0.05, kmax=4)
    tot = torch.zeros(1, dtype=torch.int64, device=dev)

    def timed(fn):
        ts = []
        for r in range(a.reps + 2):
            flush.zero_()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(); fn(); e1.record(); torch.cuda.synchronize()
            if r >= 2:
                ts.append(e0.elapsed_time(e1))
        return float(np.median(ts))

    def kernels(fn):
        from torch.profiler import profile, ProfilerActivity
        fn(); torch.cuda.synchronize()
        with profile(activities=[ProfilerActivity.CUDA]) as prof:
            fn(); torch.cuda.synchronize()
        out = {}
        for ev in prof.key_averages():
            if ev.device_type.name == "CUDA" and "sshopm" in ev.key:
                k = ev.key.split("<")[0].replace("void sshopm::", "")
                out[k] = round(out.get(k, 0.0) + ev.device_time_total / 1000.0, 4)
        return out

    raw = None
    ded = None

    def two_pass():
        nonlocal raw, ded
        raw = solver.solve(ent, st, alpha=cfg["alpha"], tol=cfg["tol"], maxit=cfg["maxit"], out=raw)
        ded = solver.dedup(raw[0], raw[1], raw[3], lam_tol=1e-2, ang_tol=0.05, kmax=4, out=ded)

    tot.zero_()
    raw = solver.solve(ent, st, alpha=cfg["alpha"], tol=cfg["tol"], maxit=cfg["maxit"], total_iters=tot)
    torch.cuda.synchronize()
    its = int(tot.item())
    ms2 = timed(two_pass)
    ref = [t.clone() for t in ded]
    k2 = kernels(two_pass)
    F = solver.exec_flops_per_iter - (2 * n if cfg["alpha"] == 0.0 else 0)
    fe = (F - 2 * n if cfg["alpha"] != 0.0 else F) - (2 * n - 1) - n
    flops = F * its + fe * N * S
    peak = 148 * 128 * 2 * 1.965e9

    def frac(ms):
        return round(flops / (ms * 1e-3) / peak, 4)

    ks = [v for k, v in k2.items() if "solve_kernel" in k]
    print(json.dumps({"config": a.config, "N": N, "path": "two_pass", "ms_step": round(ms2, 4), "kernels_ms": k2,
                      "solve_frac": frac(ks[0]) if ks else None}), flush=True)
    dout = None
    for spec in a.sets.split(","):
        K, U = (int(v) for v in spec.split(":"))

        def rec():
            nonlocal dout
            _, dout = solver.solve_dedup(ent, st, **kw, dedup_out=dout, records=True, refill_threshold=K, unit_starts=U)

        ms = timed(rec)
        same = all(bool(torch.equal(x, y)) for x, y in zip(ref, dout))
        tot.zero_()
        _, d2 = solver.solve_dedup(ent, st, **kw, records=True, refill_threshold=K, unit_starts=U, total_iters=tot)
        torch.cuda.synchronize()
        kr = kernels(rec)
        ksr = [v for k, v in kr.items() if "rec_kernel" in k]
        print(json.dumps({"config": a.config, "N": N, "path": "records", "K": K, "unit": U, "ms_step": round(ms, 4),
                          "kernels_ms": kr, "solve_frac": frac(ksr[0]) if ksr else None,
                          "dedup_bitwise_equal_two_pass": same, "iters_equal": int(tot.item()) == its}), flush=True)


if __name__ == "__main__":
    main()
