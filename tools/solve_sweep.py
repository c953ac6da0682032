"""Solve-kernel sweep on one GPU: time sshopm_solve over a config for a list of
(schedule, refill K, chunk) settings and library builds, check that every
setting's outputs are bitwise equal to the first one's, print JSON lines.

    python tools/solve_sweep.py --config C2 --sets "1:0:0,1:4:0,1:6:0,6:8:0" [--libs a.so,b.so] [--reps 5]

Each set is schedule:refill_K:chunk_tensors (0 = library default).  --libs
loads variant builds (SSHOPM_LIBRARY, one subprocess per build); the product
library is the default.  Time = CUDA events around the solve (pack + solve
kernels) on the current stream, L2 flushed before each rep, median of reps.
"""
import argparse
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def run_one(args):
    import numpy as np
    import torch
    import synthetic as syn
    import paper_conf_ipps_ballardkp11_b200 as sh

    cfg = dict(syn.CONFIGS[args.config])
    N = args.voxels or cfg["N"]
    m, n, S = cfg["m"], cfg["n"], cfg["S"]
    dev = torch.device("cuda:0")
    ent = torch.from_numpy(syn.gen_voxels(m, n, 0, N, seed=0)).to(dev)
    st = torch.from_numpy(syn.gen_starts(S, n, seed=0)).to(dev)
    solver = sh.Solver(m, n)
    flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)
    ref = None
    tot = torch.zeros(1, dtype=torch.int64, device=dev)
    for spec in args.sets.split(","):
        sched, k, chunk = (int(v) for v in spec.split(":"))
        out = None
        times = []
        for rep in range(args.reps + 2):
            flush.zero_()
            if rep == 0 or not args.no_total:
                tot.zero_()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            count = rep == 0 or not args.no_total       # --no-total: time without the iteration counter
            out = solver.solve(ent, st, alpha=cfg["alpha"], tol=cfg["tol"], maxit=cfg["maxit"], out=out,
                               refill_threshold=k, schedule=sched, chunk_tensors=chunk,
                               total_iters=tot if count else None)
            e1.record()
            torch.cuda.synchronize()
            if rep >= 2:
                times.append(e0.elapsed_time(e1))
        ms = float(np.median(times))
        its = int(tot.item())                            # from rep 0 (every rep when counting)
        F = solver.exec_flops_per_iter
        if cfg["alpha"] == 0.0:
            F -= 2 * n                       # alpha = 0: no shift FMAs (bench.py's count)
        fe = (F - 2 * n if cfg["alpha"] != 0.0 else F) - (2 * n - 1) - n   # lambda_0 = A x_0^m per lane
        flops = F * its + fe * N * S
        frac = flops / (ms * 1e-3) / (148 * 128 * 2 * 1.965e9)
        same = None
        if ref is None:
            ref = [o.clone() for o in out]
        else:
            same = all(bool(torch.equal(a, b)) for a, b in zip(ref, out))
        print(json.dumps({"lib": os.path.basename(sh.library_path), "config": args.config, "N": N, "schedule": sched,
                          "refill": k, "chunk": chunk, "ms": round(ms, 4), "ms_min": round(min(times), 4),
                          "iters": its, "frac_alg": round(frac, 4), "bitwise_equal_first": same}), flush=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C2")
    ap.add_argument("--voxels", type=int, default=0)
    ap.add_argument("--sets", default="1:0:0")
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--libs", default="")
    ap.add_argument("--no-total", action="store_true")
    a = ap.parse_args()
    if a.libs and "SSHOPM_LIBRARY" not in os.environ:
        for lib in a.libs.split(","):
            env = dict(os.environ, SSHOPM_LIBRARY=os.path.abspath(lib))
            cmd = [sys.executable, __file__, "--config", a.config, "--voxels", str(a.voxels), "--sets", a.sets,
                   "--reps", str(a.reps)] + (["--no-total"] if a.no_total else [])
            subprocess.run(cmd, env=env, check=False)
        return
    run_one(a)


if __name__ == "__main__":
    main()
