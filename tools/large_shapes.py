"""Table-driven kernels on larger (m, n): solve time of the item-per-lane
general kernel (schedule 3), the block-per-tensor one (4) and the blocked warp-per-tensor one (5).

    python tools/large_shapes.py [--tensors 16384] [--starts 128]

One JSON line per (shape, schedule): ms per solve (CUDA events, median of 3 after a warm-up), mean
iterations, and algorithmic GFLOP/s = (2*T1 + monomials + 5n) per evaluation."""
import argparse
import json
import os
import sys
from math import comb

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ipps_ballardkp11_b200 as sh  # noqa: E402
import synthetic as syn  # noqa: E402

SHAPES = [((4, 3), 0.0), ((5, 4), 1.0), ((6, 4), 0.5), ((3, 6), 1.0), ((4, 5), 0.0), ((7, 3), 1.0),
          ((4, 8), 0.0), ((5, 6), 1.0), ((6, 6), 0.5), ((4, 10), 0.0), ((3, 16), 1.0)]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--tensors", type=int, default=16384)
    ap.add_argument("--starts", type=int, default=128)
    ap.add_argument("--schedules", default="3,4,5")
    ap.add_argument("--shapes", default="", help="m,n;m,n;... (default: the built-in list)")
    a = ap.parse_args()
    dev = torch.device("cuda:0")
    shapes = SHAPES
    if a.shapes:
        want = {tuple(int(v) for v in t.split(",")) for t in a.shapes.split(";")}
        shapes = [sa for sa in SHAPES if sa[0] in want]
    for (m, n), alpha in shapes:
        ent_h = syn.gen_voxels(m, n, 0, a.tensors, 0) if m % 2 == 0 else syn.gen_uniform_tensors(m, n, a.tensors, 0)
        ent = torch.from_numpy(ent_h).to(dev)
        st = torch.from_numpy(syn.gen_starts(a.starts, n, 0)).to(dev)
        s = sh.Solver(m, n)
        Q, L = comb(m + n - 2, m - 1), comb(m - 1 + n, m - 1) - 1
        f_eval = 2 * n * Q + (L - n) + 5 * n
        for sched in [int(v) for v in a.schedules.split(",")]:
            ti = torch.zeros(1, dtype=torch.int64, device=dev)
            try:
                s.solve(ent, st, alpha, 1e-6, 100, schedule=sched, total_iters=ti)
            except Exception as e:  # noqa: BLE001  (unsupported combination: report and go on)
                print(json.dumps({"m": m, "n": n, "schedule": sched, "error": str(e)[:120]}), flush=True)
                continue
            torch.cuda.synchronize()
            ts = []
            for _ in range(3):
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                ti.zero_()
                e0.record()
                lam, x, it, cv = s.solve(ent, st, alpha, 1e-6, 100, schedule=sched, total_iters=ti)
                e1.record()
                torch.cuda.synchronize()
                ts.append(e0.elapsed_time(e1))
            ms = float(np.median(ts))
            iters = int(ti.item())
            evals = iters + a.tensors * a.starts
            print(json.dumps({"m": m, "n": n, "U": comb(m + n - 1, m), "alpha": alpha, "schedule": sched,
                              "tensors": a.tensors, "starts": a.starts, "ms": round(ms, 3),
                              "mean_iters": iters / (a.tensors * a.starts), "converged": float(cv.float().mean()),
                              "alg_gflops": round(f_eval * evals / ms / 1e6, 1)}), flush=True)


if __name__ == "__main__":
    main()
