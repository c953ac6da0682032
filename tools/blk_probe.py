"""Blocked-kernel timing probe: every repetition's time for a few (m, n, N)."""
import sys, os, json
import numpy as np
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ipps_ballardkp11_b200 as sh
import synthetic as syn

dev = torch.device("cuda:0")
for (m, n), alpha in [((3, 6), 1.0), ((3, 4), 1.0), ((5, 4), 1.0)]:
    s = sh.Solver(m, n)
    for N in [16384, 32768, 65536]:
        ent = torch.from_numpy(syn.gen_uniform_tensors(m, n, N, 0)).to(dev)
        st = torch.from_numpy(syn.gen_starts(128, n, 0)).to(dev)
        ts = []
        for r in range(5):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(); s.solve(ent, st, alpha, 1e-6, 100, schedule=5); e1.record(); torch.cuda.synchronize()
            ts.append(round(e0.elapsed_time(e1), 2))
        print(json.dumps({"m": m, "n": n, "N": N, "ms": ts}), flush=True)
