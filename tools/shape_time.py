"""Solve time of an arbitrary (m, n) on synthetic voxel tensors: python tools/shape_time.py m n N [alpha] [reps]
(SSHOPM_LIBRARY selects a variant build)."""
import json, os, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np, torch
import synthetic as syn
import paper_conf_ipps_ballardkp11_b200 as sh
m, n, N = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3])
alpha = float(sys.argv[4]) if len(sys.argv) > 4 else 0.0
reps = int(sys.argv[5]) if len(sys.argv) > 5 else 5
dev = torch.device("cuda:0")
ent = torch.from_numpy(syn.gen_voxels(m, n, 0, N, 0)).to(dev)
st = torch.from_numpy(syn.gen_starts(128, n, 0)).to(dev)
s = sh.Solver(m, n)
out = s.solve(ent, st, alpha, 1e-6, 100)
ts = []
for r in range(reps + 1):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(); out = s.solve(ent, st, alpha, 1e-6, 100, out=out); e1.record(); torch.cuda.synchronize()
    if r: ts.append(e0.elapsed_time(e1))
print(json.dumps({"lib": os.path.basename(sh.library_path), "m": m, "n": n, "N": N, "ms": round(float(np.median(ts)), 4)}))
