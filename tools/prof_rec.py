"""Run records-path solve_dedup calls of one config (for ncu captures): python tools/prof_rec.py C2 <reps> [K] [unit]"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402
import synthetic as syn  # noqa: E402
import paper_conf_ipps_ballardkp11_b200 as sh  # noqa: E402

cfg = syn.CONFIGS[sys.argv[1] if len(sys.argv) > 1 else "C2"]
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 3
K = int(sys.argv[3]) if len(sys.argv) > 3 else 0
U = int(sys.argv[4]) if len(sys.argv) > 4 else 0
dev = torch.device("cuda:0")
ent = torch.from_numpy(syn.gen_voxels(cfg["m"], cfg["n"], 0, cfg["N"], 0)).to(dev)
st = torch.from_numpy(syn.gen_starts(cfg["S"], cfg["n"], 0)).to(dev)
s = sh.Solver(cfg["m"], cfg["n"])
d = None
for _ in range(reps):
    _, d = s.solve_dedup(ent, st, cfg["alpha"], cfg["tol"], cfg["maxit"], 1e-2, 0.05, 4, dedup_out=d, records=True,
                         refill_threshold=K, unit_starts=U)
torch.cuda.synchronize()
print("done")
