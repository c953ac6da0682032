"""One C2 solve_dedup in a given fused mode (for ncu launch lists): python tools/prof_fused.py ws|ring|two"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402
import synthetic as syn  # noqa: E402
import paper_conf_ipps_ballardkp11_b200 as sh  # noqa: E402

mode = sys.argv[1]
dev = torch.device("cuda:0")
cfg = syn.CONFIGS["C2"]
s = sh.Solver(4, 3)
ent = torch.from_numpy(syn.gen_voxels(4, 3, 0, cfg["N"], 0)).to(dev)
st = torch.from_numpy(syn.gen_starts(128, 3, 0)).to(dev)
for _ in range(2):
    if mode == "two":
        r = s.solve(ent, st, 0.0, 1e-6, 100)
        s.dedup(r[0], r[1], r[3], 1e-2, 0.05, 4)
    else:
        s.solve_dedup(ent, st, 0.0, 1e-6, 100, 1e-2, 0.05, 4, fused=(mode == "ring"), warp_specialized=(mode == "ws"))
torch.cuda.synchronize()
