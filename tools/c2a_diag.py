import sys, json, numpy as np, torch
sys.path.insert(0, '.')
import paper_conf_ipps_ballardkp11_b200 as sh, synthetic as syn
from tests import parity as PR
c = syn.CONFIGS["C2a"]; m, n, N, S = c["m"], c["n"], c["N"], c["S"]
dev = torch.device("cuda:0")
ent = syn.gen_voxels(m, n, 0, N, seed=0); st = syn.gen_starts(S, n, seed=0)
s = sh.Solver(m, n)
lam, x, it, cv = s.solve(torch.from_numpy(ent).to(dev), torch.from_numpy(st).to(dev), c["alpha"], c["tol"], c["maxit"])
torch.cuda.synchronize()
idx = np.unique(np.linspace(0, N - 1, 384).astype(np.int64))
sel = torch.from_numpy(idx).to(dev)
gpu = tuple(t.index_select(0, sel).cpu().numpy() for t in (lam, x, it, cv))
rep = PR.solve_parity(ent[idx], st, m, n, c["alpha"], c["tol"], c["maxit"], gpu)
print(json.dumps({k: v for k, v in rep.items() if k != "details"}))
for d in rep["details"][:12]: print(json.dumps(d))
