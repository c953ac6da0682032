"""Solve a full config on the GPU and save the sampled tensors' outputs (for CPU-side analysis)."""
import sys, numpy as np, torch
sys.path.insert(0, '.')
import paper_conf_ipps_ballardkp11_b200 as sh, synthetic as syn
name, k = sys.argv[1], int(sys.argv[2])
c = syn.CONFIGS[name]
ent = syn.gen_voxels(c['m'], c['n'], 0, c['N'], 0); st = syn.gen_starts(c['S'], c['n'], 0)
s = sh.Solver(c['m'], c['n'])
out = s.solve(torch.from_numpy(ent).cuda(), torch.from_numpy(st).cuda(), c['alpha'], c['tol'], c['maxit'])
idx = np.unique(np.linspace(0, c['N'] - 1, k).astype(np.int64))
sel = torch.from_numpy(idx).cuda()
lam, x, it, cv = (t.index_select(0, sel).cpu().numpy() for t in out)
np.savez(f'gpurun_out/sample_{name}.npz', idx=idx, lam=lam, x=x, it=it, cv=cv)
