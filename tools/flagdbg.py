import sys, json, numpy as np, torch
sys.path.insert(0, '.')
import paper_conf_ipps_ballardkp11_b200 as sh, synthetic as syn
from tests import parity as PR
dev = torch.device('cuda:0')
out = {}
cases = [("C1", 4,3,None,0.0), ("m4a-", 4,3,128,-0.5), ("m3n2", 3,2,64,0.5), ("m5n3",5,3,32,0.5)]
for name,m,n,V,alpha in cases:
    if name == "C1":
        ent = syn.gen_voxels(m,n,0,1024,0); st = syn.gen_starts(128,n,0)
    else:
        ent = syn.gen_voxels(m, n, 12345, V, 2) if m % 2 == 0 else syn.gen_uniform_tensors(m, n, V, 2)
        st = syn.gen_starts(128, n, 5)
    s = sh.Solver(m,n)
    r = s.solve(torch.from_numpy(ent).to(dev), torch.from_numpy(st).to(dev), alpha, 1e-6, 100)
    gpu = tuple(t.cpu().numpy() for t in r)
    np.savez(f'gpurun_out/dbg_{name}.npz', lam=gpu[0], x=gpu[1], it=gpu[2], cv=gpu[3])
    rep = PR.solve_parity(ent, st, m, n, alpha, 1e-6, 100, gpu)
    out[name] = rep
    print(name, json.dumps(rep, indent=None)[:3000])
json.dump(out, open('gpurun_out/flagdbg.json','w'), indent=1)
