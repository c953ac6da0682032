import time, torch, sys
sys.path.insert(0, '.')
import paper_conf_ipps_ballardkp11_b200 as sh, synthetic as syn
s = sh.Solver(4, 3)
e = torch.from_numpy(syn.gen_voxels(4, 3, 0, 1024, 0)).cuda(); st = torch.from_numpy(syn.gen_starts(128, 3, 0)).cuda()
out = s.solve(e, st); dd = s.dedup(out[0], out[1], out[3]); torch.cuda.synchronize()
for name, fn in [("solve", lambda: s.solve(e, st, out=out)), ("dedup", lambda: s.dedup(out[0], out[1], out[3], out=dd))]:
    torch.cuda.synchronize(); t = time.perf_counter()
    for _ in range(200): fn()
    t1 = time.perf_counter(); torch.cuda.synchronize()
    print(name, "host us/call", round((t1 - t) / 200 * 1e6, 1))
