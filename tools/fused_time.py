"""C2 step timings: two-pass (solve + dedup), fused solve_dedup (schedule-1 ring), records-only (schedule 7)."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402
import synthetic as syn  # noqa: E402
import paper_conf_ipps_ballardkp11_b200 as sh  # noqa: E402

dev = torch.device("cuda:0")
cfg = syn.CONFIGS["C2"]
m, n, N, S = cfg["m"], cfg["n"], cfg["N"], cfg["S"]
s = sh.Solver(m, n)
ent = torch.from_numpy(syn.gen_voxels(m, n, 0, N, 0)).to(dev)
st = torch.from_numpy(syn.gen_starts(S, n, 0)).to(dev)
flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)
raw = s.solve(ent, st, 0.0, 1e-6, 100)
dd = s.dedup(raw[0], raw[1], raw[3], 1e-2, 0.05, 4)


def timeit(fn, reps=5):
    ts = []
    for r in range(reps + 2):
        flush.zero_()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        fn()
        e1.record()
        torch.cuda.synchronize()
        if r >= 2:
            ts.append(e0.elapsed_time(e1))
    return float(np.median(ts))


lib = os.path.basename(sh.library_path)
# correctness first: fused_ws == two-pass bit for bit (raw and records), incl. slow lanes (ring overflow)
for V, maxit in [(3000, 100), (2000, 3000), (50000, 100)]:
    e = torch.from_numpy(syn.gen_voxels(m, n, 0, V, 4)).to(dev)
    if maxit > 1000:
        e[::40] = torch.from_numpy(syn.gen_uniform_tensors(m, n, V // 40, 9)).to(dev)
    ra, da = s.solve_dedup(e, st, 0.0, 1e-6, maxit, 1e-2, 0.05, 4)
    rb, db = s.solve_dedup(e, st, 0.0, 1e-6, maxit, 1e-2, 0.05, 4, warp_specialized=True)
    torch.cuda.synchronize()
    print(json.dumps({"V": V, "maxit": maxit, "ws_equal": [bool(torch.equal(a, b)) for a, b in zip(ra + da, rb + db)]}), flush=True)
for name, fn in [("two_pass", lambda: (s.solve(ent, st, 0.0, 1e-6, 100, out=raw), s.dedup(raw[0], raw[1], raw[3], 1e-2, 0.05, 4, out=dd))),
                 ("fused_ring", lambda: s.solve_dedup(ent, st, 0.0, 1e-6, 100, 1e-2, 0.05, 4, out=raw, dedup_out=dd, fused=True)),
                 ("fused_ws", lambda: s.solve_dedup(ent, st, 0.0, 1e-6, 100, 1e-2, 0.05, 4, out=raw, dedup_out=dd, warp_specialized=True)),
                 ("records_only", lambda: s.solve_dedup(ent, st, 0.0, 1e-6, 100, 1e-2, 0.05, 4, out=raw, dedup_out=dd, records_only=True))]:
    print(json.dumps({"lib": lib, "step": name, "ms": round(timeit(fn), 4)}), flush=True)
