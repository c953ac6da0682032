"""Schedule 7 (warp-tensor pipeline) quick check on a GPU: bitwise equality with schedule 1 (raw outputs),
records equality with the two-pass path (MODE 2 fused, MODE 1 records-only), then C2 timings."""
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
m, n = 4, 3
s = sh.Solver(m, n)
for V, S, maxit in [(3000, 128, 100), (777, 100, 100), (50, 300, 100), (5, 7, 100), (2000, 128, 3000)]:
    ent = syn.gen_voxels(m, n, 0, V, 4)
    if maxit > 1000:
        ent[::40] = syn.gen_uniform_tensors(m, n, V // 40, 9)
    st = syn.gen_starts(S, n, 0)
    e, t = torch.from_numpy(ent).to(dev), torch.from_numpy(st).to(dev)
    a = [u.cpu().numpy() for u in s.solve(e, t, 0.0, 1e-6, maxit, schedule=1)]
    b = [u.cpu().numpy() for u in s.solve(e, t, 0.0, 1e-6, maxit, schedule=7)]
    eq = [bool(np.array_equal(u, v)) for u, v in zip(a, b)]
    ra, da = s.solve_dedup(e, t, 0.0, 1e-6, maxit, 1e-2, 0.05, 4, schedule=1)
    rb, db = s.solve_dedup(e, t, 0.0, 1e-6, maxit, 1e-2, 0.05, 4, schedule=7, fused=True)
    rc, dc = s.solve_dedup(e, t, 0.0, 1e-6, maxit, 1e-2, 0.05, 4, records_only=True)
    torch.cuda.synchronize()
    eq2 = [bool(torch.equal(u, v)) for u, v in zip(da, db)] + [bool(torch.equal(u, v)) for u, v in zip(ra, rb)]
    eq3 = [bool(torch.equal(u, v)) for u, v in zip(da, dc)]
    print(json.dumps({"V": V, "S": S, "maxit": maxit, "raw_equal": eq, "mode2_equal": eq2, "mode1_records_equal": eq3}),
          flush=True)

cfg = syn.CONFIGS["C2"]
N, S = cfg["N"], cfg["S"]
ent = torch.from_numpy(syn.gen_voxels(m, n, 0, N, 0)).to(dev)
st = torch.from_numpy(syn.gen_starts(S, n, 0)).to(dev)
flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)
out = None
dd = None


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


for sched, k in [(1, 8), (7, 8), (7, 6), (7, 4), (7, 12)]:
    ms = timeit(lambda: s.solve(ent, st, 0.0, 1e-6, 100, out=out, schedule=sched, refill_threshold=k))
    print(json.dumps({"solve_schedule": sched, "refill": k, "ms": round(ms, 4)}), flush=True)
raw = s.solve(ent, st, 0.0, 1e-6, 100)
ms = timeit(lambda: (s.solve(ent, st, 0.0, 1e-6, 100, out=raw, schedule=1), s.dedup(raw[0], raw[1], raw[3], 1e-2, 0.05, 4)))
print(json.dumps({"step": "solve+dedup two-pass", "ms": round(ms, 4)}), flush=True)
for k in (8, 6):
    ms = timeit(lambda: s.solve_dedup(ent, st, 0.0, 1e-6, 100, 1e-2, 0.05, 4, out=raw, records_only=True, refill_threshold=k))
    print(json.dumps({"step": "records-only schedule 7", "refill": k, "ms": round(ms, 4)}), flush=True)
