"""Per-call wall times of run_host at C2 (pinned host buffers) — the distribution behind bench.py's e2e."""
import os, sys, time
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np, torch
import synthetic as syn
import paper_conf_ipps_ballardkp11_b200 as sh
N = int(os.environ.get("N", 1 << 20)); chunk = int(os.environ.get("CHUNK", 65536))
ent = torch.from_numpy(syn.gen_voxels(4, 3, 0, N, 0)).pin_memory()
st = torch.from_numpy(syn.gen_starts(128, 3, 0)).pin_memory()
s = sh.Solver(4, 3)
outs = {"count": torch.empty(N, dtype=torch.int32).pin_memory(), "lambda": torch.empty((N, 4)).pin_memory(),
        "x": torch.empty((N, 4, 3)).pin_memory(), "mult": torch.empty((N, 4), dtype=torch.int32).pin_memory()}
ts = []
for i in range(25):
    t0 = time.perf_counter()
    s.run_host(ent, st, 0.0, 1e-6, 100, 1e-2, 0.05, 4, chunk_tensors=chunk, out=outs)
    ts.append((time.perf_counter() - t0) * 1e3)
ts = np.array(ts[3:])
print("chunk", chunk, "median %.3f min %.3f max %.3f mean %.3f" % (np.median(ts), ts.min(), ts.max(), ts.mean()))
print(" ".join("%.2f" % t for t in ts))
