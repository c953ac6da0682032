"""C2 dedup kernel timing (median of reps, L2 flushed) and bitwise check against a reference library's
records: python tools/dedup_time.py [reps]; SSHOPM_LIBRARY selects the library."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402
import synthetic as syn  # noqa: E402
import paper_conf_ipps_ballardkp11_b200 as sh  # noqa: E402

reps = int(sys.argv[1]) if len(sys.argv) > 1 else 7
dev = torch.device("cuda:0")
cfg = syn.CONFIGS["C2"]
s = sh.Solver(4, 3)
ent = torch.from_numpy(syn.gen_voxels(4, 3, 0, cfg["N"], 0)).to(dev)
st = torch.from_numpy(syn.gen_starts(128, 3, 0)).to(dev)
raw = s.solve(ent, st, 0.0, 1e-6, 100)
flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)
out = s.dedup(raw[0], raw[1], raw[3], 1e-2, 0.05, 4)
ts = []
for r in range(reps + 2):
    flush.zero_()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    s.dedup(raw[0], raw[1], raw[3], 1e-2, 0.05, 4, out=out)
    e1.record()
    torch.cuda.synchronize()
    if r >= 2:
        ts.append(e0.elapsed_time(e1))
h = [o.cpu().numpy() for o in out]
digest = [int(np.frombuffer(a.tobytes(), np.uint8).astype(np.uint64).sum()) for a in h]
print(json.dumps({"lib": os.path.basename(sh.library_path), "dedup_ms": round(float(np.median(ts)), 4),
                  "min_ms": round(min(ts), 4), "digest": digest}), flush=True)
