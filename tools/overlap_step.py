"""C2 step with the dedup of chunk c overlapped with the solve of chunk c+1 (two streams), against the
two-pass step: python tools/overlap_step.py [chunks] [ctas_per_sm].  SSHOPM_DEDUP_WARPS sets the dedup CTA
size so a dedup CTA fits beside the solve CTAs on an SM.  Prints JSON lines (medians of 7, L2 flushed) and
checks the records against the two-pass step bit for bit."""
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
N, S, m, n = cfg["N"], cfg["S"], cfg["m"], cfg["n"]
s = sh.Solver(m, n)
ent = torch.from_numpy(syn.gen_voxels(m, n, 0, N, 0)).to(dev)
st = torch.from_numpy(syn.gen_starts(S, n, 0)).to(dev)
raw = s.solve(ent, st, 0.0, 1e-6, 100)
ref = [t.clone() for t in s.dedup(raw[0], raw[1], raw[3], 1e-2, 0.05, 4)]
dd = [torch.empty_like(t) for t in ref]
flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)
sa = torch.cuda.current_stream()
sb = torch.cuda.Stream()


def two_pass():
    s.solve(ent, st, 0.0, 1e-6, 100, out=raw)
    s.dedup(raw[0], raw[1], raw[3], 1e-2, 0.05, 4, out=dd)


def overlapped(C, cps):
    b = [i * N // C for i in range(C + 1)]
    evs = [torch.cuda.Event() for _ in range(C)]
    for c in range(C):
        v0, v1 = b[c], b[c + 1]
        o = tuple(t[v0:v1] for t in raw)
        s.solve(ent[v0:v1], st, 0.0, 1e-6, 100, out=o, ctas_per_sm=cps, stream=sa)
        evs[c].record(sa)
        with torch.cuda.stream(sb):
            sb.wait_event(evs[c])
            s.dedup(o[0], o[1], o[3], 1e-2, 0.05, 4, out=tuple(t[v0:v1] for t in dd), stream=sb)
    sa.wait_stream(sb)


def timeit(fn, reps=7):
    ts = []
    for r in range(reps + 2):
        flush.zero_()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(sa)
        fn()
        e1.record(sa)
        torch.cuda.synchronize()
        if r >= 2:
            ts.append(e0.elapsed_time(e1))
    return float(np.median(ts))


print(json.dumps({"step": "two_pass", "ms": round(timeit(two_pass), 4),
                  "dedup_warps": os.environ.get("SSHOPM_DEDUP_WARPS", "8")}), flush=True)
for C in [int(v) for v in (sys.argv[1] if len(sys.argv) > 1 else "4,8,16").split(",")]:
    for cps in [int(v) for v in (sys.argv[2] if len(sys.argv) > 2 else "0,3").split(",")]:
        ms = timeit(lambda: overlapped(C, cps))
        same = all(bool(torch.equal(a, b)) for a, b in zip(ref, dd))
        print(json.dumps({"step": "overlapped", "chunks": C, "ctas_per_sm": cps, "ms": round(ms, 4),
                          "records_equal": same, "dedup_warps": os.environ.get("SSHOPM_DEDUP_WARPS", "8")}),
              flush=True)
