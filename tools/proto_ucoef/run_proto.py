"""Prototype check: constant-bank (uniform-operand) warp-per-tensor (4,3) solve vs the library's schedule 1.
Bitwise comparison of all four outputs, timing (median of reps), sweeps over nmod / K / park."""
import ctypes, json, os, sys, time
import numpy as np
import torch
HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(os.path.dirname(HERE))
sys.path.insert(0, ROOT)
import synthetic as syn
import paper_conf_ipps_ballardkp11_b200 as sh

N = int(os.environ.get("UC_N", 1 << 20)); S = 128
dev = torch.device("cuda:0")
ent = torch.from_numpy(syn.gen_voxels(4, 3, 0, N, seed=0)).to(dev)
st = torch.from_numpy(syn.gen_starts(S, 3, seed=0)).to(dev)
solver = sh.Solver(4, 3)
tot = torch.zeros(1, dtype=torch.int64, device=dev)
ref = solver.solve(ent, st, alpha=0.0, tol=1e-6, maxit=100, total_iters=tot)
torch.cuda.synchronize()
its = int(tot.item())
F = solver.exec_flops_per_iter - 6
fe = F - 5 - 3
flops = F * its + fe * N * S
def frac(ms): return flops / (ms * 1e-3) / (148 * 128 * 2 * 1.965e9)

def timeit(fn, reps=7):
    ts = []
    for r in range(reps + 2):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(); fn(); e1.record(); torch.cuda.synchronize()
        if r >= 2: ts.append(e0.elapsed_time(e1))
    return float(np.median(ts))

out = [torch.empty_like(o) for o in ref]
ms_ref = timeit(lambda: solver.solve(ent, st, alpha=0.0, tol=1e-6, maxit=100, out=out))
print(json.dumps({"impl": "schedule1", "N": N, "ms": round(ms_ref, 4), "frac": round(frac(ms_ref), 4), "iters": its}), flush=True)

L = ctypes.CDLL(os.path.join(HERE, "uc_host.so"))
P, I, I64, F32 = ctypes.c_void_p, ctypes.c_int, ctypes.c_int64, ctypes.c_float
L.uc_init.argtypes = [ctypes.c_char_p, I]
L.uc_ws_bytes.restype = ctypes.c_size_t; L.uc_ws_bytes.argtypes = [I64, I]
args_t = [I64, P, I, P, F32, I, I, I, P, P, P, P, P, I, P]
L.uc_solve.argtypes = args_t; L.uc_wide.argtypes = [I64, P, I, P, F32, I, I, I, P, P, P, P, P, P]; L.uc_wide_replay.argtypes = [P]; L.uc_capture.argtypes = args_t; L.uc_replay.argtypes = [P]
NMOD = int(os.environ.get("UC_NMOD", 16))
rc = L.uc_init(os.path.join(HERE, "uc_kern.cubin").encode(), NMOD)
assert rc == 0, rc
ws = torch.empty(L.uc_ws_bytes(N, S), dtype=torch.uint8, device=dev)
ts = torch.cuda.Stream(); torch.cuda.set_stream(ts); stream = ts.cuda_stream

def call(fn, nmod, K, park):
    o = [torch.full_like(r, 0) for r in ref]
    def f():
        r = fn(N, ent.data_ptr(), S, st.data_ptr(), 1e-6, 100, K, park, *(t.data_ptr() for t in o), ws.data_ptr(), nmod, stream)
        assert r == 0, r
    return o, f

if os.environ.get("UC_WIDE"):
    for spec in os.environ["UC_WIDE"].split(","):
        K, park = (int(v) for v in spec.split(":"))
        o = [torch.full_like(x, 0) for x in ref]
        t0 = time.time()
        r = L.uc_wide(N, ent.data_ptr(), S, st.data_ptr(), 1e-6, 100, K, park, *(t.data_ptr() for t in o), ws.data_ptr(), stream)
        assert r == 0, r
        tb = time.time() - t0
        L.uc_wide_replay(stream); torch.cuda.synchronize()
        eq = [bool(torch.equal(a, b)) for a, b in zip(ref, o)]
        ms = timeit(lambda: L.uc_wide_replay(stream))
        print(json.dumps({"impl": "ucoef_wide_graph", "K": K, "park": park, "bitwise": eq, "build_s": round(tb, 2),
                          "ms": round(ms, 4), "frac": round(frac(ms), 4)}), flush=True)
if os.environ.get("UC_BREAKDOWN"):
    for spec in os.environ["UC_BREAKDOWN"].split(","):
        nmod, K, park = (int(v) for v in spec.split(":"))
        o, f = call(L.uc_solve, nmod, K, park)
        res = {}
        for ph in ("3", "1", "2", "4"):
            os.environ["UC_PHASES"] = "3"; f(); torch.cuda.synchronize()
            os.environ["UC_PHASES"] = ph
            res["ms_phase" + ph] = round(timeit(f), 4)
        os.environ["UC_PHASES"] = "3"
        print(json.dumps({"impl": "ucoef_breakdown", "nmod": nmod, "K": K, "park": park, **res}), flush=True)
for spec in os.environ.get("UC_SETS", "16:1:8,16:4:8,16:1:4,16:1:0,8:1:8,32:1:8").split(","):
    if spec == "none": continue
    nmod, K, park = (int(v) for v in spec.split(":"))
    if nmod > NMOD: continue
    o, f = call(L.uc_solve, nmod, K, park)
    f(); torch.cuda.synchronize()
    eq = [bool(torch.equal(a, b)) for a, b in zip(ref, o)]
    nbad = int((ref[0] != o[0]).sum())
    parked = int(ws[:4].view(torch.int32).item())
    ms = timeit(f)
    o2, _ = call(L.uc_capture, nmod, K, park)
    r = L.uc_capture(N, ent.data_ptr(), S, st.data_ptr(), 1e-6, 100, K, park, *(t.data_ptr() for t in o2), ws.data_ptr(), nmod, stream)
    assert r == 0, r
    msg = timeit(lambda: L.uc_replay(stream))
    eq2 = [bool(torch.equal(a, b)) for a, b in zip(ref, o2)]
    print(json.dumps({"impl": "ucoef", "nmod": nmod, "K": K, "park": park, "bitwise": eq, "bitwise_graph": eq2,
                      "lam_mismatch": nbad, "parked": parked, "ms": round(ms, 4), "frac": round(frac(ms), 4),
                      "ms_graph": round(msg, 4), "frac_graph": round(frac(msg), 4)}), flush=True)
