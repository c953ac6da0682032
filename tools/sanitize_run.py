"""Small runs of every solve / dedup path for compute-sanitizer (memcheck, racecheck, synccheck, initcheck):
    compute-sanitizer --tool racecheck python tools/sanitize_run.py <case>
cases: two_pass (C1 tensors x 128 starts, default schedule 1: pack + solve + dedup), lean (schedule 6),
tpl (schedule 2), wt / wt_records (schedule 7 raw / fused + records-only), fused (fuse_dedup = 1: in-kernel ring + list kernel, forced overflow), blocked ((4,10),
V = 6, schedule 5, two tensor buffers per warp), general (schedule 3), classify, run_host, records (records
path, session 4), horner ((6,3) / (8,3) / (4,6) Horner steps and apply, session 4); two_pass at C1 size runs the
small-problem item-chunk instance of schedule 1."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402
import synthetic as syn  # noqa: E402
import paper_conf_ipps_ballardkp11_b200 as sh  # noqa: E402

case = sys.argv[1] if len(sys.argv) > 1 else "two_pass"
dev = torch.device("cuda:0")


def t(a):
    return torch.from_numpy(np.ascontiguousarray(a)).to(dev)


if case in ("two_pass", "legacy", "tpl", "fused", "classify", "lean", "wt", "wt_records"):
    V = 1024 if case != "fused" else 2000
    ent = syn.gen_voxels(4, 3, 0, V, 0)
    if case == "fused":
        ent[::40] = syn.gen_uniform_tensors(4, 3, V // 40, 9)   # slow lanes: ring overflow
    st = syn.gen_starts(128, 3, 0)
    s = sh.Solver(4, 3)
    if case == "fused":
        s.solve_dedup(t(ent), t(st), 0.0, 1e-6, 1000, 1e-2, 0.05, 4, fused=True)
    elif case == "wt_records":
        s.solve_dedup(t(ent), t(st), 0.0, 1e-6, 100, 1e-2, 0.05, 4, records_only=True)
        s.solve_dedup(t(ent), t(st), 0.0, 1e-6, 100, 1e-2, 0.05, 4, schedule=7, fused=True)
    else:
        sched = {"two_pass": 0, "legacy": 1, "lean": 6, "tpl": 2, "classify": 0, "wt": 7}[case]
        lam, x, it, cv = s.solve(t(ent), t(st), 0.0, 1e-6, 100, schedule=sched)
        cnt, cl, cx, mu, rp = s.dedup(lam, x, cv, 1e-2, 0.05, 8)
        if case == "classify":
            s.classify(t(ent), cnt, cl, cx, 1e-3)
elif case == "blocked":
    ent = syn.gen_voxels(4, 10, 0, 6, 5)
    st = syn.gen_starts(32, 10, 4)
    sh.Solver(4, 10).solve(t(ent), t(st), 0.0, 1e-6, 300, schedule=5)
elif case == "general":
    ent = syn.gen_voxels(6, 4, 0, 16, 3)
    st = syn.gen_starts(64, 4, 1)
    sh.Solver(6, 4).solve(t(ent), t(st), 0.5, 1e-6, 200, schedule=3)
elif case == "records":      # records path (fuse_dedup = 4): lane-owned units, 16-byte records, record dedup
    ent = syn.gen_voxels(4, 3, 0, 1024, 0)
    st = syn.gen_starts(128, 3, 0)
    sh.Solver(4, 3).solve_dedup(t(ent), t(st), 0.0, 1e-6, 100, 1e-2, 0.05, 4, records=True, unit_starts=32)
    e6 = syn.gen_voxels(4, 6, 0, 64, 2)                     # two float4 per record (n = 6), S != 128
    s6 = syn.gen_starts(100, 6, 1)
    sh.Solver(4, 6).solve_dedup(t(e6), t(s6), 0.0, 1e-6, 100, 1e-2, 0.05, 4, records=True, unit_starts=7)
elif case == "horner":       # Horner evaluations: (6,3) B-form FFMA2, (8,3) raw divided powers, (4,6) hornerN
    for (m, n, a) in ((6, 3, 0.25), (8, 3, 0.5), (4, 6, 0.0)):
        ent = syn.gen_voxels(m, n, 0, 256, 3)
        st = syn.gen_starts(128, n, 2)
        s = sh.Solver(m, n)
        lam, x, it, cv = s.solve(t(ent), t(st), a, 1e-6, 100)
        s.dedup(lam, x, cv, 1e-2, 0.05, 4)
        s.apply(t(ent), t(syn.gen_starts(256, n, 5)))
elif case == "run_host":
    ent = syn.gen_voxels(4, 3, 0, 3000, 9)
    st = syn.gen_starts(128, 3, 0)
    sh.Solver(4, 3).run_host(ent, st, 0.0, 1e-6, 100, 1e-2, 0.05, 8, raw=True, chunk_tensors=700)
torch.cuda.synchronize()
print("ok", case)
