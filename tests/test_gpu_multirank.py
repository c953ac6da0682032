"""The bench's multi-rank path (tensor-range shards + one gather, max-over-ranks timing) on one GPU:
two torchrun ranks share cuda:0 through the gloo backend (NCCL would refuse a duplicated GPU)."""
import json
import os
import socket
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def test_bench_two_ranks_gloo():
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
           "--master-addr", "127.0.0.1", "--master-port", str(_port()), os.path.join(ROOT, "bench.py"),
           "--gpus", "2", "--steps", "3", "--warmup", "3", "--backend", "gloo", "--no-cpu", "--voxels", "65536"]
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=600, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1                                   # rank 0 prints one line
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["scaling"] == "weak"
    assert d["config"]["tensors_total"] == 2 * 65536
    assert d["value"] > 0 and d["e2e"]["h2d_bytes_per_step"] > 0


def test_bench_self_launch_two_ranks_gloo():
    """`python bench.py --gpus 2` with no torchrun wrapper starts the two ranks itself (VERDICT r1 Next 2)."""
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    env = {k: v for k, v in os.environ.items() if k not in ("WORLD_SIZE", "RANK", "LOCAL_RANK")}
    cmd = [sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "2", "--steps", "3", "--warmup", "3",
           "--backend", "gloo", "--no-cpu", "--no-e2e", "--voxels", "16384"]
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=600, cwd=ROOT, env=env)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["config"]["tensors_total"] == 2 * 16384


@pytest.mark.parametrize("world,gather", [(2, "nccl"), (2, "p2p"), (4, "nccl"), (4, "p2p")])
def test_chunked_gather_bitwise_equal_to_one_process(tmp_path, world, gather):
    """C5 invariant: dedup records gathered from P = 2 and 4 ranks, each solving its range
    in 3 chunks, equal bit for bit those of one process solving the whole volume in one call — through the
    collective (gloo stands in for NCCL on one GPU) and through peer memory (the dedup kernels of ranks
    1..P-1 storing into rank 0's IPC-mapped buffer)."""
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import numpy as np
    import paper_conf_ipps_ballardkp11_b200 as sh
    import synthetic as syn
    nloc, kmax = 16384 // world, 4
    dump = str(tmp_path / "rec.npz")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", str(world),
           "--master-addr", "127.0.0.1", "--master-port", str(_port()), os.path.join(ROOT, "bench.py"),
           "--gpus", str(world), "--steps", "1", "--warmup", "3", "--backend", "gloo", "--no-cpu", "--no-e2e",
           "--voxels", str(nloc), "--gather-chunks", "3", "--dump-records", dump, "--gather", gather]
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=600, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-2000:]
    got = np.load(dump)
    cfg = syn.CONFIGS["C2"]
    m, n, S = cfg["m"], cfg["n"], cfg["S"]
    dev = torch.device("cuda:0")
    ent = torch.from_numpy(syn.gen_voxels(m, n, 0, world * nloc, seed=0)).to(dev)
    st = torch.from_numpy(syn.gen_starts(S, n, seed=0)).to(dev)
    solver = sh.Solver(m, n)
    lam, x, it, cv = solver.solve(ent, st, cfg["alpha"], cfg["tol"], cfg["maxit"])
    ref = solver.dedup(lam, x, cv, 1e-2, 0.05, kmax)
    torch.cuda.synchronize()
    for name, a in zip(("count", "lam", "x", "mult", "rep"), ref):
        a = a.cpu().numpy()
        b = got[name]
        assert a.shape == b.shape, name
        assert np.array_equal(a.view(np.int32) if a.dtype == np.float32 else a,
                              b.view(np.int32) if b.dtype == np.float32 else b), name
