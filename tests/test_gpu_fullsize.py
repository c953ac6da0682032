"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py times.

The GPU solves the whole configured volume through the C ABI (same defaults
as bench.py); the oracle then recomputes a fixed, spread sample of tensors
one by one (regenerated from the counter-based generator) and the sampled
outputs must satisfy the parity contract (tests/parity.py).  Properties that
hold at any size (unit norm, iteration bounds, flag/iteration consistency)
are checked on every lane.
"""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import paper_conf_ipps_ballardkp11_b200 as sh  # noqa: E402
import synthetic as syn  # noqa: E402
from tests import parity as PR  # noqa: E402

# config -> number of sampled tensors checked against the oracle
SAMPLES = {"C2": 512, "C2a": 384, "C3": 192, "C4a": 32, "C4b": 128, "C5": 512}


@pytest.fixture(scope="module")
def dev():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    return torch.device("cuda:0")


@pytest.mark.parametrize("cfg_name", ["C2", "C2a", "C3", "C4a", "C4b", "C5"])
def test_fullsize_sampled_parity(dev, cfg_name):
    """C5 is the whole 2^23-tensor volume on one GPU (the multi-GPU config's data)."""
    c = syn.CONFIGS[cfg_name]
    m, n, N, S = c["m"], c["n"], c["N"], c["S"]
    ent = syn.gen_voxels(m, n, 0, N, seed=0)
    st = syn.gen_starts(S, n, seed=0)
    solver = sh.Solver(m, n)
    lam, x, it, cv = solver.solve(torch.from_numpy(ent).to(dev), torch.from_numpy(st).to(dev),
                                  c["alpha"], c["tol"], c["maxit"])
    torch.cuda.synchronize()
    # properties on every lane
    nx = torch.linalg.vector_norm(x, dim=2)
    assert float((nx - 1).abs().max()) < 2e-6
    assert int(it.min()) >= 0 and int(it.max()) <= c["maxit"]
    assert bool(((cv == 1) <= (it >= 1)).all())          # converged lanes made at least one update
    assert float((cv == 1).float().mean()) > 0.98
    # sampled tensors vs the oracle
    k = SAMPLES[cfg_name]
    idx = np.unique(np.linspace(0, N - 1, k).astype(np.int64))
    sel = torch.from_numpy(idx).to(dev)
    gpu = tuple(t.index_select(0, sel).cpu().numpy() for t in (lam, x, it, cv))
    rep = PR.solve_parity(ent[idx], st, m, n, c["alpha"], c["tol"], c["maxit"], gpu)
    print(cfg_name, {kk: v for kk, v in rep.items() if kk != "details"})
    PR.record(f"test_fullsize_sampled_parity[{cfg_name}]", dict(rep, tensors=N, sampled_tensors=int(len(idx))))
    assert rep["flag_unexplained"] == 0, rep
    assert rep["lam_unexplained"] == 0, rep
    assert rep["angle_unexplained"] == 0, rep
    # C2a (alpha = 0.5) converges slowly, so more lanes end at the stopping boundary, where FP32 / FP64
    # rounding decides the flag (measured: 76 of 49,152 sampled lanes, all at the boundary, 60 of them
    # also witness-sensitive): DESIGN.md P0 caps explained lanes at 0.5% there, 0.1% elsewhere
    assert rep["sensitive_frac"] <= (5e-3 if cfg_name == "C2a" else 1e-3), rep


@pytest.mark.parametrize("m,n,N,alpha,k", [(4, 10, 16384, 0.0, 24), (6, 6, 16384, 0.5, 16)])
def test_blocked_default_sampled_parity(dev, m, n, N, alpha, k):
    """Larger shapes through the default table-driven path (the blocked kernel) at the size
    tools/large_shapes.py times: every-lane properties, and a spread sample of tensors vs the oracle."""
    ent = syn.gen_voxels(m, n, 0, N, seed=0)
    st = syn.gen_starts(128, n, seed=0)
    solver = sh.Solver(m, n)
    lam, x, it, cv = solver.solve(torch.from_numpy(ent).to(dev), torch.from_numpy(st).to(dev), alpha, 1e-6, 100)
    torch.cuda.synchronize()
    nx = torch.linalg.vector_norm(x, dim=2)
    assert float((nx - 1).abs().max()) < 5e-6
    assert int(it.min()) >= 0 and int(it.max()) <= 100
    assert float((cv == 1).float().mean()) > 0.95
    idx = np.unique(np.linspace(0, N - 1, k).astype(np.int64))
    sel = torch.from_numpy(idx).to(dev)
    gpu = tuple(t.index_select(0, sel).cpu().numpy() for t in (lam, x, it, cv))
    rep = PR.solve_parity(ent[idx], st, m, n, alpha, 1e-6, 100, gpu)
    print((m, n), {kk: v for kk, v in rep.items() if kk != "details"})
    PR.record(f"test_blocked_default_sampled_parity[{m}-{n}]", dict(rep, tensors=N, sampled_tensors=int(len(idx))))
    assert rep["flag_unexplained"] == 0, rep
    assert rep["lam_unexplained"] == 0, rep
    assert rep["angle_unexplained"] == 0, rep
    assert rep["sensitive_frac"] <= 0.02, rep
