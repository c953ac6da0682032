"""GPU parity tests: CUDA path (through the C ABI) vs the FP64 oracle.

Run on a B200 with ``pytest -m gpu``.  Inputs come from synthetic/ (seeded);
expected values come only from oracle/.
"""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import paper_conf_ipps_ballardkp11_b200 as sh  # noqa: E402
import synthetic as syn  # noqa: E402
from oracle import sshopm as O  # noqa: E402
from oracle import dedup as D  # noqa: E402
from tests import parity as PR  # noqa: E402


@pytest.fixture(scope="module")
def dev():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    return torch.device("cuda:0")


def _solve(dev, m, n, ent, st, alpha, tol, maxit, **kw):
    s = sh.Solver(m, n)
    out = s.solve(torch.from_numpy(ent).to(dev), torch.from_numpy(st).to(dev), alpha, tol, maxit, **kw)
    torch.cuda.synchronize()
    return tuple(t.cpu().numpy() for t in out)


_CURRENT = {"name": None}


@pytest.fixture(autouse=True)
def _test_name(request):
    _CURRENT["name"] = request.node.name
    yield
    _CURRENT["name"] = None


def _record(rep, **extra):
    """Write the parity report of the running test to gpurun_out/parity/<test>.json (the auditable evidence
    of how many lanes each rule explained; summarised under profiles/ by tools/parity_summary.py)."""
    PR.record(_CURRENT["name"] or "unnamed", dict(rep, **extra))


def _assert_parity(rep, max_sensitive=1e-3):
    """P1-P3 with zero unexplained lanes; explained (precision-sensitive) lanes must stay rare."""
    print({k: v for k, v in rep.items() if k != "details"})
    _record(rep, max_sensitive=max_sensitive)
    assert rep["flag_unexplained"] == 0, rep
    assert rep["lam_unexplained"] == 0, rep
    assert rep.get("angle_unexplained", 0) == 0, rep
    assert rep["sensitive_frac"] <= max_sensitive, rep


# ---------------------------------------------------------------- apply (T2) --
def _exact_inputs(m, n, count, seed):
    amax = 5
    xmax = 3 if m <= 4 else 1
    return syn.gen_small_int(m, n, count, seed, amax), syn.gen_int_vectors(count, n, seed + 1, xmax)


@pytest.mark.parametrize("m,n", [(2, 2), (2, 3), (2, 4), (3, 2), (3, 3), (3, 4), (4, 2), (4, 3), (4, 4), (4, 5),
                                 (4, 6), (5, 3), (6, 2), (6, 3), (8, 3)])
def test_apply_exact_on_integers(dev, m, n):
    """Eq. 6 and Eq. 4 (Euler) in FP32 == FP64 full-tensor oracle, bit-exact on small integers."""
    ent, x = _exact_inputs(m, n, 1000, m * 7 + n)
    s = sh.Solver(m, n)
    g, lam = s.apply(torch.from_numpy(ent).to(dev), torch.from_numpy(x).to(dev))
    full = O.expand_full(ent, m, n)
    g_ref = O.axm1(full, x.astype(np.float64))
    lam_ref = O.axm(full, x.astype(np.float64))
    assert np.abs(g_ref).max() < 2 ** 24 and np.abs(lam_ref).max() < 2 ** 24
    assert np.array_equal(g.cpu().numpy().astype(np.float64), g_ref)
    assert np.array_equal(lam.cpu().numpy().astype(np.float64), lam_ref)


def test_apply_random_close(dev):
    m, n = 4, 3
    ent = syn.gen_voxels(m, n, 0, 4096, 1)
    x = O.normalise_starts(syn.gen_starts(4096, n, 3)).astype(np.float32)
    g, lam = sh.Solver(m, n).apply(torch.from_numpy(ent).to(dev), torch.from_numpy(x).to(dev))
    full = O.expand_full(ent, m, n)
    assert np.allclose(g.cpu().numpy(), O.axm1(full, x.astype(np.float64)), atol=2e-6)
    assert np.allclose(lam.cpu().numpy(), O.axm(full, x.astype(np.float64)), atol=2e-6)


# ------------------------------------------------------------ solve parity --
def test_parity_C1_full(dev):
    """Config C1: all 1024 x 128 lanes, alpha = 0, tol 1e-6, maxit 100."""
    c = syn.CONFIGS["C1"]
    m, n = c["m"], c["n"]
    ent = syn.gen_voxels(m, n, 0, c["N"], 0)
    st = syn.gen_starts(c["S"], n, 0)
    gpu = _solve(dev, m, n, ent, st, c["alpha"], c["tol"], c["maxit"])
    rep = PR.solve_parity(ent, st, m, n, c["alpha"], c["tol"], c["maxit"], gpu)
    _assert_parity(rep)
    assert rep["gpu_converged"] > 0.99
    assert np.allclose(np.linalg.norm(gpu[1], axis=2), 1.0, atol=1e-6)


@pytest.mark.parametrize("m,n,V,alpha", [(4, 3, 256, 0.5), (4, 3, 128, -0.5), (6, 3, 128, 0.25), (8, 3, 24, 0.5),
                                         (4, 6, 64, 0.0), (2, 3, 64, 1.0), (3, 3, 64, 1.0), (3, 2, 64, 0.5),
                                         (4, 5, 32, 0.0), (5, 3, 32, 0.5), (6, 2, 64, 0.25), (4, 4, 64, 0.25)])
def test_parity_shapes(dev, m, n, V, alpha):
    """Other orders / dimensions / shifts.  Odd m uses unstructured U[-1,1] tensors and alpha < 0 seeks
    minima below the concavity bound, so more lanes are precision-sensitive there (<= 5%)."""
    ent = syn.gen_voxels(m, n, 12345, V, 2) if m % 2 == 0 else syn.gen_uniform_tensors(m, n, V, 2)
    st = syn.gen_starts(128, n, 5)
    gpu = _solve(dev, m, n, ent, st, alpha, 1e-6, 100)
    stress = m % 2 == 1 or alpha < 0
    _assert_parity(PR.solve_parity(ent, st, m, n, alpha, 1e-6, 100, gpu), 0.05 if stress else 1e-3)


@pytest.mark.parametrize("alpha,K", [(0.0, 1), (0.0, 5), (0.0, 10), (0.5, 5), (0.5, 10)])
def test_fixed_k(dev, alpha, K):
    m, n = 4, 3
    ent = syn.gen_voxels(m, n, 0, 256, 0)
    st = syn.gen_starts(128, n, 0)
    lam, x, it, cv = _solve(dev, m, n, ent, st, alpha, -1.0, K)
    assert (it == K).all() and not cv.any()
    r = PR.fixed_k_parity(ent, st, m, n, alpha, K, lam)
    print(r)
    _record(r)
    assert r["unexplained"] == 0, r


@pytest.mark.parametrize("K", [1, 5, 10])
@pytest.mark.parametrize("m,n,V,alpha,schedule", [(6, 3, 96, 0.25, 0), (8, 3, 24, 0.5, 0), (4, 6, 48, 0.0, 0),
                                                  (4, 3, 64, 0.5, 5), (5, 4, 24, 4.0, 5), (6, 4, 16, 0.5, 3),
                                                  (4, 3, 64, 0.0, 2)])
def test_fixed_k_shapes(dev, m, n, V, alpha, schedule, K):
    """Fixed-K lambda (tol < 0: exactly K updates, Fig. 1) within 1e-5 relative of the FP64 oracle (P4) for
    the C3 / C4a / C4b shapes on their unrolled kernels, the blocked (5) and item-per-lane (3) table-driven
    kernels and the tensor-per-lane schedule (2)."""
    ent = syn.gen_voxels(m, n, 300, V, 6) if m % 2 == 0 else syn.gen_uniform_tensors(m, n, V, 6)
    st = syn.gen_starts(64, n, 3)
    lam, x, it, cv = _solve(dev, m, n, ent, st, alpha, -1.0, K, schedule=schedule)
    assert (it == K).all() and not cv.any()
    r = PR.fixed_k_parity(ent, st, m, n, alpha, K, lam)
    print(r)
    _record(r)
    assert r["unexplained"] == 0, r


@pytest.mark.parametrize("m,n,schedule", [(4, 3, 0), (4, 3, 5), (4, 3, 3), (5, 4, 0)])
def test_special_cases(dev, m, n, schedule):
    """maxit = 0 -> (lam_0, x_0); zero start -> 0; odd S, N not a multiple of anything — for the
    unrolled kernel, the blocked (5) and item-per-lane (3) table-driven kernels, and a shape without
    a compiled kernel (default: blocked)."""
    ent = syn.gen_voxels(m, n, 0, 37, 0) if m % 2 == 0 else syn.gen_uniform_tensors(m, n, 37, 0)
    alpha = 0.0 if m % 2 == 0 else 2.0
    st = syn.gen_starts(13, n, 0)
    st[4] = 0.0
    lam, x, it, cv = _solve(dev, m, n, ent, st, alpha, 1e-6, 0, schedule=schedule)
    assert (it == 0).all() and not cv.any()
    x0 = O.normalise_starts(st)
    assert np.allclose(x, np.broadcast_to(x0, x.shape), atol=1e-7)
    full = O.expand_full(ent, m, n)
    lam0 = O.axm(np.repeat(full, 13, 0), np.tile(x0, (37, 1))).reshape(37, 13)
    assert np.allclose(lam, lam0, atol=1e-5)
    lam, x, it, cv = _solve(dev, m, n, ent, st, alpha, 1e-6, 100, schedule=schedule)
    assert (lam[:, 4] == 0).all() and (x[:, 4] == 0).all() and (it[:, 4] == 0).all() and not cv[:, 4].any()
    _assert_parity(PR.solve_parity(ent, st, m, n, alpha, 1e-6, 100, (lam, x, it, cv)), 0.05 if m % 2 else 1e-3)
    # N = 0 is a no-op
    s = sh.Solver(m, n)
    out = s.solve(torch.zeros((0, ent.shape[1]), device=dev), torch.from_numpy(st).to(dev), alpha, 1e-6, 100,
                  schedule=schedule)
    assert all(t.shape[0] == 0 for t in out)


def test_invariance_across_launch_configs(dev):
    """T4: per-lane arithmetic is order-fixed -> bitwise identical across refill thresholds / grid sizes."""
    m, n = 4, 3
    ent = syn.gen_voxels(m, n, 0, 2048, 3)
    st = syn.gen_starts(128, n, 0)
    base = _solve(dev, m, n, ent, st, 0.0, 1e-6, 100)
    for kw in [dict(refill_threshold=1), dict(refill_threshold=32), dict(ctas_per_sm=1),
               dict(refill_threshold=5, ctas_per_sm=2), {}, dict(schedule=2), dict(schedule=2, refill_threshold=3),
               dict(schedule=2, ctas_per_sm=1, refill_threshold=32), dict(schedule=1), dict(schedule=6),
               dict(schedule=6, refill_threshold=3), dict(schedule=1, chunk_tensors=1),
               dict(schedule=1, chunk_tensors=7, refill_threshold=2)]:
        other = _solve(dev, m, n, ent, st, 0.0, 1e-6, 100, **kw)
        for a, b in zip(base, other):
            assert np.array_equal(a, b), kw


def test_total_iters_counter(dev):
    m, n = 4, 3
    ent = syn.gen_voxels(m, n, 0, 512, 0)
    st = syn.gen_starts(128, n, 0)
    ti = torch.zeros(1, dtype=torch.int64, device=dev)
    lam, x, it, cv = _solve(dev, m, n, ent, st, 0.0, 1e-6, 100, total_iters=ti)
    assert int(ti.item()) == int(it.sum())


# ------------------------------------------------------------------ dedup --
def test_dedup_kernel_matches_oracle_rule_on_same_lanes(dev):
    """GPU dedup vs oracle dedup applied to the GPU's own per-lane results."""
    m, n = 4, 3
    ent = syn.gen_voxels(m, n, 0, 1024, 0)
    st = syn.gen_starts(128, n, 0)
    s = sh.Solver(m, n)
    lam, x, it, cv = s.solve(torch.from_numpy(ent).to(dev), torch.from_numpy(st).to(dev), 0.0, 1e-6, 100)
    for lt, at, kmax in [(1e-2, 0.05, 8), (1e-3, 0.01, 4), (1e-1, 0.5, 2)]:
        cnt, cl, cx, mu, rp = (t.cpu().numpy() for t in s.dedup(lam, x, cv, lt, at, kmax))
        oc, ol, ox, om, orp = D.dedup(lam.cpu().numpy(), x.cpu().numpy(), cv.cpu().numpy().astype(bool), m, lt, at, kmax)
        assert np.array_equal(cnt, oc)
        assert np.array_equal(rp, orp)
        assert np.array_equal(mu, om)
        assert np.array_equal(cl.astype(np.float64), ol)
        assert np.array_equal(cx.astype(np.float64), ox)


def test_dedup_end_to_end_vs_oracle(dev):
    """solve + dedup on GPU vs oracle solve + oracle dedup: identical cluster structure."""
    m, n = 4, 3
    ent = syn.gen_voxels(m, n, 0, 512, 4)
    st = syn.gen_starts(128, n, 0)
    s = sh.Solver(m, n)
    lam, x, it, cv = s.solve(torch.from_numpy(ent).to(dev), torch.from_numpy(st).to(dev), 0.0, 1e-6, 100)
    cnt, cl, cx, mu, rp = (t.cpu().numpy() for t in s.dedup(lam, x, cv, 1e-2, 0.05, 8))
    rl, rx, ri, rc = O.sshopm(ent, st, m, n, 0.0, 1e-6, 100)
    oc, ol, ox, om, orp = D.dedup(rl, rx, rc, m, 1e-2, 0.05, 8)
    flag_diff_vox = np.any(cv.cpu().numpy().astype(bool) != rc, axis=1)
    same = ~flag_diff_vox
    assert same.mean() > 0.98
    assert np.array_equal(cnt[same], oc[same])
    assert np.array_equal(rp[same], orp[same])
    assert np.array_equal(mu[same], om[same])
    filled = rp[same] >= 0
    assert np.all(np.abs(cl[same][filled] - ol[same][filled]) <= 1e-4 * np.maximum(1, np.abs(ol[same][filled])))
    # representatives' eigenvectors: angle to the oracle iterate of the same lane at the GPU's own
    # iteration count (trajectory alignment, parity rule P3), sign-free for even m
    vox, slot = np.nonzero(rp >= 0)
    keep = same[vox]
    vox, slot = vox[keep], slot[keep]
    st_i = rp[vox, slot]
    k_gpu = it.cpu().numpy()[vox, st_i]
    full = O.expand_full(ent, m, n)
    _, xk, _, _ = O.sshopm_lanes(lambda idx: full[vox[idx]], O.normalise_starts(st)[st_i], 0.0, -1.0,
                                 int(k_gpu.max()), k_gpu)
    ang = PR.angle(cx[vox, slot], xk, True)
    _record({"representatives": int(len(vox)), "angle_max": float(ang.max()), "voxels_compared": int(same.sum())})
    assert ang.max() <= PR.ANG_TOL, ang.max()


@pytest.mark.parametrize("S", [16, 100, 128, 200])
def test_dedup_start_counts(dev, S):
    """Register fast path (S = 128) and shared-memory general path (other S) follow the same rule."""
    m, n = 4, 3
    ent = syn.gen_voxels(m, n, 5000, 300, 0)
    st = syn.gen_starts(S, n, 2)
    s = sh.Solver(m, n)
    lam, x, it, cv = s.solve(torch.from_numpy(ent).to(dev), torch.from_numpy(st).to(dev), 0.0, 1e-6, 100)
    cnt, cl, cx, mu, rp = (t.cpu().numpy() for t in s.dedup(lam, x, cv, 1e-2, 0.05, 6))
    oc, ol, ox, om, orp = D.dedup(lam.cpu().numpy(), x.cpu().numpy(), cv.cpu().numpy().astype(bool), m, 1e-2, 0.05, 6)
    assert np.array_equal(cnt, oc) and np.array_equal(rp, orp) and np.array_equal(mu, om)
    assert np.array_equal(cl.astype(np.float64), ol) and np.array_equal(cx.astype(np.float64), ox)


@pytest.mark.parametrize("m,n,V,S", [(4, 10, 6, 32), (3, 9, 8, 40), (6, 12, 3, 16)])
def test_dedup_large_n(dev, m, n, V, S):
    """Dedup for n > 8 (the blocked kernel's shapes): the shared-memory kernel vs the oracle rule on the same
    per-start results."""
    ent = syn.gen_voxels(m, n, 0, V, 5) if m % 2 == 0 else syn.gen_uniform_tensors(m, n, V, 5)
    st = syn.gen_starts(S, n, 4)
    s = sh.Solver(m, n)
    alpha = 0.0 if m % 2 == 0 else 2.0
    lam, x, it, cv = s.solve(torch.from_numpy(ent).to(dev), torch.from_numpy(st).to(dev), alpha, 1e-6, 300)
    cnt, cl, cx, mu, rp = (t.cpu().numpy() for t in s.dedup(lam, x, cv, 1e-2, 0.05, 6))
    oc, ol, ox, om, orp = D.dedup(lam.cpu().numpy(), x.cpu().numpy(), cv.cpu().numpy().astype(bool), m, 1e-2, 0.05, 6)
    assert np.array_equal(cnt, oc) and np.array_equal(rp, orp) and np.array_equal(mu, om)
    assert np.array_equal(cl.astype(np.float64), ol) and np.array_equal(cx.astype(np.float64), ox)


def test_dedup_odd_m(dev):
    m, n = 3, 3
    ent = syn.gen_uniform_tensors(m, n, 128, 1)
    st = syn.gen_starts(128, n, 0)
    s = sh.Solver(m, n)
    lam, x, it, cv = s.solve(torch.from_numpy(ent).to(dev), torch.from_numpy(st).to(dev), 1.0, 1e-6, 200)
    cnt, cl, cx, mu, rp = (t.cpu().numpy() for t in s.dedup(lam, x, cv, 1e-2, 0.05, 8))
    oc, ol, ox, om, orp = D.dedup(lam.cpu().numpy(), x.cpu().numpy(), cv.cpu().numpy().astype(bool), m, 1e-2, 0.05, 8)
    assert np.array_equal(cnt, oc) and np.array_equal(rp, orp) and np.array_equal(mu, om)


# --------------------------------------------------------------- host path --
def test_run_host_matches_device_path(dev):
    m, n = 4, 3
    ent = syn.gen_voxels(m, n, 0, 3000, 9)
    st = syn.gen_starts(128, n, 0)
    s = sh.Solver(m, n)
    out = s.run_host(ent, st, 0.0, 1e-6, 100, 1e-2, 0.05, 8, raw=True, chunk_tensors=700)
    lam, x, it, cv = s.solve(torch.from_numpy(ent).to(dev), torch.from_numpy(st).to(dev), 0.0, 1e-6, 100)
    cnt, cl, cx, mu, rp = s.dedup(lam, x, cv, 1e-2, 0.05, 8)
    torch.cuda.synchronize()
    assert np.array_equal(out["raw_lambda"], lam.cpu().numpy())
    assert np.array_equal(out["raw_x"], x.cpu().numpy())
    assert np.array_equal(out["raw_iters"], it.cpu().numpy())
    assert np.array_equal(out["raw_converged"], cv.cpu().numpy())
    assert np.array_equal(out["count"], cnt.cpu().numpy())
    assert np.array_equal(out["rep"], rp.cpu().numpy())
    assert np.array_equal(out["lambda"], cl.cpu().numpy())
    assert out["total_iters"] == int(it.cpu().numpy().sum())


@pytest.mark.parametrize("V,chunk", [(4005, 1001), (4013, 1003), (5000, 1001)])
def test_run_host_ramp_chunk_not_multiple_of_4(dev, V, chunk):
    """run_host's ramped chunk sizes never exceed the chunk buffers (regression: with chunk % 4 != 0 the
    ramp-down chunk left - chunk/4 could exceed chunk by up to 3 tensors -> H2D past the buffer)."""
    m, n = 4, 3
    ent = syn.gen_voxels(m, n, 0, V, 9)
    st = syn.gen_starts(32, n, 0)
    s = sh.Solver(m, n)
    out = s.run_host(ent, st, 0.0, 1e-6, 100, 1e-2, 0.05, 4, chunk_tensors=chunk)
    lam, x, it, cv = s.solve(torch.from_numpy(ent).to(dev), torch.from_numpy(st).to(dev), 0.0, 1e-6, 100)
    cnt, cl, cx, mu, rp = s.dedup(lam, x, cv, 1e-2, 0.05, 4)
    torch.cuda.synchronize()
    assert np.array_equal(out["count"], cnt.cpu().numpy())
    assert np.array_equal(out["lambda"], cl.cpu().numpy())
    assert np.array_equal(out["x"], cx.cpu().numpy())


@pytest.mark.parametrize("schedule", [1, 2, 6])
@pytest.mark.parametrize("V,S", [(1, 1), (3, 1), (5, 7), (40, 2), (2, 300)])
def test_tiny_chunks(dev, V, S, schedule):
    """Chunks smaller than a warp's request (S * tensors < 32) must not overrun (regression)."""
    m, n = 4, 3
    ent = syn.gen_voxels(m, n, 77, V, 0)
    st = syn.gen_starts(S, n, 1)
    gpu = _solve(dev, m, n, ent, st, 0.0, 1e-6, 100, schedule=schedule)
    _assert_parity(PR.solve_parity(ent, st, m, n, 0.0, 1e-6, 100, gpu), max_sensitive=0.02)


def test_empty_and_tiny(dev):
    m, n = 4, 3
    s = sh.Solver(m, n)
    e0 = torch.zeros((0, 15), device=dev)
    st = torch.from_numpy(syn.gen_starts(8, 3, 0)).to(dev)
    lam, x, it, cv = s.solve(e0, st)
    assert lam.shape == (0, 8)
    ent = syn.gen_voxels(m, n, 0, 1, 0)
    st1 = syn.gen_starts(1, n, 0)
    gpu = _solve(dev, m, n, ent, st1, 0.0, 1e-6, 100)
    _assert_parity(PR.solve_parity(ent, st1, m, n, 0.0, 1e-6, 100, gpu))


# ------------------------------------------------------- fused solve->dedup --
def _two_pass(dev, m, n, ent, st, alpha, tol, maxit, lt, at, kmax, **kw):
    s = sh.Solver(m, n)
    e, t = torch.from_numpy(ent).to(dev), torch.from_numpy(st).to(dev)
    raw = s.solve(e, t, alpha, tol, maxit, **kw)
    dd = s.dedup(raw[0], raw[1], raw[3], lt, at, kmax)
    torch.cuda.synchronize()
    return [x.cpu().numpy() for x in raw], [x.cpu().numpy() for x in dd]


def _fused(dev, m, n, ent, st, alpha, tol, maxit, lt, at, kmax, **kw):
    s = sh.Solver(m, n)
    e, t = torch.from_numpy(ent).to(dev), torch.from_numpy(st).to(dev)
    raw, dd = s.solve_dedup(e, t, alpha, tol, maxit, lt, at, kmax, fused=True, **kw)
    torch.cuda.synchronize()
    return [x.cpu().numpy() for x in raw], [x.cpu().numpy() for x in dd]


@pytest.mark.parametrize("m,n,V,S,alpha,kmax", [(4, 3, 3000, 128, 0.0, 4), (4, 3, 777, 100, 0.0, 8), (6, 3, 500, 128, 0.25, 6),
                                                (3, 3, 400, 64, 1.0, 5), (4, 6, 200, 128, 0.0, 4), (8, 3, 100, 32, 0.5, 3),
                                                (4, 3, 50, 300, 0.0, 4)])
def test_fused_equals_two_pass(dev, m, n, V, S, alpha, kmax):
    """sshopm_solve_dedup == sshopm_solve + sshopm_dedup, bit for bit (raw and dedup outputs)."""
    ent = syn.gen_voxels(m, n, 900, V, 1) if m % 2 == 0 else syn.gen_uniform_tensors(m, n, V, 1)
    st = syn.gen_starts(S, n, 3)
    ra, da = _two_pass(dev, m, n, ent, st, alpha, 1e-6, 100, 1e-2, 0.05, kmax)
    rb, db = _fused(dev, m, n, ent, st, alpha, 1e-6, 100, 1e-2, 0.05, kmax)
    for a, b in zip(ra + da, rb + db):
        assert np.array_equal(a, b)


def test_fused_vs_oracle(dev):
    """The fused solve->dedup path against the FP64 oracle directly: its per-start outputs pass the parity
    contract (P1-P3) and its records equal the oracle's R16 rule applied to the same lanes; on voxels without
    a flag difference, cluster counts / representatives / multiplicities equal oracle solve + oracle dedup."""
    m, n, V, S = 4, 3, 600, 128
    ent = syn.gen_voxels(m, n, 2000, V, 7)
    st = syn.gen_starts(S, n, 0)
    raw, dd = _fused(dev, m, n, ent, st, 0.0, 1e-6, 100, 1e-2, 0.05, 8)
    _assert_parity(PR.solve_parity(ent, st, m, n, 0.0, 1e-6, 100, tuple(raw)))
    oc, ol, ox, om, orp = D.dedup(raw[0], raw[1], raw[3].astype(bool), m, 1e-2, 0.05, 8)
    for a, b in zip(dd, (oc, ol, ox, om, orp)):
        assert np.array_equal(np.asarray(a).astype(np.float64), np.asarray(b).astype(np.float64))
    rl, rx, ri, rc = O.sshopm(ent, st, m, n, 0.0, 1e-6, 100)
    oc2, ol2, ox2, om2, orp2 = D.dedup(rl, rx, rc, m, 1e-2, 0.05, 8)
    same = ~np.any(raw[3].astype(bool) != rc, axis=1)
    assert same.mean() > 0.98
    assert np.array_equal(dd[0][same], oc2[same]) and np.array_equal(dd[4][same], orp2[same])
    assert np.array_equal(dd[3][same], om2[same])


@pytest.mark.parametrize("m,n,V,S,alpha,maxit", [(4, 3, 3000, 128, 0.0, 100), (4, 3, 777, 100, 0.0, 100),
                                                  (6, 3, 300, 128, 0.25, 100), (4, 6, 100, 64, 0.0, 100),
                                                  (3, 3, 200, 128, 1.0, 100), (4, 3, 5, 7, 0.0, 100),
                                                  (4, 3, 2000, 128, 0.0, 3000)])
def test_schedule7_bitwise(dev, m, n, V, S, alpha, maxit):
    """Warp-tensor pipeline (schedule 7): raw outputs bitwise equal to schedule 1 (same per-lane arithmetic);
    fused (clustering from the staging) and records-only forms give the two-pass records bit for bit."""
    ent = syn.gen_voxels(m, n, 40, V, 4) if m % 2 == 0 else syn.gen_uniform_tensors(m, n, V, 4)
    if maxit > 1000:
        ent[::40] = syn.gen_uniform_tensors(m, n, V // 40, 9)      # slow lanes: tensors held open for long
    st = syn.gen_starts(S, n, 0)
    a = _solve(dev, m, n, ent, st, alpha, 1e-6, maxit, schedule=1)
    b = _solve(dev, m, n, ent, st, alpha, 1e-6, maxit, schedule=7)
    for u, v in zip(a, b):
        assert np.array_equal(u, v)
    ra, da = _two_pass(dev, m, n, ent, st, alpha, 1e-6, maxit, 1e-2, 0.05, 4)
    s = sh.Solver(m, n)
    e, t = torch.from_numpy(ent).to(dev), torch.from_numpy(st).to(dev)
    rb, db = s.solve_dedup(e, t, alpha, 1e-6, maxit, 1e-2, 0.05, 4, schedule=7, fused=True)
    rc, dc = s.solve_dedup(e, t, alpha, 1e-6, maxit, 1e-2, 0.05, 4, records_only=True)
    torch.cuda.synchronize()
    for u, v in zip(ra + da, [x.cpu().numpy() for x in rb + db]):
        assert np.array_equal(u, v)
    for u, v in zip(da, [x.cpu().numpy() for x in dc]):
        assert np.array_equal(u, v)


@pytest.mark.parametrize("alpha", ["per_tensor", "auto_max", 0.5, -0.5])
@pytest.mark.parametrize("schedule", [6, 7])
def test_schedules_6_7_shift_modes_bitwise(dev, alpha, schedule):
    """Schedules 6 (predicated refill) and 7 (warp-tensor pipeline) with every shift kind (per-tensor, automatic,
    positive, negative): bitwise equal to schedule 1."""
    m, n, V, S = 4, 3, 700, 100
    ent = syn.gen_voxels(m, n, 11, V, 3)
    st = syn.gen_starts(S, n, 2)
    if alpha == "per_tensor":
        rng = np.random.default_rng(5)
        alpha = torch.from_numpy(rng.choice([0.0, 0.5, -0.5, 1.0], size=V).astype(np.float32)).to(dev)
    a = _solve(dev, m, n, ent, st, alpha, 1e-6, 200, schedule=1)
    b = _solve(dev, m, n, ent, st, alpha, 1e-6, 200, schedule=schedule)
    for u, v in zip(a, b):
        assert np.array_equal(u, v)


def test_records_only_overflow(dev):
    """Records-only path with tensors of more than 32 clusters (tight tolerances on unstructured odd-m tensors):
    those tensors take the raw-output + list-kernel route; records equal the two-pass form."""
    m, n, V, S = 3, 3, 64, 128
    ent = syn.gen_uniform_tensors(m, n, V, 2)
    st = syn.gen_starts(S, n, 1)
    ra, da = _two_pass(dev, m, n, ent, st, 1.0, 1e-6, 100, 1e-7, 1e-6, 8)
    assert (da[0] > 32).any()                                    # some tensors overflow the register form
    s = sh.Solver(m, n)
    e, t = torch.from_numpy(ent).to(dev), torch.from_numpy(st).to(dev)
    rc, dc = s.solve_dedup(e, t, 1.0, 1e-6, 100, 1e-7, 1e-6, 8, records_only=True)
    torch.cuda.synchronize()
    for u, v in zip(da, [x.cpu().numpy() for x in dc]):
        assert np.array_equal(u, v)


def test_plain_sshopm_solve_entry_point(dev):
    """sshopm_solve itself: library defaults and its own cudaMallocAsync workspace, data on
    the GPU; bitwise equal to sshopm_solve_ex and within the parity contract."""
    m, n = 4, 3
    ent = syn.gen_voxels(m, n, 100, 512, 2)
    st = syn.gen_starts(128, n, 1)
    s = sh.Solver(m, n)
    e, t = torch.from_numpy(ent).to(dev), torch.from_numpy(st).to(dev)
    a = [u.cpu().numpy() for u in s.solve_plain(e, t, 0.0, 1e-6, 100)]
    b = [u.cpu().numpy() for u in s.solve(e, t, 0.0, 1e-6, 100)]
    for u, v in zip(a, b):
        assert np.array_equal(u, v)
    _assert_parity(PR.solve_parity(ent, st, m, n, 0.0, 1e-6, 100, tuple(a)))


@pytest.mark.parametrize("m,n,V,S,alpha,maxit", [(4, 3, 3000, 128, 0.0, 100), (4, 3, 777, 100, 0.0, 100),
                                                  (6, 3, 500, 128, 0.25, 100), (3, 3, 400, 64, 1.0, 100),
                                                  (4, 3, 2000, 128, 0.0, 3000)])
def test_fused_warp_specialised_equals_two_pass(dev, m, n, V, S, alpha, maxit):
    """Fused mode 3 (one dedup warp per CTA consumes the chunks the solve warps complete): raw and dedup
    outputs bit for bit those of the two-pass form, including slow tensors that overflow the rings."""
    ent = syn.gen_voxels(m, n, 900, V, 1) if m % 2 == 0 else syn.gen_uniform_tensors(m, n, V, 1)
    if maxit > 1000:
        ent[::40] = syn.gen_uniform_tensors(m, n, V // 40, 9)
    st = syn.gen_starts(S, n, 3)
    ra, da = _two_pass(dev, m, n, ent, st, alpha, 1e-6, maxit, 1e-2, 0.05, 4)
    s = sh.Solver(m, n)
    e, t = torch.from_numpy(ent).to(dev), torch.from_numpy(st).to(dev)
    rb, db = s.solve_dedup(e, t, alpha, 1e-6, maxit, 1e-2, 0.05, 4, warp_specialized=True)
    torch.cuda.synchronize()
    for a, b in zip(ra + da, [x.cpu().numpy() for x in rb + db]):
        assert np.array_equal(a, b)


def test_fused_ring_overflow(dev):
    """Chunks held open for thousands of steps by slow lanes overflow the per-warp ring; the
    follow-up list kernel must still cluster them (results identical to the two-pass form)."""
    m, n, V, S = 4, 3, 6000, 128
    ent = syn.gen_voxels(m, n, 0, V, 4)
    slow = syn.gen_uniform_tensors(m, n, V // 40, 9)      # unstructured, alpha = 0: many non-converging starts
    ent[::40] = slow
    st = syn.gen_starts(S, n, 0)
    ra, da = _two_pass(dev, m, n, ent, st, 0.0, 1e-6, 3000, 1e-2, 0.05, 4)
    rb, db = _fused(dev, m, n, ent, st, 0.0, 1e-6, 3000, 1e-2, 0.05, 4)
    assert ra[2].max() == 3000 and (ra[2] == 3000).sum() > 100    # slow lanes really ran to maxit
    for a, b in zip(ra + da, rb + db):
        assert np.array_equal(a, b)


# --------------------------------------------------------------- shift modes --
def test_per_tensor_alpha_parity(dev):
    """alpha_mode 1: one shift per tensor (mixed signs) vs the oracle with the same per-voxel shifts."""
    m, n, V = 4, 3, 256
    ent = syn.gen_voxels(m, n, 4242, V, 0)
    st = syn.gen_starts(128, n, 0)
    rng = np.random.default_rng(3)
    al = rng.choice([0.0, 0.25, 0.5, 1.0, -0.5], size=V).astype(np.float32)
    s = sh.Solver(m, n)
    out = s.solve(torch.from_numpy(ent).to(dev), torch.from_numpy(st).to(dev), torch.from_numpy(al).to(dev), 1e-6, 100)
    torch.cuda.synchronize()
    gpu = tuple(t.cpu().numpy() for t in out)
    _assert_parity(PR.solve_parity(ent, st, m, n, al.astype(np.float64), 1e-6, 100, gpu), 0.02)
    # a constant array equals the scalar path bit for bit
    c = torch.full((V,), 0.5, dtype=torch.float32, device=dev)
    a1 = [t.cpu().numpy() for t in s.solve(torch.from_numpy(ent).to(dev), torch.from_numpy(st).to(dev), c, 1e-6, 100)]
    a2 = [t.cpu().numpy() for t in s.solve(torch.from_numpy(ent).to(dev), torch.from_numpy(st).to(dev), 0.5, 1e-6, 100)]
    for a, b in zip(a1, a2):
        assert np.array_equal(a, b)


@pytest.mark.parametrize("mode,sign", [("auto_max", 1.0), ("auto_min", -1.0)])
def test_auto_shift_monotone_and_parity(dev, mode, sign):
    """alpha = +-(m-1) sum|a| (R17): every GPU lambda trajectory is monotone, all lanes converge,
    and results match the oracle run with its own independently computed shift."""
    from oracle import sshopm as OR
    m, n, V = 4, 3, 64
    ent = syn.gen_uniform_tensors(m, n, V, 8)            # unstructured: alpha = 0 would often fail
    st = syn.gen_starts(32, n, 2)
    s = sh.Solver(m, n)
    e, t = torch.from_numpy(ent).to(dev), torch.from_numpy(st).to(dev)
    prev = None
    for K in range(0, 30):
        lamK = s.solve(e, t, mode, -1.0, K)[0].cpu().numpy()
        if prev is not None:
            assert np.all(sign * (lamK - prev) >= -2e-5 * np.maximum(1, np.abs(prev)))
        prev = lamK
    lam, x, it, cv = (u.cpu().numpy() for u in s.solve(e, t, mode, 1e-6, 2000))
    assert cv.mean() > 0.99
    al = sign * OR.convexity_shift(ent, m, n)
    _assert_parity(PR.solve_parity(ent, st, m, n, al, 1e-6, 2000, (lam, x, it, cv)), 0.02)


# ------------------------------------------------------- general (table) kernel --
@pytest.mark.parametrize("m,n", [(5, 4), (7, 2), (3, 6), (9, 3), (4, 3)])
def test_general_apply_exact(dev, m, n):
    """Table-driven Eq. 6 (any (m, n)) is bit-exact on small integers like the unrolled kernels."""
    ent, x = _exact_inputs(m, n, 300, m * 11 + n)
    if m >= 7:
        ent = np.clip(ent, -2, 2)
    full = O.expand_full(ent, m, n)
    g_ref = O.axm1(full, x.astype(np.float64))
    lam_ref = O.axm(full, x.astype(np.float64))
    assert np.abs(g_ref).max() < 2 ** 24 and np.abs(lam_ref).max() < 2 ** 24
    s = sh.Solver(m, n)
    if (m, n) in set(sh.supported_shapes()):
        pytest.skip("compiled shape: apply uses the unrolled kernel")
    g, lam = s.apply(torch.from_numpy(ent).to(dev), torch.from_numpy(x).to(dev))
    assert np.array_equal(g.cpu().numpy().astype(np.float64), g_ref)
    assert np.array_equal(lam.cpu().numpy().astype(np.float64), lam_ref)


@pytest.mark.parametrize("m,n,V,alpha", [(5, 4, 24, 4.0), (6, 4, 16, 0.5), (3, 6, 16, 3.0), (10, 2, 32, 0.5), (4, 8, 8, 0.0),
                                         (6, 5, 6, 0.5), (3, 9, 8, 1.0)])
@pytest.mark.parametrize("schedule", [0, 3, 4, 5])
def test_general_solve_parity(dev, m, n, V, alpha, schedule):
    """(m, n) without a compiled kernel vs the oracle: the default choice, the item-per-lane general
    kernel (3; n = 9 takes its 16-wide register variant), the block-per-tensor one (4) and the
    blocked warp-per-tensor one (5)."""
    ent = syn.gen_voxels(m, n, 0, V, 3) if m % 2 == 0 else syn.gen_uniform_tensors(m, n, V, 3)
    st = syn.gen_starts(64, n, 1)
    gpu = _solve(dev, m, n, ent, st, alpha, 1e-6, 200, schedule=schedule)
    # even m with alpha >= 0 (structured voxel tensors): the benchmark bar, <= 0.1% precision-sensitive lanes;
    # odd m (unstructured tensors, sign-flip trajectories) keeps the stress bar
    _assert_parity(PR.solve_parity(ent, st, m, n, alpha, 1e-6, 200, gpu), 1e-3 if m % 2 == 0 else 0.05)


@pytest.mark.parametrize("shift", ["auto_max", "auto_min"])
def test_general_item_kernel_shift_modes(dev, shift):
    """Item-per-lane general kernel with the automatic convex / concave shifts and ragged chunks
    (S = 100, V = 37): in fixed-K mode (tol < 0, 50 updates) its lambda_K equals the
    block-per-tensor kernel's up to FP32 summation order (both compute the same shift, R17,
    in the same class order); scalar shifts are covered against the oracle above."""
    m, n, V, S = 5, 4, 37, 100
    ent = syn.gen_uniform_tensors(m, n, V, 11)
    st = syn.gen_starts(S, n, 2)
    a = _solve(dev, m, n, ent, st, shift, -1.0, 50, schedule=3)
    b = _solve(dev, m, n, ent, st, shift, -1.0, 50, schedule=4)
    assert np.all(a[2] == 50) and np.all(b[2] == 50) and not a[3].any()
    assert np.all(np.abs(a[0] - b[0]) <= 1e-4 * np.maximum(1, np.abs(b[0])))
    if shift == "auto_max":   # convex shift: lambda_k nondecreasing, so lambda_K >= lambda_0 = A x0^m
        lam0 = _solve(dev, m, n, ent, st, shift, -1.0, 0, schedule=3)[0]
        assert np.all(a[0] >= lam0 - 1e-4 * np.maximum(1, np.abs(lam0)))


# ------------------------------------------------------- blocked kernel (8(f) row 4) --
@pytest.mark.parametrize("m,n,V,S,alpha", [(2, 5, 40, 64, 2.0), (3, 4, 33, 100, 1.5), (4, 3, 50, 128, 0.0),
                                           (4, 10, 6, 32, 0.0), (6, 6, 5, 48, 0.5), (5, 7, 7, 16, 3.0),
                                           (4, 3, 9, 300, 0.5)])
def test_blocked_solve_parity(dev, m, n, V, S, alpha):
    """Blocked warp-per-tensor kernel (schedule 5) vs the oracle: m = 2 (empty prefix) and m = 3
    (prefix = x), a compiled shape forced onto it, larger shapes ((4,10): U = 715, (6,6): U = 462),
    S < 32 (a tensor cannot fill the warp), S > 256 and ragged tensor counts (buffer hand-over)."""
    ent = syn.gen_voxels(m, n, 0, V, 5) if m % 2 == 0 else syn.gen_uniform_tensors(m, n, V, 5)
    st = syn.gen_starts(S, n, 4)
    gpu = _solve(dev, m, n, ent, st, alpha, 1e-6, 300, schedule=5)
    _assert_parity(PR.solve_parity(ent, st, m, n, alpha, 1e-6, 300, gpu), 1e-3 if m % 2 == 0 else 0.05)


@pytest.mark.parametrize("shift", ["auto_max", "auto_min", "per_tensor"])
def test_blocked_shift_modes_match_item_kernel(dev, shift):
    """Blocked kernel with per-tensor and automatic shifts: fixed-K (tol < 0) lambda_K agrees with the
    item-per-lane general kernel (same arithmetic, same shift) and iteration counts are exact."""
    m, n, V, S = 5, 4, 37, 100
    ent = syn.gen_uniform_tensors(m, n, V, 13)
    st = syn.gen_starts(S, n, 6)
    alpha = shift
    if shift == "per_tensor":   # alternating convex / concave shifts of the R17 bound: contractive runs
        from oracle import sshopm as OR
        sgn = np.where(np.arange(V) % 2 == 0, 1.0, -1.0)
        alpha = torch.from_numpy((sgn * OR.convexity_shift(ent, m, n)).astype(np.float32)).to(dev)
    a = _solve(dev, m, n, ent, st, alpha, -1.0, 40, schedule=5)
    b = _solve(dev, m, n, ent, st, alpha, -1.0, 40, schedule=3)
    assert np.all(a[2] == 40) and np.all(b[2] == 40) and not a[3].any()
    assert np.all(np.abs(a[0] - b[0]) <= 1e-4 * np.maximum(1, np.abs(b[0])))


def test_blocked_total_iters_and_tiny(dev):
    """Blocked kernel: the device iteration counter equals sum(iters); V = 1 and S = 1 work."""
    m, n = 6, 6
    for V, S in [(1, 1), (1, 40), (3, 1)]:
        ent = syn.gen_voxels(m, n, 0, V, 8)
        st = syn.gen_starts(S, n, 9)
        s = sh.Solver(m, n)
        ti = torch.zeros(1, dtype=torch.int64, device=dev)
        lam, x, it, cv = s.solve(torch.from_numpy(ent).to(dev), torch.from_numpy(st).to(dev), 0.5, 1e-6, 300,
                                 schedule=5, total_iters=ti)
        torch.cuda.synchronize()
        assert int(ti.item()) == int(it.sum().item())
        rl, rx, ri, rc = O.sshopm(ent, st, m, n, 0.5, 1e-6, 300)
        both = (cv.cpu().numpy() == 1) & rc
        assert np.all(np.abs(lam.cpu().numpy()[both] - rl[both]) <= 1e-4 * np.maximum(1, np.abs(rl[both])))


# ------------------------------------------------------------ classification --
@pytest.mark.parametrize("m,n,alpha", [(4, 3, 0.0), (6, 3, 0.25), (4, 6, 0.0), (3, 3, 1.0), (4, 3, -0.5), (8, 3, 0.5)])
def test_classify_matches_oracle(dev, m, n, alpha):
    """Reading R18 types of the GPU's dedup records == oracle types of the same records (FP64),
    except records whose oracle margin min|mu| is within a factor 10 of ctol (borderline)."""
    from oracle import classify as OC
    V = 96 if m <= 6 else 24
    ent = syn.gen_voxels(m, n, 300, V, 5) if m % 2 == 0 else syn.gen_uniform_tensors(m, n, V, 5)
    st = syn.gen_starts(128, n, 0)
    s = sh.Solver(m, n)
    e = torch.from_numpy(ent).to(dev)
    lam, x, it, cv = s.solve(e, torch.from_numpy(st).to(dev), alpha, 1e-7, 500)
    cnt, cl, cx, mu, rp = s.dedup(lam, x, cv, 1e-2, 0.05, 6)
    ctol = 1e-3
    ty = s.classify(e, cnt, cl, cx, ctol).cpu().numpy()
    ot, margin = OC.classify(ent, m, n, cnt.cpu().numpy(), cl.cpu().numpy().astype(np.float64),
                             cx.cpu().numpy().astype(np.float64), ctol)
    border = (margin > ctol / 10) & (margin < ctol * 10)
    diff = (ty != ot) & ~border
    assert not diff.any(), (np.argwhere(diff)[:5], ty[diff][:5], ot[diff][:5])
    assert set(np.unique(ty)) <= {-1, 0, 1, 2, 3}


def test_classify_convex_shift_gives_maxima(dev):
    """With the automatic convex shift lambda_k only increases, so no local minimum is ever reported; the
    lambda-stopping rule can stop on the slow ascent past a saddle, so saddles are rare but possible."""
    m, n = 4, 3
    ent = syn.gen_voxels(m, n, 0, 64, 1)
    s = sh.Solver(m, n)
    e = torch.from_numpy(ent).to(dev)
    lam, x, it, cv = s.solve(e, torch.from_numpy(syn.gen_starts(64, n, 0)).to(dev), "auto_max", 1e-9, 20000)
    cnt, cl, cx, mu, rp = s.dedup(lam, x, cv, 1e-2, 0.05, 8)
    ty = s.classify(e, cnt, cl, cx, 1e-3).cpu().numpy()
    filled = ty != 3
    assert filled.any()
    assert not (ty == -1).any()
    assert np.mean(np.isin(ty[filled], (1, 2))) >= 0.9


# ------------------------------------------------ records path (schedule 8) --
def _records(dev, m, n, ent, st, alpha, tol, maxit, lt, at, kmax, **kw):
    s = sh.Solver(m, n)
    e, t = torch.from_numpy(ent).to(dev), torch.from_numpy(st).to(dev)
    tot = torch.zeros(1, dtype=torch.int64, device=dev)
    raw, dd = s.solve_dedup(e, t, alpha, tol, maxit, lt, at, kmax, records=True, total_iters=tot, **kw)
    torch.cuda.synchronize()
    assert raw is None
    return [x.cpu().numpy() for x in dd], int(tot.item())


@pytest.mark.parametrize("m,n,V,S,alpha,kmax,unit", [(4, 3, 3000, 128, 0.0, 4, 0), (4, 3, 777, 100, 0.0, 8, 7),
                                                     (6, 3, 500, 128, 0.25, 6, 32), (3, 3, 400, 64, 1.0, 5, 1),
                                                     (4, 6, 200, 128, 0.0, 4, 0), (8, 3, 100, 32, 0.5, 3, 5),
                                                     (4, 3, 50, 300, 0.0, 4, 64), (4, 3, 70, 128, -0.5, 4, 200),
                                                     (3, 2, 33, 1, 0.0, 2, 0), (4, 3, 1, 128, 0.0, 4, 3)])
def test_records_path_equals_two_pass(dev, m, n, V, S, alpha, kmax, unit):
    """sshopm_solve_dedup on the records path (fuse_dedup = 4: lane-owned units, 16-byte per-start records,
    dedup reading the records) == sshopm_solve + sshopm_dedup, bit for bit, and the same iteration total."""
    ent = syn.gen_voxels(m, n, 900, V, 1) if m % 2 == 0 else syn.gen_uniform_tensors(m, n, V, 1)
    st = syn.gen_starts(S, n, 3)
    s = sh.Solver(m, n)
    e, t = torch.from_numpy(ent).to(dev), torch.from_numpy(st).to(dev)
    tot = torch.zeros(1, dtype=torch.int64, device=dev)
    raw = s.solve(e, t, alpha, 1e-6, 100, total_iters=tot)
    da = [x.cpu().numpy() for x in s.dedup(raw[0], raw[1], raw[3], 1e-2, 0.05, kmax)]
    db, its = _records(dev, m, n, ent, st, alpha, 1e-6, 100, 1e-2, 0.05, kmax, unit_starts=unit)
    for a, b in zip(da, db):
        assert np.array_equal(a, b)
    assert its == int(tot.item())


@pytest.mark.parametrize("mode", ["per_tensor", "auto_max", "auto_min"])
def test_records_path_shift_modes(dev, mode):
    """Per-tensor and automatic shifts on the records path equal the two-pass path bit for bit."""
    m, n, V, S = 4, 3, 300, 128
    ent = syn.gen_voxels(m, n, 50, V, 2)
    st = syn.gen_starts(S, n, 4)
    e, t = torch.from_numpy(ent).to(dev), torch.from_numpy(st).to(dev)
    alpha = (torch.linspace(-1.0, 1.0, V, device=dev, dtype=torch.float32) if mode == "per_tensor" else mode)
    s = sh.Solver(m, n)
    raw = s.solve(e, t, alpha, 1e-6, 100)
    da = [x.cpu().numpy() for x in s.dedup(raw[0], raw[1], raw[3], 1e-2, 0.05, 4)]
    _, db = s.solve_dedup(e, t, alpha, 1e-6, 100, 1e-2, 0.05, 4, records=True)
    for a, b in zip(da, [x.cpu().numpy() for x in db]):
        assert np.array_equal(a, b)


def test_records_path_vs_oracle(dev):
    """The records path against the FP64 oracle: on voxels whose converged flags all agree with the oracle's,
    cluster counts, representatives and multiplicities equal oracle solve + oracle R16 dedup, and the
    representative lambdas agree within the parity tolerance."""
    m, n, V, S = 4, 3, 400, 128
    ent = syn.gen_voxels(m, n, 1234, V, 5)
    st = syn.gen_starts(S, n, 6)
    (cnt, clam, cx, mult, rep), _ = _records(dev, m, n, ent, st, 0.0, 1e-6, 100, 1e-2, 0.05, 8)
    olam, ox, oit, oconv = O.sshopm(ent, st, m, n, 0.0, 1e-6, 100)
    gpu = _solve(dev, m, n, ent, st, 0.0, 1e-6, 100)
    ocnt, olo, oxo, omo, oro = D.dedup(olam, ox, oconv, m, 1e-2, 0.05, 8)
    same = (gpu[3].astype(bool) == oconv.astype(bool)).all(axis=1)
    assert same.mean() > 0.95
    assert np.array_equal(cnt[same], ocnt[same])
    assert np.array_equal(mult[same], omo[same])
    assert np.array_equal(rep[same], oro[same])
    np.testing.assert_allclose(clam[same], olo[same], rtol=1e-4, atol=1e-4)


@pytest.mark.parametrize("m,n,V,S,alpha", [(4, 3, 64, 128, 0.0), (4, 3, 50, 100, 0.5), (6, 3, 20, 77, 0.25),
                                           (3, 3, 9, 33, -1.0)])
def test_small_problem_item_chunks(dev, m, n, V, S, alpha):
    """Small problems (fewer whole-tensor chunks than resident warps) run schedule 1 with chunks of items
    (parts of tensors): results bit for bit those of schedule 2 (tensor per lane) and of the lean schedule,
    including a non-power-of-two S (item -> tensor by division) and per-tensor shifts."""
    ent = syn.gen_voxels(m, n, 77, V, 4) if m % 2 == 0 else syn.gen_uniform_tensors(m, n, V, 4)
    st = syn.gen_starts(S, n, 5)
    a = _solve(dev, m, n, ent, st, alpha, 1e-6, 100)
    b = _solve(dev, m, n, ent, st, alpha, 1e-6, 100, schedule=2)
    c = _solve(dev, m, n, ent, st, alpha, 1e-6, 100, schedule=6)
    for x, y, z in zip(a, b, c):
        assert np.array_equal(x, y) and np.array_equal(x, z)
    per = torch.linspace(-0.5, 0.5, V, device=dev, dtype=torch.float32)
    s = sh.Solver(m, n)
    e, t = torch.from_numpy(ent).to(dev), torch.from_numpy(st).to(dev)
    p1 = [x.cpu().numpy() for x in s.solve(e, t, per, 1e-6, 100)]
    p6 = [x.cpu().numpy() for x in s.solve(e, t, per, 1e-6, 100, schedule=6)]
    for x, y in zip(p1, p6):
        assert np.array_equal(x, y)
