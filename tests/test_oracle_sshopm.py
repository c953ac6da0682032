"""Pins for oracle/sshopm.py (Fig. 1 SS-HOPM, FP64 full tensor).

Each test ties the oracle to something other than itself: a library
eigensolver (m = 2 is the matrix power method), closed forms
(rank-1 tensors), an external worked example re-validated by residual, the
Kolda-Mayo monotonicity theorem, a brute-force sphere grid, and the
stopping-rule special cases of the DESIGN.md readings.
"""
import json
import os

import numpy as np
import pytest

from oracle import sshopm as O
from oracle import dedup as D
import synthetic as syn


def _full(entries, m, n):
    return O.expand_full(entries, m, n)


def _run(entries, starts, m, n, alpha, tol, maxit, **kw):
    return O.sshopm(np.asarray(entries, np.float64), np.asarray(starts, np.float64), m, n, alpha, tol, maxit, **kw)


def _matrix_entries(M):
    """Compressed entries (lexicographic) of a symmetric n x n matrix: a_ij for i <= j."""
    n = M.shape[0]
    return np.array([M[i, j] for i in range(n) for j in range(i, n)])


def test_m2_is_matrix_power_method_max():
    """m = 2, alpha = ||A||_2: SS-HOPM converges to lambda_max (numpy.linalg.eigh)."""
    rng = np.random.default_rng(7)
    for trial in range(40):
        n = 3 if trial < 30 else 5
        B = rng.standard_normal((n, n))
        M = (B + B.T) / 2
        w, V = np.linalg.eigh(M)
        if w[-1] - w[-2] < 0.05:
            continue
        alpha = np.linalg.norm(M, 2)
        starts = rng.uniform(-1, 1, size=(8, n))
        lam, x, it, cv = _run(_matrix_entries(M)[None], starts, 2, n, alpha, 1e-15, 20000)
        assert cv.all()
        assert np.allclose(lam, w[-1], atol=1e-10)
        assert np.allclose(np.abs(x[0] @ V[:, -1]), 1.0, atol=1e-6)


def test_m2_negative_shift_finds_min():
    """Fig. 1 line 5 (alpha < 0 branch): m = 2 converges to lambda_min."""
    rng = np.random.default_rng(8)
    for _ in range(30):
        B = rng.standard_normal((3, 3))
        M = (B + B.T) / 2
        w, V = np.linalg.eigh(M)
        if w[1] - w[0] < 0.05:
            continue
        alpha = -np.linalg.norm(M, 2)
        lam, x, it, cv = _run(_matrix_entries(M)[None], rng.uniform(-1, 1, (8, 3)), 2, 3, alpha, 1e-15, 20000)
        assert cv.all()
        assert np.allclose(lam, w[0], atol=1e-10)


@pytest.mark.parametrize("m", [4, 6, 8])
def test_rank1_exact_two_updates(m):
    """A = lam v^{(x)m} (m even), alpha = 0: x_1 = +-v, lam_1 = lam, stop at iters = 2."""
    n = 3
    rng = np.random.default_rng(m)
    for _ in range(5):
        v = rng.standard_normal(n)
        v /= np.linalg.norm(v)
        lam_true = rng.uniform(0.5, 2.0)
        ent = lam_true * syn.rank1_entries(v[None], m)
        starts = rng.uniform(-1, 1, (64, n))
        # well-conditioned starts only: (v.x0)^{m-1} must not be lost to cancellation
        starts = starts[np.abs(starts @ v) / np.linalg.norm(starts, axis=1) > 0.3][:16]
        lam, x, it, cv = _run(ent, starts, m, n, 0.0, 1e-12, 100)
        assert cv.all()
        assert (it == 2).all()
        assert np.allclose(lam, lam_true, rtol=1e-12)
        assert np.allclose(np.abs(x[0] @ v), 1.0, atol=1e-12)


def _kr(golden_dir):
    with open(os.path.join(golden_dir, "kolda_mayo_kr_example.json")) as f:
        return json.load(f)


def test_kr_example_residuals(golden_dir):
    """External example (Kolda-Mayo [1]): quoted pairs are eigenpairs to 4-digit rounding."""
    d = _kr(golden_dir)
    full = _full(np.array(d["entries"])[None], 4, 3)
    for lam, x in d["maxima_alpha_pos"] + d["minima_alpha_neg"]:
        x = np.array(x) / np.linalg.norm(x)
        r = O.residual(full, np.array([lam]), x[None])[0]
        assert r < 1e-3


@pytest.mark.parametrize("alpha,key", [(2.0, "maxima_alpha_pos"), (-2.0, "minima_alpha_neg")])
def test_kr_example_sshopm_finds_all(golden_dir, alpha, key):
    """SS-HOPM from 256 starts at alpha = +-2 finds exactly the quoted lambdas (4 digits)."""
    d = _kr(golden_dir)
    ent = np.array(d["entries"])[None]
    starts = syn.gen_starts(256, 3, seed=11)
    lam, x, it, cv = _run(ent, starts, 4, 3, alpha, 1e-14, 5000)
    assert cv.mean() > 0.99
    found = sorted(set(np.round(lam[0][cv[0]], 4)))
    expect = sorted(l for l, _ in d[key])
    assert np.allclose(found, expect, atol=1.5e-4), (found, expect)
    full = _full(ent, 4, 3)
    res = O.residual(np.repeat(full, 256, 0)[cv[0]], lam[0][cv[0]], x[0][cv[0]])
    assert res.max() < 1e-6
    # eigenvectors match the quoted ones up to sign (m even)
    for l, v in d[key]:
        sel = np.abs(lam[0] - l) < 1e-3
        v = np.array(v) / np.linalg.norm(v)
        assert np.allclose(np.abs(x[0][sel] @ v), 1.0, atol=2e-4)


def test_kr_alpha0_not_monotone(golden_dir):
    """alpha = 0 on the KR tensor is the classic S-HOPM failure: lambda is not monotone."""
    d = _kr(golden_dir)
    full = _full(np.array(d["entries"])[None], 4, 3)
    x0 = O.normalise_starts(syn.gen_starts(64, 3, seed=3))
    tr = []
    O.sshopm_lanes(lambda idx: full[np.zeros(len(idx), int)], x0, 0.0, -1.0, 20, trace=tr)
    lam_hist = np.full((21, 64), np.nan)
    for k, ids, ln, _ in tr:
        lam_hist[k, ids] = ln
    dec = np.nanmin(np.diff(lam_hist[1:], axis=0), axis=0)
    assert (dec < -1e-6).sum() > 32


@pytest.mark.parametrize("m,n", [(4, 3), (6, 3), (4, 4)])
def test_monotone_above_convexity_bound(m, n):
    """Kolda-Mayo theorem: alpha > beta(A) (bound (m-1) sum|a|) -> lam_k nondecreasing."""
    ent = syn.gen_uniform_tensors(m, n, 3, seed=m + n).astype(np.float64)
    for v in range(3):
        full = _full(ent[v:v + 1], m, n)
        alpha = (m - 1) * np.abs(full).sum()
        x0 = O.normalise_starts(syn.gen_starts(32, n, seed=v))
        lam0 = O.axm(np.repeat(full, 32, 0), x0)
        tr = []
        O.sshopm_lanes(lambda idx: full[np.zeros(len(idx), int)], x0, alpha, -1.0, 30, trace=tr)
        prev = lam0.copy()
        for k, ids, ln, _ in tr:
            assert np.all(ln >= prev[ids] - 1e-12 * np.maximum(1, np.abs(ln)))
            prev[ids] = ln


def _fib_sphere(N):
    i = np.arange(N) + 0.5
    phi = np.arccos(1 - 2 * i / N)
    th = np.pi * (1 + 5 ** 0.5) * i
    return np.stack([np.cos(th) * np.sin(phi), np.sin(th) * np.sin(phi), np.cos(phi)], 1)


def test_global_max_matches_sphere_grid():
    """alpha >= 0 finds maxima: best converged lambda equals the sphere-grid max of A x^m."""
    m, n = 4, 3
    ent = syn.gen_voxels(m, n, 0, 6, seed=5)
    grid = _fib_sphere(100000)
    lam, x, it, cv = _run(ent, syn.gen_starts(128, n, 1), m, n, 0.0, 1e-12, 1000)
    for v in range(6):
        full = _full(ent[v:v + 1], m, n)
        gmax = O.axm(np.broadcast_to(full, (len(grid),) + full.shape[1:]), grid).max()
        best = lam[v][cv[v]].max()
        assert best >= gmax - 1e-4
        assert best <= gmax + 1e-4


def test_unit_norm_and_residual_tight_tol():
    """||x|| = 1 on every output; residual <= 1e-6 when run to tol 1e-15 (Eq. 2)."""
    m, n = 4, 3
    ent = syn.gen_voxels(m, n, 100, 8, seed=0)
    lam, x, it, cv = _run(ent, syn.gen_starts(64, n, 0), m, n, 0.0, 1e-15, 10000)
    assert np.allclose(np.linalg.norm(x, axis=2), 1.0, atol=1e-14)
    full = np.repeat(_full(ent, m, n), 64, 0)
    r = O.residual(full, lam.reshape(-1), x.reshape(-1, n))
    assert r[cv.reshape(-1)].max() < 1e-6
    assert cv.mean() > 0.99


def test_residual_at_default_tol_is_small():
    """At tol = 1e-6 (R2), the stop leaves a residual ~sqrt(tol): <= 0.05."""
    m, n = 4, 3
    ent = syn.gen_voxels(m, n, 0, 32, seed=0)
    lam, x, it, cv = _run(ent, syn.gen_starts(128, n, 0), m, n, 0.0, 1e-6, 100)
    full = np.repeat(_full(ent, m, n), 128, 0)
    r = O.residual(full, lam.reshape(-1), x.reshape(-1, n))
    assert r[cv.reshape(-1)].max() < 0.05


def test_stopping_special_cases():
    """Readings R2/R6: maxit = 0, fixed-K (tol < 0), zero start."""
    m, n = 4, 3
    ent = syn.gen_voxels(m, n, 0, 2, seed=0).astype(np.float64)
    starts = syn.gen_starts(8, n, 0).astype(np.float64)
    starts[3] = 0.0
    full = _full(ent, m, n)
    x0 = O.normalise_starts(starts)
    # maxit = 0 -> (lam_0, x_0), iters 0, not converged
    lam, x, it, cv = _run(ent, starts, m, n, 0.0, 1e-6, 0)
    assert (it == 0).all() and not cv.any()
    assert np.allclose(x[0], x0)
    assert np.allclose(lam[1], O.axm(np.repeat(full[1:2], 8, 0), x0))
    # fixed-K: exactly K updates, converged = 0 (except zero start)
    lam, x, it, cv = _run(ent, starts, m, n, 0.0, -1.0, 7)
    assert not cv.any()
    assert (np.delete(it, 3, axis=1) == 7).all()
    # zero start -> lam = 0, x = 0, iters = 0
    assert (it[:, 3] == 0).all() and (lam[:, 3] == 0).all() and (x[:, 3] == 0).all()


def test_fixed_k_prefix_property():
    """Running K updates then reading x_K equals the K-th iterate of a longer run (trajectory alignment)."""
    m, n = 4, 3
    ent = syn.gen_voxels(m, n, 0, 4, seed=0)
    starts = syn.gen_starts(16, n, 0)
    lamA, xA, itA, _ = _run(ent, starts, m, n, 0.0, 1e-6, 100)
    lamB, xB, itB, _ = _run(ent, starts, m, n, 0.0, -1.0, 100, lane_maxit=itA)
    assert np.array_equal(itA, itB)
    assert np.array_equal(lamA, lamB) and np.array_equal(xA, xB)


def test_even_m_sign_symmetry():
    """m even: A(-x)^{m-1} = -(A x^{m-1}) and A(-x)^m = A x^m, so (lam, x) ~ (lam, -x)."""
    m, n = 4, 3
    ent = syn.gen_voxels(m, n, 0, 4, 0)
    full = _full(ent, m, n)
    xs = O.normalise_starts(syn.gen_starts(4, n, 2))
    assert np.allclose(O.axm(full, -xs), O.axm(full, xs))
    assert np.allclose(O.axm1(full, -xs), -O.axm1(full, xs))


def test_cluster_count_bound():
    """at most ((m-1)^n - 1)/(m-2) distinct eigenpairs -> dedup count is bounded."""
    m, n = 4, 3
    bound = ((m - 1) ** n - 1) // (m - 2)
    ent = syn.gen_voxels(m, n, 0, 64, seed=0)
    lam, x, it, cv = _run(ent, syn.gen_starts(128, n, 0), m, n, 0.0, 1e-10, 2000)
    count, *_ = D.dedup(lam, x, cv, m, 1e-3, 1e-2, 8)
    assert count.max() <= bound
    assert count.min() >= 1


def test_paper_flops_reading_r12():
    """R12 (parity unpinned): F(4,3) = 6*15 + 5*30 + 15 = 255."""
    assert O.paper_flops_per_iter(4, 3) == 255
    assert O.paper_flops_per_iter(6, 3) == 680


def test_per_voxel_alpha_equals_scalar_runs():
    """A per-voxel shift array gives exactly the per-voxel scalar runs (incl. mixed signs)."""
    m, n = 4, 3
    ent = syn.gen_voxels(m, n, 0, 6, seed=2)
    st = syn.gen_starts(32, n, 1)
    alphas = np.array([0.0, 0.5, -0.5, 2.0, -2.0, 0.25])
    lam, x, it, cv = _run(ent, st, m, n, alphas, 1e-8, 200)
    for v in range(6):
        l1, x1, i1, c1 = _run(ent[v:v + 1], st, m, n, float(alphas[v]), 1e-8, 200)
        assert np.array_equal(lam[v], l1[0]) and np.array_equal(x[v], x1[0]) and np.array_equal(it[v], i1[0])


def test_convexity_shift_bound_and_monotone():
    """R17 shift: brute-force sum over all n^m entries; lambda_k nondecreasing (+) / nonincreasing (-)."""
    m, n = 4, 3
    ent = syn.gen_uniform_tensors(m, n, 4, seed=5).astype(np.float64)
    b = O.convexity_shift(ent, m, n)
    full = O.expand_full(ent, m, n)
    for v in range(4):
        import itertools
        tot = sum(abs(full[v][t]) for t in itertools.product(range(n), repeat=m))
        assert np.isclose(b[v], (m - 1) * tot)
    for sign in (1, -1):
        x0 = O.normalise_starts(syn.gen_starts(16, n, 3))
        fl = full[0:1]
        lam0 = O.axm(np.repeat(fl, 16, 0), x0)
        tr = []
        O.sshopm_lanes(lambda idx: fl[np.zeros(len(idx), int)], x0, sign * b[0], -1.0, 25, trace=tr)
        prev = lam0.copy()
        for k, ids, ln, _ in tr:
            assert np.all(sign * (ln - prev[ids]) >= -1e-12)
            prev[ids] = ln
