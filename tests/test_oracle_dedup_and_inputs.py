"""Pins for oracle/dedup.py (reading R16) and the synthetic input module.

Dedup is checked against hand-built cases whose clustering is obvious by
construction (angles and lambda gaps far from or exactly across the
thresholds), closed-form angles, and the paper's sign convention for even m.
The generator is pinned by closed forms: v^{(x)m} x^m = (v.x)^m and
E_m x^m = ||x||^m evaluated with the oracle's full-tensor Eq. 3.
"""
import numpy as np
import pytest

from oracle import dedup as D
from oracle import sshopm as O
import synthetic as syn


def _unit(v):
    v = np.asarray(v, float)
    return v / np.linalg.norm(v)


def test_angle_closed_forms():
    assert D.angle([1, 0, 0], [1, 0, 0]) == 0.0
    assert np.isclose(D.angle([1, 0, 0], [0, 1, 0]), np.pi / 2)
    assert np.isclose(D.angle([1, 0, 0], [-1, 0, 0]), np.pi)
    t = 1e-7
    assert np.isclose(D.angle([1, 0, 0], [np.cos(t), np.sin(t), 0]), t, rtol=1e-9)


def _rot(v, t):
    """Rotate unit v by angle t in the plane of v and a fixed orthogonal direction."""
    v = _unit(v)
    w = np.cross(v, [0.3, 0.5, 0.8])
    w = _unit(w)
    return np.cos(t) * v + np.sin(t) * w


def test_dedup_hand_built():
    m = 4
    a = _unit([1, 2, 3])
    b = _unit([3, -1, 0.5])
    lam = np.array([[1.0, 1.001, 0.5, 1.0, 0.9, 1.0, 0.5, 2.0]])
    x = np.array([[a, _rot(a, 0.01), b, -a, a, _rot(a, 0.2), -b, b]])
    conv = np.array([[1, 1, 1, 1, 1, 1, 1, 0]], bool)
    count, lo, xo, mo, ro = D.dedup(lam, x, conv, m, 1e-2, 0.05, 8)
    # clusters in creation order: {0,1,3} (sign-free, small angle), {2,6}, {4} (lam gap 0.1), {5} (angle 0.2)
    assert count[0] == 4
    # sorted by lambda desc, ties by representative start
    assert list(ro[0, :4]) == [0, 5, 4, 2]
    assert list(mo[0, :4]) == [3, 1, 1, 2]
    assert list(lo[0, :4]) == [1.0, 1.0, 0.9, 0.5]
    assert (ro[0, 4:] == -1).all() and (mo[0, 4:] == 0).all()
    # kmax overflow: count still reports all clusters
    count2, lo2, xo2, mo2, ro2 = D.dedup(lam, x, conv, m, 1e-2, 0.05, 2)
    assert count2[0] == 4 and list(ro2[0]) == [0, 5]


def test_dedup_odd_m_pairs_negated():
    """R15/R16: for odd m, (lam, x) and (-lam, -x) are the same eigenpair."""
    a = _unit([1, 1, 0])
    lam = np.array([[0.7, -0.7, 0.7]])
    x = np.array([[a, -a, -a]])
    conv = np.ones((1, 3), bool)
    count, lo, xo, mo, ro = D.dedup(lam, x, conv, 3, 1e-3, 1e-3, 4)
    assert count[0] == 2 and list(mo[0, :2]) == [2, 1]


def test_dedup_none_converged():
    lam = np.zeros((2, 4))
    x = np.zeros((2, 4, 3))
    conv = np.zeros((2, 4), bool)
    count, lo, xo, mo, ro = D.dedup(lam, x, conv, 4, 1e-2, 0.05, 3)
    assert (count == 0).all() and (ro == -1).all()


@pytest.mark.parametrize("m,n", [(4, 3), (6, 3), (8, 3), (4, 6)])
def test_generator_closed_forms(m, n):
    rng = np.random.default_rng(0)
    v = rng.standard_normal((5, n))
    v /= np.linalg.norm(v, axis=1, keepdims=True)
    x = rng.standard_normal((5, n))
    full = O.expand_full(syn.rank1_entries(v, m), m, n)
    assert np.allclose(O.axm(full, x), np.sum(v * x, axis=1) ** m)
    E = O.expand_full(syn.isotropic_entries(m, n)[None], m, n)
    assert np.allclose(O.axm(np.repeat(E, 5, 0), x), np.linalg.norm(x, axis=1) ** m)


def test_generator_shard_invariant_and_seeded():
    m, n = 4, 3
    whole = syn.gen_voxels(m, n, 65536 - 100, 300, seed=3)
    a = syn.gen_voxels(m, n, 65536 - 100, 150, seed=3)
    b = syn.gen_voxels(m, n, 65536 + 50, 150, seed=3)
    assert np.array_equal(whole, np.concatenate([a, b]))
    assert whole.dtype == np.float32 and whole.shape == (300, 15)
    assert not np.array_equal(whole, syn.gen_voxels(m, n, 65536 - 100, 300, seed=4))
    s = syn.gen_starts(128, 3, 0)
    assert s.dtype == np.float32 and s.shape == (128, 3)
    assert np.array_equal(s, syn.gen_starts(128, 3, 0))
    assert np.abs(s).max() <= 1.0


def test_generator_workload_shape():
    """Recipe: the dominant eigenvalue is ~1 (+ isotropic c <= 0.25 + noise), tensors are mostly positive."""
    m, n = 4, 3
    e = syn.gen_voxels(m, n, 0, 64, seed=0)
    lam, x, it, cv = O.sshopm(e, syn.gen_starts(64, n, 0), m, n, 0.0, 1e-8, 500)
    best = np.array([lam[v][cv[v]].max() for v in range(64)])
    assert (best > 0.7).all() and (best < 1.6).all()
