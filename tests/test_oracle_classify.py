"""Pins for oracle/classify.py (eigenpair types, reading R18)."""
import numpy as np
import pytest

from oracle import classify as C
from oracle import sshopm as O
import synthetic as syn


def _matrix_entries(M):
    n = M.shape[0]
    return np.array([M[i, j] for i in range(n) for j in range(i, n)])


def test_m2_types_from_eigh():
    """m = 2: on the sphere x'Mx has its max at the top eigenvector, min at the bottom, saddles between."""
    rng = np.random.default_rng(0)
    for n in (3, 4, 5):
        B = rng.standard_normal((n, n))
        M = (B + B.T) / 2
        w, V = np.linalg.eigh(M)
        full = O.expand_full(_matrix_entries(M)[None], 2, n)[0]
        assert C.classify_one(full, w[-1], V[:, -1], 1e-9)[0] == C.MAX
        assert C.classify_one(full, w[0], V[:, 0], 1e-9)[0] == C.MIN
        for i in range(1, n - 1):
            assert C.classify_one(full, w[i], V[:, i], 1e-9)[0] == C.SADDLE
        # C's eigenvalues are exactly w_j - w_i (m - 1 = 1)
        mu = np.sort(C.classify_one(full, w[-1], V[:, -1], 1e-9)[1])
        assert np.allclose(mu, np.sort(w[:-1] - w[-1]))


@pytest.mark.parametrize("m", [4, 6])
def test_rank1_top_is_max(m):
    rng = np.random.default_rng(m)
    v = rng.standard_normal(3)
    v /= np.linalg.norm(v)
    full = O.expand_full(2.0 * syn.rank1_entries(v[None], m), m, 3)[0]
    t, mu = C.classify_one(full, 2.0, v, 1e-6)
    assert t == C.MAX
    assert np.allclose(mu, -2.0 * np.ones(2))          # (m-1) A v^{m-2} - lam I on v-perp = -lam


def test_types_agree_with_sphere_grid():
    """A pair typed MAX is a local maximum of A x^m over a cap of the sphere; MIN a local minimum."""
    m, n = 4, 3
    ent = syn.gen_uniform_tensors(m, n, 3, 4)
    full = O.expand_full(ent, m, n)
    st = syn.gen_starts(64, n, 1)
    for v in range(3):
        for sign in (1, -1):
            a = sign * O.convexity_shift(ent[v:v + 1], m, n)[0]
            lam, x, it, cv = O.sshopm(ent[v:v + 1], st, m, n, a, 1e-13, 20000)
            rng = np.random.default_rng(v)
            for s in np.nonzero(cv[0])[0][:8]:
                t, _ = C.classify_one(full[v], lam[0, s], x[0, s], 1e-6)
                if t == C.DEGENERATE:
                    continue
                assert t == (C.MAX if sign > 0 else C.MIN)    # convex shift -> local maxima (Kolda-Mayo)
                p = x[0, s] + 0.02 * rng.standard_normal((200, n))
                p /= np.linalg.norm(p, axis=1, keepdims=True)
                f = O.axm(np.repeat(full[v:v + 1], 200, 0), p)
                if t == C.MAX:
                    assert np.all(f <= lam[0, s] + 1e-9)
                else:
                    assert np.all(f >= lam[0, s] - 1e-9)


def test_kr_example_types(golden_dir):
    import json, os
    d = json.load(open(os.path.join(golden_dir, "kolda_mayo_kr_example.json")))
    full = O.expand_full(np.array(d["entries"])[None], 4, 3)[0]
    st = syn.gen_starts(256, 3, seed=11)
    for alpha, want in ((2.0, C.MAX), (-2.0, C.MIN)):
        lam, x, it, cv = O.sshopm(np.array(d["entries"])[None], st, 4, 3, alpha, 1e-14, 5000)
        for s in np.nonzero(cv[0])[0]:
            assert C.classify_one(full, lam[0, s], x[0, s], 1e-6)[0] == want
