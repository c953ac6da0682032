"""Starting vectors: deterministic evenly spaced sets cover the sphere."""
import numpy as np
import pytest

from paper_conf_ipps_ballardkp11_b200 import starts as ST


@pytest.mark.parametrize("n", [2, 3, 4, 6])
@pytest.mark.parametrize("half", [False, True])
def test_evenly_spaced_unit_and_deterministic(n, half):
    a = ST.evenly_spaced(128, n, half)
    assert a.shape == (128, n) and a.dtype == np.float32
    assert np.allclose(np.linalg.norm(a, axis=1), 1.0, atol=1e-6)
    assert np.array_equal(a, ST.evenly_spaced(128, n, half))
    if half:
        assert (a[:, -1] >= -1e-7).all()


def test_fibonacci_covers_sphere_better_than_random():
    """Covering radius (max over a dense probe set of the angle to the nearest start), n = 3, S = 128."""
    rng = np.random.default_rng(0)
    probe = rng.standard_normal((20000, 3))
    probe /= np.linalg.norm(probe, axis=1, keepdims=True)

    def cover(P):
        return np.arccos(np.clip((probe @ P.T).max(axis=1), -1, 1)).max()

    fib = ST.evenly_spaced(128, 3).astype(np.float64)
    rnd = ST.uniform_cube(128, 3, 0).astype(np.float64)
    rnd /= np.linalg.norm(rnd, axis=1, keepdims=True)
    assert cover(fib) < 0.75 * cover(rnd)
    assert cover(fib) < 0.3            # below sqrt(4 pi / 128) = 0.31


def test_hemisphere_covers_projective_plane():
    """Even m: x ~ -x, so a hemisphere set covers the sphere modulo sign."""
    rng = np.random.default_rng(1)
    probe = rng.standard_normal((20000, 3))
    probe /= np.linalg.norm(probe, axis=1, keepdims=True)
    h = ST.evenly_spaced(64, 3, half=True).astype(np.float64)
    assert np.arccos(np.clip(np.abs(probe @ h.T).max(axis=1), -1, 1)).max() < 0.25
