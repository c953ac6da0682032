"""Seeded synthetic inputs shared by the oracle tests and the CUDA path.

Holds none of SS-HOPM's arithmetic: it only draws random numbers and writes
symmetric tensors in the boundary's storage format (one value per index
class, classes in the paper's lexicographic order, P:L87 / Table I — the
class list here comes from ``itertools.combinations_with_replacement``).

Workload recipe (stands in for the unavailable SCI-Utah set, P:L313-315;
DESIGN.md "Input recipe"):

    A = v1^{(x)m} + [F == 2] * w2 * v2^{(x)m} + c * E_m + eps * N

* F in {1, 2} equiprobable ("some with one and some with two principal fiber
  directions"); v1 uniform on S^{n-1}; v2 at a crossing angle
  ~ U[45, 90] degrees from v1 in a random plane; w2 ~ U[0.5, 1];
* c ~ U[0, 0.25] and E_m the symmetric tensor with E_m x^m = ||x||^m
  (entry of class k = 2q: (m/2)! prod k_i! / (prod q_i! m!), 0 if any k_i odd);
* eps = 0.02, N's unique entries i.i.d. N(0, 1);
* everything drawn in float64, stored as float32.

Counter-based: voxels are generated in blocks of 65,536 with
``Generator(PCG64(SeedSequence([seed, m, n, block])))``, so any voxel range is
reproducible bit-identically regardless of how it is sharded.

Starts: S vectors with i.i.d. U[-1, 1] entries, NOT normalised — each
side normalises (reading R7).  Shared by every voxel.
"""
import itertools
from math import comb, factorial

import numpy as np

BLOCK = 65536
EPS = 0.02


def num_unique(m, n):
    return comb(m + n - 1, m)


def _classes(m, n):
    return np.array(list(itertools.combinations_with_replacement(range(n), m)), dtype=np.int64)


def rank1_entries(v, m):
    """Compressed entries of v^{(x)m}: class (i_1..i_m) -> prod_k v_{i_k}.  v: [B, n] -> [B, U]."""
    v = np.asarray(v, np.float64)
    cl = _classes(m, v.shape[1])
    return np.prod(v[:, cl], axis=2)


def isotropic_entries(m, n):
    """Compressed entries of E_m with E_m x^m = ||x||^m (m even)."""
    assert m % 2 == 0
    out = np.zeros(num_unique(m, n))
    for p, c in enumerate(_classes(m, n)):
        k = np.bincount(c, minlength=n)
        if np.any(k % 2):
            continue
        q = k // 2
        num = factorial(m // 2) * np.prod([factorial(int(t)) for t in k])
        den = np.prod([factorial(int(t)) for t in q]) * factorial(m)
        out[p] = num / den
    return out


def _block(m, n, seed, block):
    rng = np.random.Generator(np.random.PCG64(np.random.SeedSequence([seed, m, n, block])))
    B = BLOCK
    F = rng.integers(1, 3, size=B)
    v1 = rng.standard_normal((B, n))
    v1 /= np.linalg.norm(v1, axis=1, keepdims=True)
    w = rng.standard_normal((B, n))
    w -= np.sum(w * v1, axis=1, keepdims=True) * v1
    w /= np.linalg.norm(w, axis=1, keepdims=True)
    th = np.deg2rad(rng.uniform(45.0, 90.0, size=B))
    v2 = np.cos(th)[:, None] * v1 + np.sin(th)[:, None] * w
    w2 = rng.uniform(0.5, 1.0, size=B)
    c = rng.uniform(0.0, 0.25, size=B)
    noise = rng.standard_normal((B, num_unique(m, n)))
    A = rank1_entries(v1, m) + ((F == 2) * w2)[:, None] * rank1_entries(v2, m)
    if m % 2 == 0:
        A += c[:, None] * isotropic_entries(m, n)[None, :]
    A += EPS * noise
    return A


def gen_voxels(m, n, first, count, seed=0):
    """float32 [count, U]: voxels first .. first+count-1 of the synthetic volume."""
    U = num_unique(m, n)
    out = np.empty((count, U), dtype=np.float32)
    v = first
    end = first + count
    while v < end:
        b = v // BLOCK
        lo = v - b * BLOCK
        hi = min(BLOCK, end - b * BLOCK)
        out[v - first: v - first + (hi - lo)] = _block(m, n, seed, b)[lo:hi].astype(np.float32)
        v += hi - lo
    return out


def gen_starts(S, n, seed=0):
    """float32 [S, n], entries i.i.d. U[-1, 1], not normalised."""
    rng = np.random.Generator(np.random.PCG64(np.random.SeedSequence([seed, 0x57A27, S, n])))
    return rng.uniform(-1.0, 1.0, size=(S, n)).astype(np.float32)


def gen_small_int(m, n, count, seed=0, amax=5):
    """float32 [count, U] with integer entries in [-amax, amax] (exactness tests)."""
    rng = np.random.Generator(np.random.PCG64(np.random.SeedSequence([seed, 0x1A7, m, n])))
    return rng.integers(-amax, amax + 1, size=(count, num_unique(m, n))).astype(np.float32)


def gen_int_vectors(count, n, seed=0, xmax=3):
    """float32 [count, n] with integer entries in [-xmax, xmax]."""
    rng = np.random.Generator(np.random.PCG64(np.random.SeedSequence([seed, 0x1A8, n])))
    return rng.integers(-xmax, xmax + 1, size=(count, n)).astype(np.float32)


def gen_uniform_tensors(m, n, count, seed=0):
    """float32 [count, U], unique entries i.i.d. U[-1, 1] (unstructured stress inputs)."""
    rng = np.random.Generator(np.random.PCG64(np.random.SeedSequence([seed, 0x0F1, m, n])))
    return rng.uniform(-1.0, 1.0, size=(count, num_unique(m, n))).astype(np.float32)


# Workload configs of BASELINE.json.  alpha per reading R4.
CONFIGS = {
    "C1": dict(m=4, n=3, N=1024, S=128, alpha=0.0, tol=1e-6, maxit=100),
    "C2": dict(m=4, n=3, N=1 << 20, S=128, alpha=0.0, tol=1e-6, maxit=100),
    "C3": dict(m=6, n=3, N=1 << 20, S=128, alpha=0.25, tol=1e-6, maxit=100),
    "C4a": dict(m=8, n=3, N=1 << 18, S=128, alpha=0.5, tol=1e-6, maxit=100),
    "C4b": dict(m=4, n=6, N=1 << 18, S=128, alpha=0.0, tol=1e-6, maxit=100),
    # C5: N is the whole volume, sharded over the ranks (strong scaling); the others are per rank
    "C5": dict(m=4, n=3, N=1 << 23, S=128, alpha=0.0, tol=1e-6, maxit=100, total=True),
    # SURVEY 8(d) extra: C2 at alpha = 0.5, the paper-like iteration load (~17.8 updates per solve)
    "C2a": dict(m=4, n=3, N=1 << 20, S=128, alpha=0.5, tol=1e-6, maxit=100),
}
