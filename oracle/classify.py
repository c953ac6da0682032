"""Eigenpair type classification oracle — TEST INFRASTRUCTURE ONLY.

Fibre directions are the local maxima of D(g) = A g^m on the sphere (P:L287,
P:L301); SS-HOPM with a convex shift converges to them.  For
an eigenpair (lam, x) of Definition 3, the second-order test on the
sphere (Kolda-Mayo [1], cited P:L402) uses the projected Hessian of the
Lagrangian
    C(lam, x) = U^T [ (m-1) A x^{m-2} - lam I ] U,
U an orthonormal basis of x-perp (A x^{m-2} by Definition 2 with p = 2,
P:L39-42).  Reading R18: type +1 = local maximum (C negative
definite), -1 = local minimum (C positive definite), 0 = saddle (indefinite),
2 = degenerate (some eigenvalue of C within ctol * max(1, |lam|) of zero),
3 = empty dedup slot.
Plain numpy FP64 on the full tensor: A x^{m-2} by two trailing-mode
contractions, U from an SVD, eigenvalues by numpy.linalg.eigvalsh.
"""
import numpy as np

from oracle import sshopm as O

MAX, MIN, SADDLE, DEGENERATE, EMPTY = 1, -1, 0, 2, 3


def projected_hessian(full, lam, x):
    """C for one tensor (full [n]*m), eigenvalue lam and unit vector x -> [(n-1), (n-1)]."""
    m = full.ndim
    n = full.shape[0]
    x = np.asarray(x, np.float64)
    x = x / np.linalg.norm(x)
    H = O.ttv(full[None], x[None], 2)[0] if m > 2 else full.astype(np.float64)   # A x^{m-2}
    H = (m - 1) * H - lam * np.eye(n)
    _, _, vt = np.linalg.svd(x[None, :])
    Ub = vt[1:].T                                            # orthonormal basis of x-perp, [n, n-1]
    return Ub.T @ H @ Ub


def classify_one(full, lam, x, ctol):
    mu = np.linalg.eigvalsh(projected_hessian(full, lam, x)) if full.shape[0] > 1 else np.zeros(0)
    thr = ctol * max(1.0, abs(lam))
    if mu.size and np.min(np.abs(mu)) <= thr:
        return DEGENERATE, mu
    if np.all(mu < 0):
        return MAX, mu
    if np.all(mu > 0):
        return MIN, mu
    return SADDLE, mu


def classify(entries, m, n, count, lam, x, ctol=1e-3):
    """Types [V, kmax] int8 of the dedup records (count [V], lam [V,K], x [V,K,n]); empty slots -> 3."""
    full = O.expand_full(entries, m, n)
    V, K = lam.shape
    out = np.full((V, K), EMPTY, np.int8)
    margin = np.full((V, K), np.inf)
    for v in range(V):
        for k in range(min(int(count[v]), K)):
            t, mu = classify_one(full[v], float(lam[v, k]), x[v, k], ctol)
            out[v, k] = t
            if mu.size:
                margin[v, k] = np.min(np.abs(mu)) / max(1.0, abs(float(lam[v, k])))
    return out, margin
