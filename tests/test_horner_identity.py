"""The Horner regrouping of Eq. 6 used by the (6,3) / (8,3) / (4,6) kernels (DESIGN.md §7 "n = 3, m >= 6",
"Any n"), checked in FP64 against the oracle's full-tensor A x^{m-1} (CPU; independent of the CUDA code).

    g_j = D! sum_{d=0}^{D} x0^{D-d}/(D-d)! sum_{|t|=d} a_{class(0^{D-d} t + e_j)} prod_i x_i^{k_i}/k_i!

over tail multisets t of the variables 1..n-1 (k_i = multiplicity of i in t), evaluated by Horner in x0 with
factors x0/(D-d+1), as the kernels do (divided powers for raw rows), and in the integer-weight form of the
apply hook (weights D!/((D-d)! prod k_i!) on the plain monomials, plain Horner in x0).
"""
import itertools
import math

import numpy as np
import pytest

import synthetic as syn
from oracle import sshopm as O


def _tails(n, d):
    return list(itertools.combinations_with_replacement(range(1, n), d))


def _horner(entries, x, m, n, exact):
    D = m - 1
    cls = {tuple(c): i for i, c in enumerate(O.class_list(m, n))}
    g = np.zeros(n)
    for j in range(n):
        a = lambda q: entries[cls[tuple(sorted(q + (j,)))]]
        acc = a((0,) * D)
        for d in range(1, D + 1):
            p = 0.0
            for t in _tails(n, d):
                mono = np.prod([x[i] for i in t])
                ks = [t.count(i) for i in set(t)]
                if exact:
                    w = math.factorial(D) // (math.factorial(D - d) * int(np.prod([math.factorial(k) for k in ks])))
                    p += a((0,) * (D - d) + t) * w * mono
                else:
                    p += a((0,) * (D - d) + t) * mono / np.prod([math.factorial(k) for k in ks])
            acc = acc * (x[0] if exact else x[0] / (D - d + 1)) + p
        g[j] = acc if exact else acc * math.factorial(D)
    return g


@pytest.mark.parametrize("m,n", [(4, 3), (6, 3), (8, 3), (4, 6), (5, 4)])
@pytest.mark.parametrize("exact", [False, True])
def test_horner_regrouping_equals_full_tensor(m, n, exact):
    ent = syn.gen_uniform_tensors(m, n, 4, seed=m * 10 + n).astype(np.float64)
    xs = syn.gen_starts(4, n, seed=3).astype(np.float64)
    full = O.expand_full(ent, m, n)
    for v in range(4):
        x = xs[v] / np.linalg.norm(xs[v])
        ref = O.axm1(full[v:v + 1], x[None, :])[0]
        got = _horner(ent[v], x, m, n, exact)
        np.testing.assert_allclose(got, ref, rtol=1e-12, atol=1e-12)


def test_horner_operation_counts():
    """n (Q - 1 + D) multiply-adds + (Q - 3) shared products per step for n = 3: (6,3) 93 vs the
    monomial form's n Q + monomial products; a count of the regrouped terms, not of the formula."""
    for m, expect in ((4, 43), (6, 93), (8, 159)):
        D, n = m - 1, 3
        Q = math.comb(D + n - 1, D)
        terms = sum(len(_tails(n, d)) for d in range(0, D + 1))
        assert terms == Q                                   # every degree-D monomial appears exactly once
        shared = sum(len(_tails(n, d)) for d in range(2, D + 1))   # tail monomials of degree >= 2
        assert n * (Q - 1 + D) + shared == expect
