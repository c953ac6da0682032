"""Pin of reading R12 (the paper-style flop count per SS-HOPM update, P:L263-279,
Sec. III-B.5 / Table II only give O(.)): run the LITERAL pseudocode of Fig. 1
lines 2-8, Fig. 2 and Fig. 3 (reading R10 for
line 6) from oracle/combinatorics.py with a number type that counts every
floating-point operation it executes, and compare the tally with
oracle.sshopm.paper_flops_per_iter = (m+2) U + (m+1) T1 + 5 n.  The count is
taken from the executed operations, not from a restated formula: a dropped or
extra multiply in either kernel, a wrong term count T1, or a miscounted
normalisation changes the tally."""
import math
import random

import pytest

from oracle import combinatorics as C
from oracle.sshopm import paper_flops_per_iter


class Counted:
    """A float that counts + - * / and sqrt (integer multinomials promote through __rmul__)."""
    ops = 0

    def __init__(self, v):
        self.v = float(v)

    @staticmethod
    def _val(o):
        return o.v if isinstance(o, Counted) else float(o)

    def _op(self, v):
        Counted.ops += 1
        return Counted(v)

    def __add__(self, o): return self._op(self.v + self._val(o))
    __radd__ = __add__
    def __sub__(self, o): return self._op(self.v - self._val(o))
    def __rsub__(self, o): return self._op(self._val(o) - self.v)
    def __mul__(self, o): return self._op(self.v * self._val(o))
    __rmul__ = __mul__
    def __truediv__(self, o): return self._op(self.v / self._val(o))
    def __neg__(self): return Counted(-self.v)          # sign flip (Fig. 1 line 5): not an arithmetic op


def counted_sqrt(c):
    Counted.ops += 1
    return Counted(math.sqrt(c.v))


SHAPES = [(2, 2), (2, 3), (3, 2), (3, 3), (4, 2), (4, 3), (4, 4), (5, 3), (6, 3), (4, 6), (8, 3), (3, 5)]


@pytest.mark.parametrize("m,n", SHAPES)
def test_literal_update_executes_paper_flops(m, n):
    rng = random.Random(m * 100 + n)
    U = math.comb(m + n - 1, m)
    A = [Counted(rng.uniform(-1, 1)) for _ in range(U)]
    x = [Counted(rng.uniform(-1, 1)) for _ in range(n)]
    Counted.ops = 0
    C.sshopm_update(A, x, 0.5, m, n, sqrt=counted_sqrt)
    assert Counted.ops == paper_flops_per_iter(m, n)


@pytest.mark.parametrize("m,n", [(4, 3), (6, 3)])
def test_counted_kernels_match_their_terms(m, n):
    """Fig. 2 alone executes (m+2) per class and Fig. 3 (m+1) per (class, distinct index) term."""
    rng = random.Random(7)
    U = math.comb(m + n - 1, m)
    A = [Counted(rng.uniform(-1, 1)) for _ in range(U)]
    x = [Counted(rng.uniform(-1, 1)) for _ in range(n)]
    Counted.ops = 0
    C.symm_ttv0(A, x, m, n)
    assert Counted.ops == (m + 2) * U
    Counted.ops = 0
    C.symm_ttv1(A, x, m, n)
    terms = sum(len(set(I)) for I in C.index_classes(m, n))     # (class, unique i) pairs of Fig. 3 line 5
    assert terms == n * math.comb(m + n - 2, m - 1)
    assert Counted.ops == (m + 1) * terms


def test_literal_update_values_match_full_tensor():
    """The counted path computes the same update as the FP64 full-tensor oracle."""
    import numpy as np
    from oracle import sshopm as O
    rng = np.random.default_rng(3)
    m, n = 4, 3
    A = rng.uniform(-1, 1, O.num_unique(m, n))
    x = rng.uniform(-1, 1, n)
    x /= np.linalg.norm(x)
    lam, x1 = C.sshopm_update(list(A), list(x), 0.3, m, n)
    full = O.expand_full(A, m, n)                        # [1, n, ..., n]
    g = O.axm1(full, x[None, :])[0] + 0.3 * x
    xn = g / np.linalg.norm(g)
    assert np.allclose(x1, xn, rtol=1e-13, atol=1e-14)
    assert abs(lam - O.axm(full, xn[None, :])[0]) < 1e-12
