"""Pins for oracle/combinatorics.py and the oracle's class layout (Sec. III).

Every expectation below is a value printed in PAPER.md (cited), a counting
identity, or a brute-force evaluation of the full-tensor definition (Eq. 1) —
never a retyping of the function under test.
"""
import itertools
import json
import os
from math import factorial

import numpy as np
import pytest

from oracle import combinatorics as C
from oracle import sshopm as O
import synthetic as syn


def _pins(golden_dir):
    with open(os.path.join(golden_dir, "paper_pins.json")) as f:
        return json.load(f)


def _table1(golden_dir):
    rows = []
    with open(os.path.join(golden_dir, "table1_m3_n4.txt")) as f:
        for line in f:
            if line.startswith("#") or not line.strip():
                continue
            v = [int(t) for t in line.split()]
            rows.append((v[0], v[1:4], v[4:8]))
    return rows


def test_table1_order_fig4(golden_dir):
    """Table I: Fig. 4 successor walk reproduces the 20 rows in order."""
    rows = _table1(golden_dir)
    assert len(rows) == 20
    cl = C.index_classes(3, 4)
    assert [r[1] for r in rows] == cl
    assert [r[2] for r in rows] == [C.monomial_rep(I, 4) for I in cl]


def test_table1_order_oracle_layout(golden_dir):
    """The oracle's independent itertools enumeration gives the same Table I order."""
    rows = _table1(golden_dir)
    assert [list(np.array(c) + 1) for c in O.class_list(3, 4)] == [r[1] for r in rows]


@pytest.mark.parametrize("m,n", [(2, 2), (3, 2), (3, 4), (4, 3), (5, 2), (6, 3), (8, 3), (4, 6), (2, 7)])
def test_fig4_walk_equals_oracle_layout(m, n):
    """Fig. 4 walk == itertools order == sorted-lexicographic order for many (m, n)."""
    fig4 = C.index_classes(m, n)
    itl = [list(np.array(c) + 1) for c in O.class_list(m, n)]
    assert fig4 == itl
    assert fig4 == sorted(fig4)                      # increasing lexicographic
    mono = [C.monomial_rep(I, n) for I in fig4]
    assert mono == sorted(mono, reverse=True)        # decreasing in monomial rep


def test_successor_examples(golden_dir):
    p = _pins(golden_dir)
    for a, b in p["successors_m3_n4"]["pairs"]:
        assert C.update_index(list(a), 4) == b
    for a, b in p["successor_footnote"]["pairs"]:
        assert C.update_index(list(a), p["successor_footnote"]["n"]) == b


def test_unique_counts(golden_dir):
    """(4,3) -> 15 unique of 81 entries; (6,3) -> 28; (8,3) -> 45."""
    for m, n, U, total in _pins(golden_dir)["unique_counts"]["cases"]:
        assert len(C.index_classes(m, n)) == U
        assert O.num_unique(m, n) == U
        assert syn.num_unique(m, n) == U
        if total is not None:
            assert n ** m == total


def test_unrolled_term_counts(golden_dir):
    """for (4,3) Ax^m has 15 terms and each Ax^{m-1} entry 10 terms (classes with k_j > 0)."""
    p = _pins(golden_dir)["unrolled_term_counts_m4_n3"]
    cl = C.index_classes(4, 3)
    assert len(cl) == p["axm_terms"]
    for j in range(1, 4):
        assert sum(1 for I in cl if j in I) == p["axm1_terms_per_output"]


def test_multinomial_worked_example(golden_dir):
    """[1,2,2,5,5,5,5] -> c = 7!/48 = 105, sigma(5) = 6!/12 = 60."""
    p = _pins(golden_dir)["multinomial_example"]
    assert factorial(7) // p["divisor0"] == p["c"]
    assert C.multinomial0(p["I"]) == p["c"]
    assert factorial(6) // p["divisor1"] == p["sigma"]
    assert C.multinomial1(p["I"], p["i"]) == p["sigma"]
    # footnote 3 / P:L325: sigma = c * k_i / m
    k5 = p["I"].count(5)
    assert p["c"] * k5 // len(p["I"]) == p["sigma"]


def test_m3_n2_example(golden_dir):
    """P:L35/L69-77/L176: class [1,1,2] = {112,121,211}, c = 3, sigma(1) = 2, sigma(2) = 1."""
    p = _pins(golden_dir)["m3_n2_example"]
    assert C.monomial_rep(p["I"], 2) == p["monomial"]
    assert C.multinomial0(p["I"]) == p["c"]
    assert C.multinomial1(p["I"], 1) == p["sigma1"]
    assert C.multinomial1(p["I"], 2) == p["sigma2"]
    # brute force: tensor indices in the class, and those starting with 1 / 2
    members = [t for t in itertools.product([1, 2], repeat=3) if sorted(t) == p["I"]]
    assert len(members) == p["c"]
    assert sum(1 for t in members if t[0] == 1) == p["sigma1"]
    assert sum(1 for t in members if t[0] == 2) == p["sigma2"]


@pytest.mark.parametrize("m,n", [(2, 3), (3, 2), (3, 4), (4, 3), (5, 3), (6, 3), (4, 6)])
def test_multinomials_count_tensor_indices(m, n):
    """Property 2 by brute force: class sizes sum to n^m; sigma_c(j) sums to n^{m-1} per j."""
    cl = C.index_classes(m, n)
    sizes = {tuple(I): 0 for I in cl}
    first = {(tuple(I), j): 0 for I in cl for j in range(1, n + 1)}
    for t in itertools.product(range(1, n + 1), repeat=m):
        key = tuple(sorted(t))
        sizes[key] += 1
        first[(key, t[0])] += 1
    for I in cl:
        assert C.multinomial0(I) == sizes[tuple(I)]
        for j in set(I):
            assert C.multinomial1(I, j) == first[(tuple(I), j)]
    assert sum(C.multinomial0(I) for I in cl) == n ** m


@pytest.mark.parametrize("m,n", [(2, 3), (3, 2), (3, 3), (4, 3), (5, 2), (6, 3), (4, 4), (3, 5)])
def test_compressed_products_equal_full_bruteforce(m, n):
    """Fig. 2 / Fig. 3 (compressed, Eq. 4 / Eq. 6) == Eq. 1 on the full tensor, exactly on integers."""
    ent = syn.gen_small_int(m, n, 6, seed=m * 10 + n).astype(np.float64)
    xs = syn.gen_int_vectors(6, n, seed=m + n).astype(np.float64)
    full = O.expand_full(ent, m, n)
    # brute-force Eq. 1 with explicit loops
    for v in range(6):
        y0 = 0.0
        y1 = [0.0] * n
        for t in itertools.product(range(n), repeat=m):
            prod_all = np.prod([xs[v, i] for i in t])
            y0 += full[v][t] * prod_all
            y1[t[0]] += full[v][t] * np.prod([xs[v, i] for i in t[1:]])
        assert C.symm_ttv0(list(ent[v]), list(xs[v]), m, n) == y0
        assert C.symm_ttv1(list(ent[v]), list(xs[v]), m, n) == y1
        assert O.axm(full[v:v + 1], xs[v:v + 1])[0] == y0
        assert list(O.axm1(full[v:v + 1], xs[v:v + 1])[0]) == y1


def test_fig3_no_division_by_zero_component():
    """Reading R10: x_i = 0 must not produce NaN (Fig. 3 line 6 divides by x_i)."""
    m, n = 4, 3
    ent = syn.gen_small_int(m, n, 1, seed=3)[0].astype(np.float64)
    x = [0.0, 2.0, -1.0]
    y = C.symm_ttv1(list(ent), x, m, n)
    assert all(np.isfinite(y))
    full = O.expand_full(ent[None], m, n)
    assert list(O.axm1(full, np.array([x]))[0]) == y


def test_euler_identity_exact():
    """Definition 2: x . (A x^{m-1}) = A x^m exactly on integer data (used by the GPU's lambda fusion)."""
    for m, n in [(4, 3), (6, 3), (8, 3), (4, 6), (3, 3)]:
        ent = syn.gen_small_int(m, n, 16, seed=1)
        xs = syn.gen_int_vectors(16, n, seed=2, xmax=2)
        full = O.expand_full(ent, m, n)
        g = O.axm1(full, xs)
        assert np.array_equal(np.sum(g * xs, axis=1), O.axm(full, xs))


def test_table3_rate_time_consistency(golden_dir):
    """Table III: rate x time is one flop total (+-2%) across all 8 cells."""
    p = _pins(golden_dir)["table3_consistency"]
    prods = [g * 1e9 * t * 1e-3 for gr, tr in zip(p["gflops"], p["ms"]) for g, t in zip(gr, tr)]
    mean = np.mean(prods)
    assert all(abs(v / mean - 1) < 0.02 for v in prods)
    assert 5.8e8 < mean < 6.1e8
