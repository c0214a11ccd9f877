"""Property-based pins of the oracle (hypothesis, seeded/derandomised): on random small
inputs, every oracle function agrees with an independent exact computation written
here in plain Python integers / Fractions -- not a retyping of the oracle's loop:

* a8 SpMV on integer data: y equals the exact integer sum (Python int, no rounding),
  abs equals the exact sum of |terms|; MAX/MIN equal Python max/min over the row's
  products with the identities -inf/+inf on empty rows (R2/R5);
* a8 on real data: |y - exact| <= gamma_k * abs with the exact value from Fractions
  (the standard recursive-summation bound, k = row length), i.e. the oracle is a
  correctly ordered fp64 sum, whatever the inputs;
* a5 Fig 8: the owner of iteration j is j mod S, and every lane owns ceil/floor(trip/S);
* a1: the group count, slot size and fallback decision of PAPER.md:677-704 for any T, S,
  sharing and payload (the plain arithmetic, restated as a property: G*S == T, the slot is
  the largest multiple of 8 <= sharing/G, fallback iff payload > slot);
* a12: the row shards tile [0, n) in rank order.
"""
from fractions import Fraction

import numpy as np
from hypothesis import given, settings, strategies as st

import oracle

SET = settings(max_examples=150, deadline=None, derandomize=True)


@st.composite
def int_csr(draw, max_rows=24, max_cols=40, max_len=20):
    nrows = draw(st.integers(0, max_rows))
    ncols = draw(st.integers(1, max_cols))
    rp, col, val = [0], [], []
    for _ in range(nrows):
        k = draw(st.integers(0, min(max_len, ncols)))
        cols = sorted(draw(st.lists(st.integers(0, ncols - 1), min_size=k, max_size=k, unique=True)))
        col += cols
        val += draw(st.lists(st.integers(-9, 9), min_size=k, max_size=k))
        rp.append(len(col))
    x = draw(st.lists(st.integers(-9, 9), min_size=ncols, max_size=ncols))
    return (np.array(rp, np.int64), np.array(col, np.int32), np.array(val, np.float64),
            np.array(x, np.float64))


@SET
@given(int_csr())
def test_spmv_integer_rows_are_exact_sums(m):
    rp, col, val, x = m
    y, a = oracle.spmv_csr_f64(rp, col, val, x)
    for i in range(rp.size - 1):
        terms = [int(val[k]) * int(x[col[k]]) for k in range(rp[i], rp[i + 1])]
        assert y[i] == sum(terms) and a[i] == sum(abs(t) for t in terms)
        if not terms:
            assert not np.signbit(y[i])   # R5: empty row -> +0.0


@SET
@given(int_csr(), st.sampled_from(["max", "min"]))
def test_spmv_max_min_rows(m, op):
    rp, col, val, x = m
    y, _ = oracle.spmv_csr_f64(rp, col, val, x, op=op)
    for i in range(rp.size - 1):
        terms = [val[k] * x[col[k]] for k in range(rp[i], rp[i + 1])]
        if terms:
            assert y[i] == (max(terms) if op == "max" else min(terms))
        else:
            assert y[i] == (-np.inf if op == "max" else np.inf)


@SET
@given(int_csr(max_len=30), st.integers(0, 2**32 - 1))
def test_spmv_real_rows_within_the_summation_bound(m, seed):
    rp, col, _, _ = m
    rng = np.random.default_rng(seed)
    val = rng.uniform(-1, 1, col.size)
    x = rng.uniform(-1, 1, int(col.max()) + 1 if col.size else 1)
    y, a = oracle.spmv_csr_f64(rp, col, val, x)
    u = Fraction(1, 2**53)
    for i in range(rp.size - 1):
        ks = range(rp[i], rp[i + 1])
        exact = sum((Fraction(val[k]) * Fraction(x[col[k]]) for k in ks), Fraction(0))
        n = len(ks)
        gamma = n * u / (1 - n * u) if n else Fraction(0)
        assert abs(Fraction(y[i]) - exact) <= gamma * Fraction(a[i]) + Fraction(0)


@SET
@given(st.integers(0, 500), st.sampled_from([1, 2, 4, 8, 16, 32]))
def test_fig8_owner_is_j_mod_s(trip, S):
    own = oracle.simd_owner(trip, S)
    assert list(own) == [j % S for j in range(trip)]
    counts = np.bincount(own, minlength=S) if trip else np.zeros(S, int)
    assert counts.max() - counts.min() <= 1 and counts.sum() == trip


@SET
@given(st.sampled_from([32 * k for k in range(1, 33)]), st.sampled_from([1, 2, 4, 8, 16, 32]),
       st.integers(0, 48 * 1024), st.integers(0, 512))
def test_plan_geometry_properties(T, S, sharing, payload):
    g = oracle.plan_geometry(T, S, sharing, payload)
    G, slot, fb = g
    assert G * S == T
    assert slot % 8 == 0 and slot * G <= sharing and (slot + 8) * G > sharing
    assert fb == int(payload > slot)


@SET
@given(st.integers(0, 10**9), st.integers(1, 64))
def test_shards_tile_the_rows(n, P):
    end = 0
    for r in range(P):
        chunk, b, m = oracle.shard_rows(n, P, r)
        assert chunk == -(-n // P) and b == min(r * chunk, n) and m >= 0
        assert b == end or m == 0
        end = b + m if m else end
    assert end == n or n == 0
