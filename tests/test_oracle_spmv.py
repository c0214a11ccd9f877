"""Pins for the CSR SpMV oracle (a8) against things other than itself:
closed forms, exact brute force, and library special cases (scipy.sparse,
numpy dense matmul, math.fsum).  PAPER.md:877-884 defines the kernel
(sparse_matvec); the reduction identity/combination is DESIGN.md R2/R5."""
import math
from fractions import Fraction

import numpy as np
import pytest
import scipy.sparse as sp

import oracle
from nestgen import recipes as R

rng = np.random.default_rng(1234)


def csr_from_rows(rows):
    """rows: list of list of (col, val)."""
    rp = [0]
    col, val = [], []
    for r in rows:
        for c, v in r:
            col.append(c)
            val.append(v)
        rp.append(len(col))
    return (np.array(rp, np.int64), np.array(col, np.int32), np.array(val, np.float64))


def test_identity():
    n = 257
    rp = np.arange(n + 1, dtype=np.int64)
    col = np.arange(n, dtype=np.int32)
    x = rng.uniform(-1, 1, n)
    y, a = oracle.spmv_csr_f64(rp, col, np.ones(n), x)
    assert np.array_equal(y.view(np.int64), x.view(np.int64))
    assert np.array_equal(a, np.abs(x))


def test_diagonal():
    n = 300
    d = rng.uniform(-3, 3, n)
    x = rng.uniform(-1, 1, n)
    rp = np.arange(n + 1, dtype=np.int64)
    y, _ = oracle.spmv_csr_f64(rp, np.arange(n, dtype=np.int32), d, x)
    assert np.array_equal(y, d * x)   # one product, one rounding, +0.0 + t == t


def test_all_ones_rows():
    lens = [0, 1, 5, 8, 31, 32, 33, 64, 3]
    n = 100
    rows = [[(c, 1.0) for c in sorted(rng.choice(n, L, replace=False))] for L in lens]
    rp, col, val = csr_from_rows(rows)
    y, _ = oracle.spmv_csr_f64(rp, col, val, np.ones(n))
    assert np.array_equal(y, np.array(lens, np.float64))
    # x_j = j  ->  y_i = sum of the row's column indices (catches x[k] vs x[col[k]])
    y2, _ = oracle.spmv_csr_f64(rp, col, val, np.arange(n, dtype=np.float64))
    assert np.array_equal(y2, np.array([sum(c for c, _ in r) for r in rows], np.float64))


def test_empty_rows_are_plus_zero():
    rows = [[], [(0, -1.0)], [], [(1, 2.0), (2, -2.0)]]
    rp, col, val = csr_from_rows(rows)
    x = np.array([0.0, 1.0, 1.0])
    y, a = oracle.spmv_csr_f64(rp, col, val, x)
    assert y.tolist() == [0.0, 0.0, 0.0, 0.0]
    assert not np.signbit(y).any()        # +0.0 everywhere (R5): -1*0 = -0 adds to +0 -> +0
    assert a.tolist() == [0.0, 0.0, 0.0, 4.0]


@pytest.mark.parametrize("L", [33, 64, 1000])
def test_long_row_integer_exact(L):
    n = 2000
    c = np.sort(rng.choice(n, L, replace=False)).astype(np.int32)
    v = rng.integers(-4, 5, L).astype(np.float64)
    x = rng.integers(-8, 9, n).astype(np.float64)
    rp = np.array([0, L], np.int64)
    y, _ = oracle.spmv_csr_f64(rp, c, v, x)
    assert y[0] == float(sum(int(vv) * int(x[cc]) for cc, vv in zip(c, v)))


def test_cfg1_integer_bruteforce_fractions():
    spec = R.CFG1.integer()
    rp, col, val, x = R.spmv_inputs(spec)
    y, _ = oracle.spmv_csr_f64(rp, col, val, x)
    for i in range(spec.nrows):
        s = sum(Fraction(val[k]) * Fraction(x[col[k]]) for k in range(rp[i], rp[i + 1]))
        assert Fraction(y[i]) == s


def test_cfg1_real_vs_scipy_and_fsum():
    rp, col, val, x = R.spmv_inputs(R.CFG1)
    y, a = oracle.spmv_csr_f64(rp, col, val, x)
    A = sp.csr_matrix((val, col, rp), shape=(R.CFG1.nrows, R.CFG1.ncols))
    ys = A @ x
    assert np.all(np.abs(y - ys) <= 1e-13 * a)
    for i in range(0, R.CFG1.nrows, 7):
        terms = [val[k] * x[col[k]] for k in range(rp[i], rp[i + 1])]
        exact = math.fsum(terms)
        n = len(terms)
        gamma = n * 2.0 ** -53 / (1 - n * 2.0 ** -53)
        assert abs(y[i] - exact) <= gamma * a[i] + 1e-300
        assert a[i] == pytest.approx(math.fsum(abs(t) for t in terms), rel=1e-14)


def test_dense_as_csr_vs_numpy_matmul():
    m, n = 37, 53
    D = rng.uniform(-1, 1, (m, n))
    D[rng.random((m, n)) < 0.5] = 0.0
    x = rng.uniform(-1, 1, n)
    S = sp.csr_matrix(D)
    y, a = oracle.spmv_csr_f64(S.indptr.astype(np.int64), S.indices.astype(np.int32), S.data, x)
    assert np.all(np.abs(y - D @ x) <= 1e-13 * a + 1e-300)


@pytest.mark.parametrize("op", ["max", "min"])
def test_max_min_bruteforce(op):
    rp, col, val, x = R.spmv_inputs(R.CFG1)
    y, _ = oracle.spmv_csr_f64(rp, col, val, x, op=op)
    f = max if op == "max" else min
    for i in range(R.CFG1.nrows):
        assert y[i] == f(val[k] * x[col[k]] for k in range(rp[i], rp[i + 1]))
    # empty row -> the identity
    y0, _ = oracle.spmv_csr_f64(np.zeros(2, np.int64), np.zeros(0, np.int32), np.zeros(0), x, op=op)
    assert y0[0] == (-np.inf if op == "max" else np.inf)


def test_row_shards_concatenate():
    """CPU P-shard check: rows are independent units, so the
    oracle on each rank's equal-row shard concatenates to the whole."""
    spec = R.CFG1
    rp, col, val, x = R.spmv_inputs(spec)
    y, _ = oracle.spmv_csr_f64(rp, col, val, x)
    for P in (1, 2, 3, 4, 8):
        parts = []
        for r in range(P):
            chunk, b, cnt = oracle.shard_rows(spec.nrows, P, r)
            assert chunk == -(-spec.nrows // P)
            rpl, cl, vl = R.spmv_matrix(spec, row_begin=b, nrows=cnt)
            assert np.array_equal(rpl + rp[b], rp[b:b + cnt + 1])
            parts.append(oracle.spmv_csr_f64(rpl, cl, vl, x)[0])
        assert np.array_equal(np.concatenate(parts), y)


def test_threaded_oracle_is_bit_identical_to_the_sequential_one():
    """The all-cores baseline runs the same per-row loop on
    several threads: rows are independent, so any thread count gives the same
    bits as the one-thread oracle (ragged rows, empty rows, every op)."""
    import numpy as np
    rng = np.random.default_rng(5)
    lens = rng.integers(0, 40, 5003)
    lens[::97] = 0
    rp = np.concatenate([[0], np.cumsum(lens)]).astype(np.int64)
    col = rng.integers(0, 3000, rp[-1]).astype(np.int32)
    val = rng.standard_normal(rp[-1])
    x = rng.standard_normal(3000)
    for op in ("sum", "max", "min"):
        y1, a1 = oracle.spmv_csr_f64(rp, col, val, x, op=op)
        for t in (1, 2, 3, 8):
            yt, at, used = oracle.spmv_csr_f64_threads(rp, col, val, x, t, op=op)
            assert 1 <= used <= t
            assert np.array_equal(y1.view(np.int64), yt.view(np.int64)) and np.array_equal(a1, at)
