"""The seeded input generators: determinism, independent regeneration of any
row range, and the structure the recipe states."""
import numpy as np

import nestgen
from nestgen import recipes as R


def test_deterministic_and_row_ranges_regenerate():
    spec = R.SpmvSpec("t", 7, 5000, 6000, 4, 12)
    rp, col, val = R.spmv_matrix(spec)
    rp2, col2, val2 = R.spmv_matrix(spec)
    assert np.array_equal(rp, rp2) and np.array_equal(col, col2) and np.array_equal(val, val2)
    b, n = 1234, 777
    rpl, cl, vl = R.spmv_matrix(spec, row_begin=b, nrows=n)
    assert np.array_equal(rpl + rp[b], rp[b:b + n + 1])
    assert np.array_equal(cl, col[rp[b]:rp[b + n]])
    assert np.array_equal(vl, val[rp[b]:rp[b + n]])
    x = R.spmv_x(spec)
    assert np.array_equal(R.spmv_x(spec, begin=100, n=50), x[100:150])


def test_structure_banded_far():
    spec = R.SpmvSpec("t", 11, 20000, 20000, 4, 12)
    rp, col, val = R.spmv_matrix(spec)
    lens = np.diff(rp)
    assert lens.min() >= 4 and lens.max() <= 12 and abs(lens.mean() - 8) < 0.1
    rows = np.repeat(np.arange(spec.nrows), lens)
    near = np.abs(col.astype(np.int64) - rows) <= spec.band_w
    # far columns are uniform, so a few land in the band anyway
    assert 0.93 < near.mean() < 0.96
    for i in range(0, spec.nrows, 997):
        c = col[rp[i]:rp[i + 1]]
        assert np.all(np.diff(c) > 0)          # distinct, ascending
    assert np.all((val >= -1) & (val < 1))


def test_integer_values_and_vectors():
    spec = R.CFG1.integer()
    rp, col, val, x = R.spmv_inputs(spec)
    assert np.all(val == np.round(val)) and val.min() >= -4 and val.max() <= 4
    assert np.all(x == np.round(x)) and x.min() >= -8 and x.max() <= 8
    assert len(set(np.unique(val).tolist())) == 9
    a = nestgen.vec_f32(5, 1, 1000)
    assert a.dtype == np.float32 and np.all((a >= -1) & (a < 1))


def test_stencil_and_batched_recipes():
    inp, coef, w = R.stencil_inputs(64, 8)
    assert inp.size == 64 * 8 + 2 and coef.size == 8 and w.size == 64
    assert np.all(w[::8] == 0) and np.all(w[1::8] >= 0.5)
    A, x = R.batched_inputs(3)
    assert A.size == 3 * 64 * 64 and x.size == 3 * 64
