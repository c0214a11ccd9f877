"""Seeded synthetic inputs shared by the oracle and the CUDA path.

This package holds NO arithmetic of the method (no SpMV, no reduction, no
mapping); it only draws inputs, from the counter-based generator in
``nestgen.c``.  Every element is a pure function of (seed, stream, index), so a
row range regenerates independently (multi-GPU shards, bounded CPU samples).

The workload recipes (shapes, distributions, seeds) are in ``recipes.py`` and
are stated in DESIGN.md ("Input recipe"), following SURVEY.md §8(d).
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "libnestgen.so")
_lib = None

UNIFORM, BANDED_FAR = 0, 1
REAL_PM1, INT, REAL_HALF_3HALF = 0, 1, 2

# disjoint streams for vectors (matrix streams 1..3 live in nestgen.c)
STREAM_X = 11
STREAM_BATCH_A = 21
STREAM_BATCH_X = 22
STREAM_ST_IN = 31
STREAM_ST_COEF = 32
STREAM_ST_W = 33

_VKIND = {"real": REAL_PM1, "int": INT, "half3half": REAL_HALF_3HALF}
_STRUCT = {"uniform": UNIFORM, "banded_far": BANDED_FAR}


def lib():
    global _lib
    if _lib is None:
        if not os.path.exists(_LIB_PATH):
            raise RuntimeError(f"{_LIB_PATH} missing: run `make -C {os.path.dirname(_HERE)}`")
        L = ctypes.CDLL(_LIB_PATH)
        i64, u64, i32, vp = ctypes.c_int64, ctypes.c_uint64, ctypes.c_int32, ctypes.c_void_p
        L.nestgen_csr_rowptr.argtypes = [u64, i64, i64, i64, i32, i32, vp]
        L.nestgen_csr_rowptr.restype = i64
        L.nestgen_csr_fill.argtypes = [u64, i64, i64, i64, i32, i64, i32, i32, i64, i64, vp, vp, vp]
        L.nestgen_csr_fill.restype = ctypes.c_int
        for f in (L.nestgen_vec_f64, L.nestgen_vec_f32):
            f.argtypes = [u64, u64, i64, i64, i32, i64, i64, vp]
            f.restype = ctypes.c_int
        _lib = L
    return _lib


def _ptr(a):
    return ctypes.c_void_p(a.ctypes.data) if a is not None and a.size else None


def _out(out, n, dtype):
    if out is None:
        return np.empty(n, dtype=dtype)
    assert out.dtype == dtype and out.size >= n and out.flags.c_contiguous
    return out[:n]


def csr_rowptr(seed, nrows, ncols, nnz_min, nnz_max, row_begin=0, out=None):
    rp = _out(out, nrows + 1, np.int64)
    nnz = lib().nestgen_csr_rowptr(seed, row_begin, nrows, ncols, nnz_min, nnz_max, _ptr(rp))
    if nnz < 0:
        raise ValueError("nestgen_csr_rowptr: bad arguments")
    return rp


def csr_fill(seed, rowptr, ncols, structure="banded_far", band_w=4096, far_den=16,
             values="real", vlo=-4, vhi=4, row_begin=0, col_out=None, val_out=None):
    nrows = rowptr.size - 1
    nnz = int(rowptr[-1])
    col = _out(col_out, nnz, np.int32)
    val = _out(val_out, nnz, np.float64)
    rc = lib().nestgen_csr_fill(seed, row_begin, nrows, ncols, _STRUCT[structure], band_w, far_den,
                                _VKIND[values], vlo, vhi, _ptr(rowptr), _ptr(col), _ptr(val))
    if rc:
        raise ValueError("nestgen_csr_fill: bad arguments")
    return col, val


def csr(seed, nrows, ncols, nnz_min, nnz_max, structure="banded_far", band_w=4096, far_den=16,
        values="real", vlo=-4, vhi=4, row_begin=0):
    """CSR (rowptr int64[nrows+1], colind int32[nnz], val f64[nnz]) for global rows
    [row_begin, row_begin+nrows).  rowptr is local (rowptr[0] == 0)."""
    rp = csr_rowptr(seed, nrows, ncols, nnz_min, nnz_max, row_begin)
    col, val = csr_fill(seed, rp, ncols, structure, band_w, far_den, values, vlo, vhi, row_begin)
    return rp, col, val


def vec_f64(seed, stream, n, values="real", vlo=-8, vhi=8, begin=0, out=None):
    o = _out(out, n, np.float64)
    if lib().nestgen_vec_f64(seed, stream, begin, n, _VKIND[values], vlo, vhi, _ptr(o)):
        raise ValueError("nestgen_vec_f64: bad arguments")
    return o


def vec_f32(seed, stream, n, values="real", vlo=-3, vhi=3, begin=0, out=None):
    o = _out(out, n, np.float32)
    if lib().nestgen_vec_f32(seed, stream, begin, n, _VKIND[values], vlo, vhi, _ptr(o)):
        raise ValueError("nestgen_vec_f32: bad arguments")
    return o
