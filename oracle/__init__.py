"""CPU oracle -- TEST INFRASTRUCTURE ONLY.

Thin ctypes wrappers over ``oracle.c`` (plain sequential C, fp64,
-ffp-contract=off).  Only ``tests/``, ``__graft_entry__.smoke()`` and
``bench.py``'s ``cpu_baseline`` / ``--impl reference`` legs may import this
package.  The product package never imports it and shares no code with it.
Each function cites the PAPER.md passage it follows (see oracle.c).
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "liboracle.so")
_lib = None

SUM, MAX, MIN = 0, 1, 2
_OPS = {"sum": SUM, "max": MAX, "min": MIN}


def lib():
    global _lib
    if _lib is None:
        if not os.path.exists(_LIB_PATH):
            raise RuntimeError(f"{_LIB_PATH} missing: run `make -C {os.path.dirname(_HERE)}`")
        L = ctypes.CDLL(_LIB_PATH)
        i64, i32, vp = ctypes.c_int64, ctypes.c_int32, ctypes.c_void_p
        L.oracle_spmv_csr_f64.argtypes = [i64, vp, vp, vp, vp, ctypes.c_int, vp, vp]
        L.oracle_spmv_csr_f64_threads.argtypes = [i64, vp, vp, vp, vp, ctypes.c_int, vp, vp, ctypes.c_int]
        L.oracle_spmv_csr_f64_threads.restype = ctypes.c_int
        L.oracle_batched_matvec_f32.argtypes = [i64, i32, i32, vp, vp, ctypes.c_int, vp, vp]
        L.oracle_nested_stencil_f64.argtypes = [i64, i32, vp, vp, vp, ctypes.c_int, vp, vp, vp]
        L.oracle_group_map.argtypes = [i32, i32, vp]
        L.oracle_simd_owner.argtypes = [i64, i32, vp]
        L.oracle_plan_geometry.argtypes = [i32, i32, i32, i32, vp]
        L.oracle_shard_rows.argtypes = [i64, i32, i32, vp]
        L.oracle_laplace3d_f64.argtypes = [i64, i64, i64, ctypes.c_double, vp, vp]
        for f in (L.oracle_spmv_csr_f64, L.oracle_batched_matvec_f32, L.oracle_nested_stencil_f64,
                  L.oracle_group_map, L.oracle_simd_owner, L.oracle_plan_geometry,
                  L.oracle_shard_rows, L.oracle_laplace3d_f64):
            f.restype = ctypes.c_int
        _lib = L
    return _lib


def _p(a):
    return ctypes.c_void_p(a.ctypes.data) if a is not None and a.size else None


def _c(a, dtype):
    return np.ascontiguousarray(a, dtype=dtype)


def _op(op):
    return _OPS[op] if isinstance(op, str) else int(op)


def spmv_csr_f64(rowptr, col, val, x, op="sum"):
    """a8: y_i = (+)_k val_k * x[col_k] per row, storage order.  Returns (y, abs)."""
    rowptr, col, val, x = _c(rowptr, np.int64), _c(col, np.int32), _c(val, np.float64), _c(x, np.float64)
    n = rowptr.size - 1
    y = np.empty(n, np.float64)
    a = np.empty(n, np.float64)
    if lib().oracle_spmv_csr_f64(n, _p(rowptr), _p(col), _p(val), _p(x), _op(op), _p(y), _p(a)):
        raise ValueError("oracle_spmv_csr_f64: bad arguments")
    return y, a


def spmv_csr_f64_threads(rowptr, col, val, x, threads, op="sum"):
    """a8 on `threads` host threads (OpenMP over rows, the same per-row loop):
    bit-identical to spmv_csr_f64.  Returns (y, abs, threads actually used)."""
    rowptr, col, val, x = _c(rowptr, np.int64), _c(col, np.int32), _c(val, np.float64), _c(x, np.float64)
    n = rowptr.size - 1
    y = np.empty(n, np.float64)
    a = np.empty(n, np.float64)
    used = lib().oracle_spmv_csr_f64_threads(n, _p(rowptr), _p(col), _p(val), _p(x), _op(op), _p(y), _p(a),
                                             int(threads))
    if used < 1:
        raise ValueError("oracle_spmv_csr_f64_threads: bad arguments")
    return y, a, used


def batched_matvec_f32(A, x, batch, m=64, n=64, op="sum"):
    """a9: y[b][r] = (float)(fp64 (+)_k A[b][r][k] x[b][k]).  Returns (y f32[batch*m], abs)."""
    A, x = _c(A, np.float32), _c(x, np.float32)
    y = np.empty(batch * m, np.float32)
    a = np.empty(batch * m, np.float64)
    if lib().oracle_batched_matvec_f32(batch, m, n, _p(A), _p(x), _op(op), _p(y), _p(a)):
        raise ValueError("oracle_batched_matvec_f32: bad arguments")
    return y, a


def nested_stencil_f64(inp, coef, w, nouter, L, op="sum"):
    """a10: the nested loop with a sequential prologue.  Returns (out, abs, visits)."""
    inp, coef, w = _c(inp, np.float64), _c(coef, np.float64), _c(w, np.float64)
    out = np.empty(nouter, np.float64)
    a = np.empty(nouter, np.float64)
    v = np.zeros(1, np.uint64)
    if lib().oracle_nested_stencil_f64(nouter, L, _p(inp), _p(coef), _p(w), _op(op), _p(out),
                                       _p(a), _p(v)):
        raise ValueError("oracle_nested_stencil_f64: bad arguments")
    return out, a, int(v[0])


def group_map(T, S):
    """a2: per thread {group, id, size, leader, mask} (mask as int32 bit pattern)."""
    out = np.empty(T * 5, np.int32)
    if lib().oracle_group_map(T, S, _p(out)):
        raise ValueError("oracle_group_map: bad arguments")
    return out.reshape(T, 5)


def simd_owner(trip, S):
    """a5: owner lane of each simd iteration under Fig 8."""
    out = np.empty(max(trip, 0), np.int32)
    if lib().oracle_simd_owner(trip, S, _p(out)):
        raise ValueError("oracle_simd_owner: bad arguments")
    return out


def plan_geometry(T, S, sharing_bytes=2048, payload_bytes=0):
    """a1: (groups_per_team, slot_bytes, uses_global_fallback) or None if invalid."""
    out = np.zeros(3, np.int32)
    if lib().oracle_plan_geometry(T, S, sharing_bytes, payload_bytes, _p(out)):
        return None
    return tuple(int(v) for v in out)


def shard_rows(n, P, r):
    """a12: (chunk, row_begin, nrows_local) of rank r."""
    out = np.zeros(3, np.int64)
    if lib().oracle_shard_rows(n, P, r, _p(out)):
        raise ValueError("oracle_shard_rows: bad arguments")
    return tuple(int(v) for v in out)


def laplace3d_f64(u, nz, ny, nx, alpha, out=None):
    """NEXT-2: one Jacobi heat step on the interior; boundary of `out` copied from
    `out` (default: a copy of u)."""
    u = _c(u, np.float64)
    o = u.copy() if out is None else _c(out, np.float64).copy()
    if lib().oracle_laplace3d_f64(nz, ny, nx, float(alpha), _p(u), _p(o)):
        raise ValueError("oracle_laplace3d_f64: bad arguments")
    return o
