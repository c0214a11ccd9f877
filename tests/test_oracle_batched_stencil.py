"""Pins for the batched-matvec (a9) and nested-stencil (a10) oracles:
closed forms, exact integer brute force, numpy special cases."""
import numpy as np
import pytest

import oracle
from nestgen import recipes as R

rng = np.random.default_rng(99)


# ---------------------------------------------------------------- a9 batched
def test_batched_identity():
    B, m = 5, 64
    A = np.tile(np.eye(m, dtype=np.float32), (B, 1, 1))
    x = rng.uniform(-1, 1, (B, m)).astype(np.float32)
    y, _ = oracle.batched_matvec_f32(A, x, B)
    assert np.array_equal(y.reshape(B, m), x)


def test_batched_ones_and_r_plus_k():
    B, m, n = 3, 64, 64
    x = rng.integers(-3, 4, (B, n)).astype(np.float32)
    y, _ = oracle.batched_matvec_f32(np.ones((B, m, n), np.float32), x, B)
    assert np.array_equal(y.reshape(B, m), np.repeat(x.sum(1, keepdims=True), m, 1))
    r, k = np.meshgrid(np.arange(m), np.arange(n), indexing="ij")
    A = np.tile((r + k).astype(np.float32), (B, 1, 1))
    y2, _ = oracle.batched_matvec_f32(A, np.ones((B, n), np.float32), B)
    assert np.array_equal(y2.reshape(B, m), np.tile(64.0 * np.arange(m) + 2016.0, (B, 1)))


def test_batched_integer_vs_int64_einsum():
    B = 200
    A, x = R.batched_inputs(B, values="int")
    y, _ = oracle.batched_matvec_f32(A, x, B)
    ref = np.einsum("brk,bk->br", A.reshape(B, 64, 64).astype(np.int64), x.reshape(B, 64).astype(np.int64))
    assert np.array_equal(y.reshape(B, 64), ref.astype(np.float32))


def test_batched_rectangular_catches_transpose():
    B, m, n = 4, 3, 5
    A = rng.uniform(-1, 1, (B, m, n)).astype(np.float32)
    x = rng.uniform(-1, 1, (B, n)).astype(np.float32)
    y, a = oracle.batched_matvec_f32(A, x, B, m, n)
    ref = np.einsum("brk,bk->br", A.astype(np.float64), x.astype(np.float64))
    assert np.all(np.abs(y.reshape(B, m) - ref) <= 1e-7 * a.reshape(B, m) + 1e-30)


def test_batched_real_vs_numpy():
    B = 100
    A, x = R.batched_inputs(B)
    y, a = oracle.batched_matvec_f32(A, x, B)
    ref = np.einsum("brk,bk->br", A.reshape(B, 64, 64).astype(np.float64), x.reshape(B, 64).astype(np.float64))
    assert np.all(np.abs(y - ref.ravel()) <= 6e-8 * np.abs(ref.ravel()) + 1e-13 * a)


@pytest.mark.parametrize("op", ["max", "min"])
def test_batched_max_min(op):
    B = 50
    A, x = R.batched_inputs(B)
    y, _ = oracle.batched_matvec_f32(A, x, B, op=op)
    prod = A.reshape(B, 64, 64).astype(np.float64) * x.reshape(B, 1, 64).astype(np.float64)
    ref = (prod.max(2) if op == "max" else prod.min(2)).astype(np.float32)
    assert np.array_equal(y.reshape(B, 64), ref)


# ---------------------------------------------------------------- a10 stencil
@pytest.mark.parametrize("L", R.STENCIL_LS)
def test_stencil_constant_input(L):
    N, c0 = 97, 3.0
    inp = np.full(N * L + 2, c0)
    w = rng.integers(0, 8, N).astype(np.float64)
    out, _, visits = oracle.nested_stencil_f64(inp, np.ones(L), w, N, L)
    assert np.array_equal(out, w * 4 * c0 * L)
    assert visits == N


@pytest.mark.parametrize("L", [4, 33])
def test_stencil_linear_input(L):
    N = 50
    inp = np.arange(N * L + 2, dtype=np.float64)
    coef = rng.integers(-4, 5, L).astype(np.float64)
    w = rng.integers(1, 8, N).astype(np.float64)
    out, _, _ = oracle.nested_stencil_f64(inp, coef, w, N, L)
    for i in range(N):
        base = 1 + i * L
        assert out[i] == w[i] * sum(coef[j] * 4 * (base + j) for j in range(L))


def test_stencil_skip_branch_plus_zero_any_op():
    L, N = 8, 16
    inp, coef, w = R.stencil_inputs(N, L)
    for op in ("sum", "max", "min"):
        out, a, visits = oracle.nested_stencil_f64(inp, coef, w, N, L, op=op)
        z = w == 0
        assert z.sum() == 2 and visits == N
        assert np.all(out[z] == 0.0) and not np.signbit(out[z]).any()
        assert np.all(a[z] == 0.0)


@pytest.mark.parametrize("L", R.STENCIL_LS)
def test_stencil_vs_numpy(L):
    N = 300
    for values in ("int", "real"):
        inp, coef, w = R.stencil_inputs(N, L, values=values)
        out, a, _ = oracle.nested_stencil_f64(inp, coef, w, N, L)
        t = (inp[:-2] + 2 * inp[1:-1] + inp[2:]).reshape(N, L)
        ref = w * (t @ coef)
        ref[w == 0] = 0.0
        if values == "int":
            assert np.array_equal(out, ref)
        else:
            assert np.all(np.abs(out - ref) <= 1e-13 * a + 1e-300)
        for op, f in (("max", np.max), ("min", np.min)):
            o2, _, _ = oracle.nested_stencil_f64(inp, coef, w, N, L, op=op)
            ref2 = w * f(t * coef, axis=1)
            ref2[w == 0] = 0.0
            assert np.array_equal(o2, ref2)


# ---------------------------------------------------------------- NEXT-2 laplace3d
def test_laplace_constant_and_linear_fields_are_fixed_points():
    nz, ny, nx = 7, 6, 9
    i, j, k = np.meshgrid(np.arange(nz), np.arange(ny), np.arange(nx), indexing="ij")
    for u in (np.full((nz, ny, nx), 3.0), (2.0 * i - 3.0 * j + 5.0 * k + 1.0)):
        out = oracle.laplace3d_f64(u.ravel(), nz, ny, nx, 0.25).reshape(nz, ny, nx)
        assert np.array_equal(out, u)   # the discrete Laplacian of an affine field is 0


def test_laplace_quadratic_closed_form_and_boundary():
    nz, ny, nx = 5, 5, 8
    i, j, k = np.meshgrid(np.arange(nz), np.arange(ny), np.arange(nx), indexing="ij")
    u = (k * k + 2 * i * i).astype(np.float64)   # lap = 2 + 4 = 6 everywhere
    out = oracle.laplace3d_f64(u.ravel(), nz, ny, nx, 0.5).reshape(nz, ny, nx)
    assert np.array_equal(out[1:-1, 1:-1, 1:-1], u[1:-1, 1:-1, 1:-1] + 3.0)
    mask = np.ones_like(u, bool)
    mask[1:-1, 1:-1, 1:-1] = False
    assert np.array_equal(out[mask], u[mask])     # boundary untouched


def test_laplace_vs_numpy_slicing():
    nz, ny, nx = 9, 11, 13
    u = R.laplace_inputs(nz, ny, nx).reshape(nz, ny, nx)
    out = oracle.laplace3d_f64(u.ravel(), nz, ny, nx, 0.1).reshape(nz, ny, nx)
    c = u[1:-1, 1:-1, 1:-1]
    lap = (u[:-2, 1:-1, 1:-1] + u[2:, 1:-1, 1:-1] + u[1:-1, :-2, 1:-1] + u[1:-1, 2:, 1:-1]
           + u[1:-1, 1:-1, :-2] + u[1:-1, 1:-1, 2:]) - 6 * c
    assert np.array_equal(out[1:-1, 1:-1, 1:-1], c + 0.1 * lap)   # same order, no FMA in numpy
