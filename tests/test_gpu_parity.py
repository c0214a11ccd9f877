"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle on the
same seeded inputs.  Bars (north_star; R3/R4):
  * integer and index outputs, integer-valued fp reductions: bit-exact;
  * general fp: |gpu - oracle| <= tol * abs_ref per row, tol = 1e-12 (fp64),
    1e-5 (fp32), abs_ref = sum |terms| (cancellation-safe); abs_ref == 0
    requires an exact +0.0;
  * MAX/MIN: equal by value (the sign of a zero tie is unordered);
  * the modes (SPMD, GENERIC_SMEM, GENERIC_SHFL) and U agree bit-for-bit at
    the same simdlen.
"""
import numpy as np
import pytest

import oracle
from nestgen import recipes as R

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

SIMDLENS = (1, 2, 4, 8, 16, 32)
MODES = ("spmd", "generic_smem", "generic_shfl")


@pytest.fixture(scope="module")
def P():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_icpp_wrightdtcc23_b200 as P
    return P


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


def host(t):
    return t.cpu().numpy()


def assert_close(y, ref, absref, tol):
    y = np.asarray(y, np.float64)
    zero = absref == 0
    assert np.all(y[zero] == 0.0) and not np.signbit(y[zero]).any(), "abs_ref == 0 must give +0.0"
    err = np.abs(y - ref)
    bad = err > tol * absref
    assert not bad.any(), f"{bad.sum()} rows beyond {tol}*abs: worst {np.max(err[~zero] / absref[~zero]):.3e}"


def bits(a):
    a = np.ascontiguousarray(a)
    return a.view(np.int64 if a.dtype == np.float64 else np.int32)


# ------------------------------------------------------------------ a2/a5/a6 probe
@pytest.mark.parametrize("S", SIMDLENS)
@pytest.mark.parametrize("mode", MODES)
@pytest.mark.parametrize("T", [32, 256, 1024])
def test_probe_mapping(P, S, mode, T):
    teams = 3
    G = T // S
    for trip in sorted({0, 1, max(S - 1, 0), S, S + 1, 3 * S + 1, 77}):
        mp, hits, owner, totals = P.probe_mapping(teams, trip, simdlen=S, mode=mode, threads_per_team=T)
        ref = oracle.group_map(T, S)
        m = host(mp).reshape(teams, T, 5)
        for b in range(teams):
            assert np.array_equal(m[b], ref)
        assert np.all(host(hits) == teams * G)                       # every j once per group
        assert np.array_equal(host(owner), oracle.simd_owner(trip, S))  # Fig 8 owner
        assert np.all(host(totals) == float(trip))                   # reduction of the counts


def test_probe_generic_fallback(P):
    # 0-byte slots force the global fallback of the sharing space
    for S in (2, 4, 32):
        for sharing in (64, 2048, 16):
            _, hits, owner, totals = P.probe_mapping(5, 40, simdlen=S, mode="generic_smem",
                                                     sharing_bytes=sharing)
            assert np.all(host(hits) == 5 * 256 // S)
            assert np.array_equal(host(owner), oracle.simd_owner(40, S))
            assert np.all(host(totals) == 40.0)


# ------------------------------------------------------------------ a8 SpMV
@pytest.fixture(scope="module")
def cfg1():
    out = {}
    for spec in (R.CFG1, R.CFG1.integer()):
        rp, col, val, x = R.spmv_inputs(spec)
        y, a = oracle.spmv_csr_f64(rp, col, val, x)
        out[spec.values] = (rp, col, val, x, y, a)
    return out


@pytest.mark.parametrize("S", SIMDLENS)
@pytest.mark.parametrize("U", [1, 2, 4])
def test_spmv_cfg1_all_modes(P, cfg1, S, U):
    for values in ("int", "real"):
        rp, col, val, x, yref, aref = cfg1[values]
        t = [dev(rp), dev(col), dev(val), dev(x)]
        ys = {}
        for mode in MODES:
            for hints in (False, True):
                y = host(P.spmv_csr_f64(*t, simdlen=S, mode=mode, outer_unroll=U, stream_hints=hints))
                ys[(mode, hints)] = y
                if values == "int":
                    assert np.array_equal(bits(y), bits(yref)), (mode, hints)
                else:
                    assert_close(y, yref, aref, 1e-12)
        first = next(iter(ys.values()))
        for k, y in ys.items():
            assert np.array_equal(bits(y), bits(first)), f"mode/hints {k} differs bitwise"


@pytest.mark.parametrize("S", SIMDLENS)
def test_spmv_transpose_reduce_is_the_butterfly(P, cfg1, S):
    """SPMD with U loops in flight reduces all of them at once (engine.cuh
    transpose_reduce): the same pairs in the same order as the butterfly, so real
    results are bit-identical to U = 1 -- for SUM, MAX and MIN."""
    rp, col, val, x, _, _ = cfg1["real"]
    t = [dev(rp), dev(col), dev(val), dev(x)]
    for op in ("sum", "max", "min"):
        y1 = host(P.spmv_csr_f64(*t, simdlen=S, reduce=op, outer_unroll=1))
        for U in (2, 4):
            for T, blocked in ((256, False), (1024, True), (64, False)):
                y = host(P.spmv_csr_f64(*t, simdlen=S, reduce=op, outer_unroll=U, threads_per_team=T, blocked=blocked))
                assert np.array_equal(bits(y), bits(y1)), (op, U, T)


def test_spmv_unroll_and_simdlen_integer_invariance(P, cfg1):
    rp, col, val, x, yref, _ = cfg1["int"]
    t = [dev(rp), dev(col), dev(val), dev(x)]
    for S in SIMDLENS:
        for T in (32, 128, 512, 1024):
            for teams in (0, 1, 3):
                y = host(P.spmv_csr_f64(*t, simdlen=S, threads_per_team=T, num_teams=teams))
                assert np.array_equal(bits(y), bits(yref)), (S, T, teams)


@pytest.mark.parametrize("op", ["max", "min"])
def test_spmv_max_min(P, cfg1, op):
    rp, col, val, x, _, _ = cfg1["real"]
    yref, _ = oracle.spmv_csr_f64(rp, col, val, x, op=op)
    t = [dev(rp), dev(col), dev(val), dev(x)]
    for S in SIMDLENS:
        for mode in MODES:
            y = host(P.spmv_csr_f64(*t, simdlen=S, mode=mode, reduce=op))
            assert np.array_equal(y, yref), (S, mode)


def _rows_matrix(lens, ncols, seed):
    rng = np.random.default_rng(seed)
    rp = np.concatenate([[0], np.cumsum(lens)]).astype(np.int64)
    col = np.concatenate([np.sort(rng.choice(ncols, L, replace=False)) for L in lens] or [[]]).astype(np.int32)
    val = rng.integers(-4, 5, rp[-1]).astype(np.float64)
    x = rng.integers(-8, 9, ncols).astype(np.float64)
    return rp, col, val, x


def test_spmv_edge_rows(P):
    # empty rows, a lone row, tails for every S (33, 64 nnz), a long row, ragged count
    lens = [0, 0, 1, 33, 64, 0, 1000, 7, 31, 32, 5] * 7 + [2]
    rp, col, val, x = _rows_matrix(lens, 2000, 3)
    yref, _ = oracle.spmv_csr_f64(rp, col, val, x)
    t = [dev(rp), dev(col), dev(val), dev(x)]
    for S in SIMDLENS:
        for mode in MODES:
            for U in (1, 2, 4):
                for sharing in (0, 64):
                    y = host(P.spmv_csr_f64(*t, simdlen=S, mode=mode, outer_unroll=U, sharing_bytes=sharing))
                    assert np.array_equal(bits(y), bits(yref)), (S, mode, U, sharing)
    # empty rows give +0.0 and MAX gives -inf
    y = host(P.spmv_csr_f64(*t, simdlen=8, reduce="max"))
    assert y[0] == -np.inf


def test_spmv_zero_nnz_and_zero_rows(P):
    rp = np.zeros(6, np.int64)
    y = host(P.spmv_csr_f64(dev(rp), torch.zeros(0, dtype=torch.int32, device="cuda"),
                            torch.zeros(0, dtype=torch.float64, device="cuda"),
                            torch.zeros(3, dtype=torch.float64, device="cuda"), simdlen=4, mode="generic_smem"))
    assert np.all(y == 0) and not np.signbit(y).any()
    y0 = P.spmv_csr_f64(torch.zeros(1, dtype=torch.int64, device="cuda"),
                        torch.zeros(0, dtype=torch.int32, device="cuda"),
                        torch.zeros(0, dtype=torch.float64, device="cuda"),
                        torch.zeros(3, dtype=torch.float64, device="cuda"))
    assert y0.numel() == 0


def test_fallback_concurrent_streams(P, banded):
    """Generic-SMEM launches whose payload exceeds the slot use the library's global
    fallback; two of them in flight on different streams must not
    share slots (one scratch buffer per stream)."""
    rp, col, val, x, yref, aref = banded["int"]
    t = [dev(rp), dev(col), dev(val), dev(x)]
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
    torch.cuda.synchronize()
    ys = []
    for _ in range(4):
        for st in (s1, s2):
            y = torch.empty(rp.size - 1, dtype=torch.float64, device="cuda")
            P.spmv_csr_f64(*t, y, simdlen=2, mode="generic_smem", sharing_bytes=64, stream=st)
            ys.append(y)
    torch.cuda.synchronize()
    info = P.plan(rp.size - 1, 24, simdlen=2, mode="generic_smem", sharing_bytes=64)
    assert info["uses_global_fallback"] == 1
    for y in ys:
        assert np.array_equal(bits(host(y)), bits(yref))


def test_csr_validate(P, cfg1):
    rp, col, val, x, _, _ = cfg1["real"]
    assert P.csr_validate(dev(rp), dev(col), 1024) == 0
    bad = col.copy()
    bad[5] = 1024
    assert P.csr_validate(dev(rp), dev(bad), 1024) & 4
    rp2 = rp.copy()
    rp2[10] = rp2[12]
    assert P.csr_validate(dev(rp2), dev(col), 1024) & 2


def test_spmv_hostio_e2e(P, cfg1):
    rp, col, val, x, yref, aref = cfg1["real"]
    pin = lambda a: torch.from_numpy(np.ascontiguousarray(a)).pin_memory()
    hy = torch.empty(rp.size - 1, dtype=torch.float64).pin_memory()
    ws = torch.empty(P.hostio_workspace_bytes(rp.size - 1, x.size, val.size), dtype=torch.uint8, device="cuda")
    P.spmv_csr_f64_hostio(pin(rp), pin(col), pin(val), pin(x), hy, ws, simdlen=8)
    torch.cuda.synchronize()
    assert_close(hy.numpy(), yref, aref, 1e-12)


def test_spmv_cfg2_full_size_sampled(P):
    """BASELINE configs[1] at full size (10M rows) in the bench launch
    configurations; sampled rows compared against the oracle run on the same
    rows regenerated independently."""
    spec = R.CFG2
    rp, col, val = R.spmv_matrix(spec)
    x = R.spmv_x(spec)
    t = [dev(rp), dev(col), dev(val), dev(x)]
    rng = np.random.default_rng(7)
    starts = np.concatenate([[0, spec.nrows - 64], rng.integers(0, spec.nrows - 64, 30)])
    ref = {}
    for s in starts:
        rpl, cl, vl = R.spmv_matrix(spec, row_begin=int(s), nrows=64)
        ref[int(s)] = oracle.spmv_csr_f64(rpl, cl, vl, x)
    for S in SIMDLENS:
        for mode in MODES:
            for U, hints in ((1, False), (2, True), (4, True)):
                y = host(P.spmv_csr_f64(*t, simdlen=S, mode=mode, outer_unroll=U, stream_hints=hints))
                for s, (yr, ar) in ref.items():
                    assert_close(y[s:s + 64], yr, ar, 1e-12)
    # the bench's candidate set (bench.CANDIDATES: blocked teams of 1024, 128-bit pairs / quads, the
    # lean SPMD driver) including the headline and the simdlen-1 comparison point, plus team chunks
    for S, mode, flags, chunk in ((2, "spmd", "bv", 0), (1, "spmd", "bv", 0), (1, "spmd", "bq", 0),
                                  (2, "spmd", "bq", 0), (4, "spmd", "bv", 0), (2, "spmd", "b", 0),
                                  (1, "spmd", "b", 0), (2, "generic_smem", "b", 0), (2, "spmd", "bv", 2048),
                                  (8, "generic_shfl", "bv", 4096)):
        y = host(P.spmv_csr_f64(*t, simdlen=S, mode=mode, threads_per_team=1024, blocked="b" in flags,
                                vec128="v" in flags or "q" in flags, quad="q" in flags, team_chunk=chunk))
        for s, (yr, ar) in ref.items():
            assert_close(y[s:s + 64], yr, ar, 1e-12)
    del t
    torch.cuda.empty_cache()


def test_spmv_g100_and_uniform_full_size_sampled(P):
    """The 100M-nnz gate matrix (G100) and the all-far cfg2 variant at full size in
    the bench headline configuration: sampled 64-row windows against the oracle
    on the same rows regenerated independently (R3 tolerance)."""
    for spec in (R.G100, R.CFG2_UNIFORM):
        rp, col, val = R.spmv_matrix(spec)
        x = R.spmv_x(spec)
        t = [dev(rp), dev(col), dev(val), dev(x)]
        del rp, col, val
        rng = np.random.default_rng(11)
        starts = np.concatenate([[0, spec.nrows - 64], rng.integers(0, spec.nrows - 64, 16)])
        for S, flags in ((2, "bv"), (1, "bv")):
            y = host(P.spmv_csr_f64(*t, simdlen=S, threads_per_team=1024, blocked=True, vec128=True))
            for s in starts:
                rpl, cl, vl = R.spmv_matrix(spec, row_begin=int(s), nrows=64)
                yr, ar = oracle.spmv_csr_f64(rpl, cl, vl, x)
                assert_close(y[s:s + 64], yr, ar, 1e-12)
        del t
        torch.cuda.empty_cache()


# ------------------------------------------------------------------ a9 batched
@pytest.fixture(scope="module")
def batched():
    out = {}
    B = 777
    for values in ("int", "real"):
        A, x = R.batched_inputs(B, values=values)
        y, a = oracle.batched_matvec_f32(A, x, B)
        out[values] = (B, A, x, y, a)
    return out


@pytest.mark.parametrize("S", SIMDLENS)
@pytest.mark.parametrize("mode", MODES)
def test_batched(P, batched, S, mode):
    ys = []
    for values in ("int", "real"):
        B, A, x, yref, aref = batched[values]
        for U in (1, 2, 4):
            y = host(P.batched_matvec_f32(dev(A), dev(x), B, simdlen=S, mode=mode, outer_unroll=U))
            if values == "int":
                assert np.array_equal(bits(y), bits(yref))
            else:
                assert_close(y, yref, aref, 1e-5)
                ys.append(y)
    assert all(np.array_equal(bits(ys[0]), bits(v)) for v in ys)


@pytest.mark.parametrize("op", ["max", "min"])
def test_batched_max_min_and_rect(P, op):
    B, m, n = 300, 5, 37
    A, x = R.batched_inputs(B, m, n)
    yref, _ = oracle.batched_matvec_f32(A, x, B, m, n, op=op)
    for S in (1, 4, 32):
        y = host(P.batched_matvec_f32(dev(A), dev(x), B, m, n, simdlen=S, reduce=op, mode="generic_smem"))
        assert np.array_equal(y, yref)


# ------------------------------------------------------------------ a10 stencil
@pytest.mark.parametrize("L", R.STENCIL_LS + (1, 33))
@pytest.mark.parametrize("mode", MODES)
def test_stencil(P, L, mode):
    N = 4099
    for values in ("int", "real"):
        inp, coef, w = R.stencil_inputs(N, L, values=values)
        yref, aref, vref = oracle.nested_stencil_f64(inp, coef, w, N, L)
        t = [dev(inp), dev(coef), dev(w)]
        outs = []
        for S in SIMDLENS:
            for U in (1, 2):
                visits = torch.zeros(1, dtype=torch.int64, device="cuda")
                y = host(P.nested_stencil_f64(*t, N, L, visits=visits, simdlen=S, mode=mode, outer_unroll=U))
                assert int(visits.item()) == vref == N            # guarded side effect: once per i
                if values == "int":
                    assert np.array_equal(bits(y), bits(yref)), (S, U)
                else:
                    assert_close(y, yref, aref, 1e-12)
                outs.append(y)


def test_stencil_max_and_cfg3_full(P):
    N = 1 << 20
    for L in (4, 64):
        inp, coef, w = R.stencil_inputs(N, L)
        yref, aref, _ = oracle.nested_stencil_f64(inp, coef, w, N, L)
        t = [dev(inp), dev(coef), dev(w)]
        for S in (1, 8, 32):
            for mode in MODES:
                y = host(P.nested_stencil_f64(*t, N, L, simdlen=S, mode=mode))
                assert_close(y, yref, aref, 1e-12)
        ymax, _, _ = oracle.nested_stencil_f64(inp, coef, w, N, L, op="max")
        assert np.array_equal(host(P.nested_stencil_f64(*t, N, L, simdlen=16, reduce="max")), ymax)


# ------------------------------------------------------------------ a8 SpMV, x ring
@pytest.fixture(scope="module")
def banded():
    out = {}
    for values in ("int", "real"):
        spec = R.SpmvSpec("band", 4242, 50_000, 50_000, 0, 20, band_w=700, far_den=8, values=values)
        rp, col, val, x = R.spmv_inputs(spec)
        y, a = oracle.spmv_csr_f64(rp, col, val, x)
        out[values] = (rp, col, val, x, y, a)
    return out


# (x_halo, rows per group per round, T, num_teams, teams_per_sm, tuples: 0 scalar / 2 pairs / 4 quads)
RING_CASES = ((700, 1, 256, 0, 0, 0), (64, 2, 512, 0, 0, 2), (4096, 4, 256, 0, 0, 0),
              (1, 1, 768, 0, 2, 2), (700, 2, 256, 5, 0, 0), (3000, 1, 128, 1, 0, 2),
              (4096, 1, 1024, 0, 1, 2), (700, 1, 64, 3, 0, 0), (900, 1, 768, 0, 2, 4), (50, 2, 256, 7, 0, 4))


@pytest.mark.parametrize("S", SIMDLENS)
@pytest.mark.parametrize("mode", MODES)
def test_spmv_ring(P, banded, S, mode):
    """x ring (spmv_ring_kernel) against the oracle, and bit-identical to nest_kernel
    at the same simdlen, mode and loads (same per-lane order, R1/R20)."""
    for values in ("int", "real"):
        rp, col, val, x, yref, aref = banded[values]
        t = [dev(rp), dev(col), dev(val), dev(x)]
        ynest = {v: host(P.spmv_csr_f64(*t, simdlen=S, mode=mode, vec128=v > 0, quad=v == 4)) for v in (0, 2, 4)}
        for halo, U, T, teams, tps, vec in RING_CASES:
            cfg = dict(simdlen=S, mode=mode, outer_unroll=U, threads_per_team=T, x_halo=halo, num_teams=teams,
                       teams_per_sm=tps, vec128=vec > 0, quad=vec == 4)
            assert P.spmv_plan(rp.size - 1, x.size, val.size, **cfg)["kernel"] == 1
            y = host(P.spmv_csr_f64(*t, **cfg))
            if values == "int":
                assert np.array_equal(bits(y), bits(yref)), cfg
            else:
                assert_close(y, yref, aref, 1e-12)
            assert np.array_equal(bits(y), bits(ynest[vec])), cfg


@pytest.mark.parametrize("op", ["max", "min"])
def test_spmv_ring_max_min(P, banded, op):
    rp, col, val, x, _, _ = banded["real"]
    yref, _ = oracle.spmv_csr_f64(rp, col, val, x, op=op)
    t = [dev(rp), dev(col), dev(val), dev(x)]
    for S, mode, vec in ((1, "spmd", True), (4, "generic_smem", False), (32, "generic_shfl", True)):
        y = host(P.spmv_csr_f64(*t, simdlen=S, mode=mode, reduce=op, x_halo=700, vec128=vec, threads_per_team=512))
        assert np.array_equal(y, yref)


def test_spmv_ring_cfg1_and_rectangular(P, cfg1):
    rp, col, val, x, yref, aref = cfg1["int"]
    t = [dev(rp), dev(col), dev(val), dev(x)]
    for S in (1, 8, 32):
        for halo in (1, 100, 5000):
            y = host(P.spmv_csr_f64(*t, simdlen=S, x_halo=halo, mode="generic_smem", sharing_bytes=64))
            assert np.array_equal(bits(y), bits(yref))
    # more rows than columns: windows past the last column are empty
    rp2 = np.arange(0, 2 * 3000 + 1, 2, dtype=np.int64)
    col2 = np.tile(np.array([0, 3], np.int32), 3000)
    x2 = np.array([1.5, 0, 0, 2.0])
    y = host(P.spmv_csr_f64(dev(rp2), dev(col2), dev(np.ones(6000)), dev(x2), simdlen=2, x_halo=8))
    assert np.all(y == 3.5)


def test_spmv_ring_long_rows_and_odd_sizes(P):
    # rows far longer than a round's share, odd nnz / ncols (the copy engine's hand-copied
    # tails), empty matrices and empty rows, more teams than rows
    for lens, ncols in (([0, 3, 40000, 7, 1, 0, 25000, 5] * 3 + [1], 60001),
                        ([1] * 999 + [2], 1001), ([0] * 50, 7), ([3] * 5, 257)):
        rp, col, val, x = _rows_matrix(lens, ncols, 11)
        yref, _ = oracle.spmv_csr_f64(rp, col, val, x)
        t = [dev(rp), dev(col), dev(val), dev(x)]
        for S in (1, 4, 32):
            for mode in MODES:
                for halo, T, teams in ((3, 256, 0), (1000, 128, 0), (300, 1024, 40)):
                    for vec in (0, 2, 4):
                        y = host(P.spmv_csr_f64(*t, simdlen=S, mode=mode, x_halo=halo, threads_per_team=T,
                                                num_teams=teams, vec128=vec > 0, quad=vec == 4))
                        assert np.array_equal(bits(y), bits(yref)), (lens[:3], S, mode, halo, T, vec)


def test_spmv_ring_misaligned_rowptr_and_x(P, banded):
    """rowptr at an 8-byte (not 16-byte) offset: the copy engine copies the first
    entry of such a round by hand (no misaligned bulk copy); an
    unaligned x is refused before any launch."""
    rp, col, val, x, yref, _ = banded["int"]
    big = torch.from_numpy(np.concatenate([[0], rp])).cuda()
    rp_off = big[1:]
    assert rp_off.data_ptr() % 16 == 8
    for S, U, T in ((2, 1, 1024), (4, 2, 256), (1, 1, 128)):
        y = host(P.spmv_csr_f64(rp_off, dev(col), dev(val), dev(x), simdlen=S, x_halo=700, outer_unroll=U,
                                threads_per_team=T))
        assert np.array_equal(bits(y), bits(yref))
    xb = torch.from_numpy(np.concatenate([[0.0], x])).cuda()[1:]
    with pytest.raises(P.NestError) as e:
        P.spmv_csr_f64(dev(rp), dev(col), dev(val), xb, x_halo=700)
    assert e.value.status == 2


def test_spmv_ring_too_big_is_unsupported(P, cfg1):
    rp, col, val, x, _, _ = cfg1["int"]
    with pytest.raises(P.NestError) as e:
        P.spmv_csr_f64(dev(rp), dev(col), dev(val), dev(x), simdlen=1, threads_per_team=1024,
                       outer_unroll=4, x_halo=20000)
    assert e.value.status == 2
    with pytest.raises(P.NestError) as e:   # the copy warp needs a consumer warp beside it
        P.spmv_csr_f64(dev(rp), dev(col), dev(val), dev(x), x_halo=100, threads_per_team=32)
    assert e.value.status == 1


# ------------------------------------------------------------------ a8 SpMV, blocked team schedule
@pytest.mark.parametrize("S", SIMDLENS)
@pytest.mark.parametrize("mode", MODES)
def test_spmv_blocked(P, banded, S, mode):
    for values in ("int", "real"):
        rp, col, val, x, yref, aref = banded[values]
        t = [dev(rp), dev(col), dev(val), dev(x)]
        y0 = host(P.spmv_csr_f64(*t, simdlen=S, mode=mode))
        # team_chunk: round-robin team chunks (rounded up to a multiple of G)
        for U, T, teams, chunk in ((1, 1024, 0, 0), (2, 256, 0, 0), (4, 512, 7, 0), (1, 64, 1, 0),
                                   (1, 1024, 0, 1), (2, 256, 3, 100), (1, 128, 0, 3000), (4, 64, 5, 64)):
            y = host(P.spmv_csr_f64(*t, simdlen=S, mode=mode, outer_unroll=U, threads_per_team=T,
                                    num_teams=teams, blocked=True, team_chunk=chunk))
            # the schedule never changes a row's arithmetic: bit-identical to the cyclic run
            assert np.array_equal(bits(y), bits(y0)), (U, T, teams, chunk)
            if values == "int":
                assert np.array_equal(bits(y), bits(yref)), (U, T, teams, chunk)
            else:
                assert_close(y, yref, aref, 1e-12)
    # stencil and batched under the blocked schedule too (the flag is generic)
    N, L = 3001, 8
    inp, coef, w = R.stencil_inputs(N, L, values="int")
    yref, _, _ = oracle.nested_stencil_f64(inp, coef, w, N, L)
    visits = torch.zeros(1, dtype=torch.int64, device="cuda")
    for chunk in (0, 37, 1000):
        visits.zero_()
        y = host(P.nested_stencil_f64(dev(inp), dev(coef), dev(w), N, L, visits=visits, simdlen=S, mode=mode,
                                      blocked=True, team_chunk=chunk))
        assert np.array_equal(bits(y), bits(yref)) and int(visits.item()) == N, chunk


# ------------------------------------------------------------------ a8 SpMV, 128-bit pair loads
@pytest.mark.parametrize("S", SIMDLENS)
@pytest.mark.parametrize("mode", MODES)
def test_spmv_vec128(P, banded, cfg1, S, mode):
    for data in (banded, cfg1):
        for values in ("int", "real"):
            rp, col, val, x, yref, aref = data[values]
            t = [dev(rp), dev(col), dev(val), dev(x)]
            for U, T, blocked, quad in ((1, 256, False, False), (2, 1024, True, True), (4, 128, False, False),
                                        (1, 1024, True, False), (1, 512, False, True), (4, 256, True, True)):
                y = host(P.spmv_csr_f64(*t, simdlen=S, mode=mode, outer_unroll=U, threads_per_team=T,
                                        blocked=blocked, vec128=True, quad=quad))
                if values == "int":
                    assert np.array_equal(bits(y), bits(yref)), (U, T, blocked)
                else:
                    assert_close(y, yref, aref, 1e-12)


def test_spmv_vec128_odd_tails(P):
    # odd nnz (the last pair would read past the arrays), empty and 1-nnz rows
    for lens in ([1, 0, 3, 2, 5, 0, 1], [7] * 33, [0, 0, 1], [2, 1, 64, 33]):
        rp, col, val, x = _rows_matrix(lens, 200, 5)
        yref, _ = oracle.spmv_csr_f64(rp, col, val, x)
        t = [dev(rp), dev(col), dev(val), dev(x)]
        for S in SIMDLENS:
            for mode in MODES:
                for quad in (False, True):
                    y = host(P.spmv_csr_f64(*t, simdlen=S, mode=mode, vec128=True, quad=quad, sharing_bytes=64))
                    assert np.array_equal(bits(y), bits(yref)), (lens, S, mode, quad)
    rp, col, val, x = _rows_matrix([3, 4], 50, 6)
    dval = torch.from_numpy(np.concatenate([[0.0], val])).cuda()[1:]
    with pytest.raises(P.NestError) as e:
        P.spmv_csr_f64(dev(rp), dev(col), dval, dev(x), vec128=True)
    assert e.value.status == 2


@pytest.mark.parametrize("S", SIMDLENS)
@pytest.mark.parametrize("mode", MODES)
def test_batched_vec128(P, batched, S, mode):
    for values in ("int", "real"):
        B, A, x, yref, aref = batched[values]
        for U, T, blocked in ((1, 256, False), (2, 1024, True), (4, 128, False)):
            y = host(P.batched_matvec_f32(dev(A), dev(x), B, simdlen=S, mode=mode, outer_unroll=U,
                                          threads_per_team=T, blocked=blocked, vec128=True))
            if values == "int":
                assert np.array_equal(bits(y), bits(yref))
            else:
                assert_close(y, yref, aref, 1e-5)
    with pytest.raises(P.NestError):
        P.batched_matvec_f32(dev(A[: 3 * 64 * 62].copy()), dev(x[: 3 * 62].copy()), 3, 64, 62, vec128=True)


# ------------------------------------------------------------------ NEXT-2 laplace3d (no reduction)
@pytest.mark.parametrize("S", SIMDLENS)
@pytest.mark.parametrize("mode", MODES)
def test_laplace3d(P, S, mode):
    for (nz, ny, nx), values in (((9, 11, 37), "real"), ((5, 34, 66), "int"), ((3, 3, 3), "real"),
                                 ((2, 5, 5), "real")):
        u = R.laplace_inputs(nz, ny, nx, values=values)
        ref = oracle.laplace3d_f64(u, nz, ny, nx, 0.125)
        for U, blocked in ((1, False), (2, True), (4, False)):
            out = dev(u.copy())
            P.laplace3d_f64(dev(u), out, nz, ny, nx, 0.125, simdlen=S, mode=mode, outer_unroll=U, blocked=blocked)
            assert np.array_equal(bits(host(out)), bits(ref)), (nz, ny, nx, U, blocked)


# ------------------------------------------------------------------ NEXT-1 two-level teams-generic baseline
def test_spmv_teams_generic_baseline(P, cfg1, banded):
    for data in (cfg1, banded):
        for values in ("int", "real"):
            rp, col, val, x, yref, aref = data[values]
            t = [dev(rp), dev(col), dev(val), dev(x)]
            for T, teams in ((32, 0), (64, 0), (256, 0), (32, 7), (992, 0)):
                y = host(P.spmv_csr_f64(*t, simdlen=1, mode="teams_generic", threads_per_team=T, num_teams=teams))
                if values == "int":
                    assert np.array_equal(bits(y), bits(yref)), (T, teams)
                else:
                    assert_close(y, yref, aref, 1e-12)
    rp, col, val, x, _, _ = cfg1["real"]
    for op in ("max", "min"):
        yr, _ = oracle.spmv_csr_f64(rp, col, val, x, op=op)
        y = host(P.spmv_csr_f64(dev(rp), dev(col), dev(val), dev(x), simdlen=1, mode="teams_generic", reduce=op))
        assert np.array_equal(y, yr)
    with pytest.raises(P.NestError):
        P.spmv_csr_f64(dev(rp), dev(col), dev(val), dev(x), simdlen=2, mode="teams_generic")
    lens = [0, 0, 1, 33, 64, 0, 1000, 7] * 5
    rp2, col2, val2, x2 = _rows_matrix(lens, 2000, 9)
    yr2, _ = oracle.spmv_csr_f64(rp2, col2, val2, x2)
    y2 = host(P.spmv_csr_f64(dev(rp2), dev(col2), dev(val2), dev(x2), simdlen=1, mode="teams_generic"))
    assert np.array_equal(bits(y2), bits(yr2))


# ------------------------------------------------------------------ a10 stencil, 128-bit pairs
@pytest.mark.parametrize("L", (2, 4, 8, 16, 32, 64, 34))
@pytest.mark.parametrize("mode", MODES)
def test_stencil_vec128(P, L, mode):
    """Pair tuples (NEST_F_VEC128): integer data bit-exact against the oracle,
    real data within R3; every simdlen, U = 1/2; the guarded visit count once per i."""
    N = 4099
    for values in ("int", "real"):
        inp, coef, w = R.stencil_inputs(N, L, values=values)
        yref, aref, vref = oracle.nested_stencil_f64(inp, coef, w, N, L)
        t = [dev(inp), dev(coef), dev(w)]
        for S in SIMDLENS:
            for U in (1, 2):
                visits = torch.zeros(1, dtype=torch.int64, device="cuda")
                y = host(P.nested_stencil_f64(*t, N, L, visits=visits, simdlen=S, mode=mode, outer_unroll=U,
                                              vec128=True))
                assert int(visits.item()) == vref == N
                if values == "int":
                    assert np.array_equal(bits(y), bits(yref)), (S, U)
                else:
                    assert_close(y, yref, aref, 1e-12)


def test_stencil_vec128_full_and_rejects(P):
    N = 1 << 20
    for L in (4, 64):
        inp, coef, w = R.stencil_inputs(N, L)
        yref, aref, _ = oracle.nested_stencil_f64(inp, coef, w, N, L)
        t = [dev(inp), dev(coef), dev(w)]
        for S in (2, 8, 32):
            y = host(P.nested_stencil_f64(*t, N, L, simdlen=S, vec128=True))
            assert_close(y, yref, aref, 1e-12)
        ymax, _, _ = oracle.nested_stencil_f64(inp, coef, w, N, L, op="max")
        assert np.array_equal(host(P.nested_stencil_f64(*t, N, L, simdlen=16, reduce="max", vec128=True)), ymax)
    inp, coef, w = R.stencil_inputs(64, 3)
    with pytest.raises(Exception, match="even L"):
        P.nested_stencil_f64(dev(inp), dev(coef), dev(w), 64, 3, vec128=True)


@pytest.mark.parametrize("S", SIMDLENS)
@pytest.mark.parametrize("mode", MODES)
def test_laplace3d_vec128(P, S, mode):
    """Aligned pairs over whole lines (NEST_F_VEC128, even nx): bit-identical to the
    oracle, boundary points untouched."""
    for (nz, ny, nx), values in (((9, 11, 38), "real"), ((5, 34, 66), "int"), ((3, 3, 4), "real"),
                                 ((4, 5, 2), "real"), ((6, 7, 130), "real")):
        u = R.laplace_inputs(nz, ny, nx, values=values)
        ref = oracle.laplace3d_f64(u, nz, ny, nx, 0.125)
        for U, blocked in ((1, False), (2, True), (4, False)):
            out = dev(u.copy())
            P.laplace3d_f64(dev(u), out, nz, ny, nx, 0.125, simdlen=S, mode=mode, outer_unroll=U, blocked=blocked,
                            vec128=True)
            assert np.array_equal(bits(host(out)), bits(ref)), (nz, ny, nx, U, blocked)


def test_laplace3d_vec128_rejects_odd_nx(P):
    u = R.laplace_inputs(4, 4, 5)
    with pytest.raises(Exception, match="even nx"):
        P.laplace3d_f64(dev(u), dev(u.copy()), 4, 4, 5, 0.125, vec128=True)


# ------------------------------------------------------------------ a8 SpMV, x persisting in L2
@pytest.mark.parametrize("S", (1, 2, 8))
def test_spmv_x_l2_persist_is_a_cache_policy_only(P, banded, cfg1, S):
    # NEST_F_X_L2_PERSIST changes where x lives in L2, never a result: bit-identical to the
    # same launch without it, and to the oracle (integer data) / within R3 (real data)
    for data in (banded, cfg1):
        for values in ("int", "real"):
            rp, col, val, x, yref, aref = data[values]
            t = [dev(rp), dev(col), dev(val), dev(x)]
            for cfg in (dict(), dict(blocked=True, threads_per_team=1024, vec128=True, quad=True),
                        dict(blocked=True, vec128=True, mode="generic_smem"), dict(outer_unroll=2, mode="generic_shfl")):
                y0 = host(P.spmv_csr_f64(*t, simdlen=S, **cfg))
                y1 = host(P.spmv_csr_f64(*t, simdlen=S, x_l2_persist=True, **cfg))
                assert np.array_equal(bits(y1), bits(y0)), cfg
                if values == "int":
                    assert np.array_equal(bits(y1), bits(yref)), cfg
                else:
                    assert_close(y1, yref, aref, 1e-12)


def test_spmv_x_l2_persist_with_the_x_ring(P, banded):
    # the x ring (shared staging of x) takes the window too: same bits
    rp, col, val, x, yref, aref = banded["int"]
    t = [dev(rp), dev(col), dev(val), dev(x)]
    for S, vec, quad in ((2, True, False), (4, False, False), (2, True, True)):
        cfg = dict(simdlen=S, x_halo=700, threads_per_team=768, vec128=vec, quad=quad)
        y0 = host(P.spmv_csr_f64(*t, **cfg))
        y1 = host(P.spmv_csr_f64(*t, x_l2_persist=True, **cfg))
        assert np.array_equal(bits(y1), bits(y0)) and np.array_equal(bits(y1), bits(yref)), cfg
    info = P.spmv_plan(rp.size - 1, x.size, val.size, simdlen=2, x_halo=700, threads_per_team=768,
                       x_l2_persist=True)
    assert info["kernel"] == 1 and info["l2_window_bytes"] == x.size * 8


def test_spmv_x_l2_persist_plan_and_flush(P, banded):
    rp, col, val, x, yref, aref = banded["real"]
    n = rp.size - 1
    info = P.spmv_plan(n, x.size, val.size, simdlen=2, blocked=True, threads_per_team=1024, vec128=True, quad=True,
                       x_l2_persist=True)
    props = torch.cuda.get_device_properties(0)
    assert info["l2_window_bytes"] == x.size * 8           # x (400 KB) is under the window whole
    assert 0 < info["l2_setaside_bytes"] <= props.L2_cache_size
    plain = P.spmv_plan(n, x.size, val.size, simdlen=2)
    assert plain["l2_window_bytes"] == 0 and plain["l2_setaside_bytes"] == 0
    # the flush utility returns persisting lines to normal and still flushes
    t = [dev(rp), dev(col), dev(val), dev(x)]
    buf = torch.empty(64 << 20, dtype=torch.uint8, device="cuda")
    for _ in range(3):
        y = P.spmv_csr_f64(*t, simdlen=2, blocked=True, threads_per_team=1024, vec128=True, quad=True,
                           x_l2_persist=True)
        P.l2_flush(buf)
    torch.cuda.synchronize()
    assert_close(host(y), yref, aref, 1e-12)
    # the hostio (end-to-end) call takes the flag too: bit-identical to the device call
    h = [torch.from_numpy(a).pin_memory() for a in (rp, col, val, x)]
    h_y = torch.empty(n, dtype=torch.float64).pin_memory()
    ws = torch.empty(P.hostio_workspace_bytes(n, x.size, val.size), dtype=torch.uint8, device="cuda")
    P.spmv_csr_f64_hostio(*h, h_y, ws, simdlen=2, blocked=True, threads_per_team=1024, vec128=True, quad=True,
                          x_l2_persist=True)
    torch.cuda.synchronize()
    assert np.array_equal(bits(h_y.numpy()), bits(host(y)))
    # nest_shutdown restores the persisting-L2 limit the library raised (0 on a fresh context)
    from cuda.bindings import runtime as rt
    lim = lambda: rt.cudaDeviceGetLimit(rt.cudaLimit.cudaLimitPersistingL2CacheSize)[1]
    during = lim()
    assert during > 0 and info["l2_setaside_bytes"] > 0
    P.shutdown()
    assert lim() < during


def test_c_example_runs(P):
    # examples/spmv_c.c: the headline and a generic-SMEM configuration through the C ABI from
    # plain C, bit-exact against a C loop on integer-valued data (exit status 0)
    import os
    import subprocess
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    assert subprocess.run(["make", "-C", root, "examples/spmv_c"], capture_output=True).returncode == 0
    r = subprocess.run([os.path.join(root, "examples", "spmv_c")], capture_output=True, text=True, timeout=300)
    assert r.returncode == 0, r.stdout + r.stderr
    assert r.stdout.count(": 0 mismatching rows") == 2, r.stdout
