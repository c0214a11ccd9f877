"""Property-based GPU parity (hypothesis, derandomised): random small CSR matrices with
integer data (exact in fp64, so the bar is bit-exactness, R4) against the
oracle, under random launch configurations -- simdlen, mode, team size, outer unroll,
schedule (cyclic / blocked / team chunks), loads (scalar / pairs / quads), explicit
team counts, small sharing spaces (global fallback), the x ring and the persisting
window.  Configurations the library rejects as NEST_ERR_UNSUPPORTED (a variant's
register-limited team size) are skipped; anything else must match bit for bit."""
import numpy as np
import pytest
from hypothesis import assume, given, settings, strategies as st

import oracle

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

SET = settings(max_examples=600, deadline=None, derandomize=True)


@pytest.fixture(scope="module")
def P():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_icpp_wrightdtcc23_b200 as P
    return P


@st.composite
def int_csr(draw):
    nrows = draw(st.integers(0, 3000))
    ncols = draw(st.integers(1, 5000))
    long_rows = draw(st.booleans())
    seed = draw(st.integers(0, 2**32 - 1))
    rng = np.random.default_rng(seed)
    lens = rng.integers(0, 80 if long_rows else 14, nrows)
    lens = np.minimum(lens, ncols)
    rp = np.zeros(nrows + 1, np.int64)
    rp[1:] = np.cumsum(lens)
    col = np.empty(int(rp[-1]), np.int32)
    for i in range(nrows):
        col[rp[i]:rp[i + 1]] = np.sort(rng.choice(ncols, int(lens[i]), replace=False))
    val = rng.integers(-7, 8, col.size).astype(np.float64)
    x = rng.integers(-7, 8, ncols).astype(np.float64)
    return rp, col, val, x


@st.composite
def launch(draw):
    S = draw(st.sampled_from([1, 2, 4, 8, 16, 32]))
    cfg = dict(simdlen=S, mode=draw(st.sampled_from(["spmd", "generic_smem", "generic_shfl"])),
               threads_per_team=draw(st.sampled_from([32, 64, 128, 256, 512, 768, 1024])),
               outer_unroll=draw(st.sampled_from([1, 1, 2, 4])),
               sharing_bytes=draw(st.sampled_from([0, 0, 64, 256])),
               num_teams=draw(st.sampled_from([0, 0, 1, 3, 7])))
    loads = draw(st.sampled_from(["scalar", "pairs", "quads"]))
    cfg["vec128"], cfg["quad"] = loads != "scalar", loads == "quads"
    kind = draw(st.sampled_from(["cyclic", "blocked", "chunks", "ring", "persist"]))
    if kind == "blocked":
        cfg["blocked"] = True
    elif kind == "chunks":
        cfg.update(blocked=True, team_chunk=draw(st.sampled_from([1, 64, 1000])))
    elif kind == "ring":
        cfg["x_halo"] = draw(st.sampled_from([1, 64, 700]))
        cfg["threads_per_team"] = max(64, cfg["threads_per_team"])
        cfg["x_l2_persist"] = draw(st.booleans())
    else:
        cfg.update(blocked=draw(st.booleans()), x_l2_persist=kind == "persist")
    return cfg


def bits(a):
    return np.ascontiguousarray(a).view(np.int64)


@SET
@given(int_csr(), launch())
def test_spmv_random_matrices_and_launches_bit_exact(P, m, cfg):
    rp, col, val, x = m
    yref, _ = oracle.spmv_csr_f64(rp, col, val, x)
    t = [torch.from_numpy(a).cuda() for a in (rp, col, val, x)]
    try:
        y = P.spmv_csr_f64(*t, **cfg).cpu().numpy()
    except P.NestError as e:
        assume(e.status != P._nest.NEST_ERR_UNSUPPORTED)
        raise
    assert np.array_equal(bits(y), bits(yref)), cfg


@SET
@given(int_csr(), st.sampled_from(["max", "min"]), launch())
def test_spmv_random_max_min(P, m, op, cfg):
    rp, col, val, x = m
    yref, _ = oracle.spmv_csr_f64(rp, col, val, x, op=op)
    t = [torch.from_numpy(a).cuda() for a in (rp, col, val, x)]
    try:
        y = P.spmv_csr_f64(*t, reduce=op, **cfg).cpu().numpy()
    except P.NestError as e:
        assume(e.status != P._nest.NEST_ERR_UNSUPPORTED)
        raise
    assert np.array_equal(y, yref), cfg   # by value: the sign of a zero tie is unordered (R17)


@st.composite
def body_launch(draw):
    S = draw(st.sampled_from([1, 2, 4, 8, 16, 32]))
    return dict(simdlen=S, mode=draw(st.sampled_from(["spmd", "generic_smem", "generic_shfl"])),
                threads_per_team=draw(st.sampled_from([32, 128, 256, 512, 1024])),
                outer_unroll=draw(st.sampled_from([1, 1, 2, 4])),
                sharing_bytes=draw(st.sampled_from([0, 0, 64])),
                num_teams=draw(st.sampled_from([0, 0, 1, 5])),
                blocked=draw(st.booleans()), vec128=draw(st.booleans()))


def _run(P, fn):
    try:
        return fn()
    except P.NestError as e:
        assume(e.status != P._nest.NEST_ERR_UNSUPPORTED)
        raise


@settings(max_examples=300, deadline=None, derandomize=True)
@given(st.integers(0, 5000), st.integers(1, 70), st.integers(0, 2**32 - 1), body_launch())
def test_stencil_random_bit_exact_and_visits(P, N, L, seed, cfg):
    # a10: integer data (exact), the guarded side effect counted once per outer iteration
    from nestgen import recipes as R
    if cfg["vec128"] and L % 2:
        L += 1
    inp, coef, w = R.stencil_inputs(N, L, values="int", cfg_seed=seed % 100000)
    yref, _, vref = oracle.nested_stencil_f64(inp, coef, w, N, L)
    visits = torch.zeros(1, dtype=torch.int64, device="cuda")
    t = [torch.from_numpy(a).cuda() for a in (inp, coef, w)]
    out = _run(P, lambda: P.nested_stencil_f64(*t, N, L, visits=visits, **cfg)).cpu().numpy()
    assert np.array_equal(bits(out), bits(yref)) and int(visits.item()) == vref == N, cfg


@settings(max_examples=200, deadline=None, derandomize=True)
@given(st.integers(0, 400), st.sampled_from([1, 3, 16, 64]), st.sampled_from([4, 8, 36, 64]),
       st.integers(0, 2**32 - 1), body_launch())
def test_batched_random_bit_exact(P, B, m, n, seed, cfg):
    # a9: integer data (partial sums < 2^24: exact in fp32), any m x n
    from nestgen import recipes as R
    A, x = R.batched_inputs(B, m, n, values="int", cfg_seed=seed % 100000)
    yref, _ = oracle.batched_matvec_f32(A, x, B, m, n)
    y = _run(P, lambda: P.batched_matvec_f32(torch.from_numpy(A).cuda(), torch.from_numpy(x).cuda(), B, m, n,
                                             **cfg)).cpu().numpy()
    assert np.array_equal(y.view(np.int32), yref.view(np.int32)), cfg


@settings(max_examples=150, deadline=None, derandomize=True)
@given(st.integers(1, 12), st.integers(1, 12), st.integers(1, 70), st.integers(0, 2**32 - 1), body_launch())
def test_laplace_random_bit_exact(P, nz, ny, nx, seed, cfg):
    # NEXT-2 (R21): bit-identical to the oracle, boundary points untouched
    from nestgen import recipes as R
    if cfg["vec128"] and nx % 2:
        nx += 1
    u = R.laplace_inputs(nz, ny, nx, values="real", cfg_seed=seed % 100000)
    ref = oracle.laplace3d_f64(u, nz, ny, nx, 0.125)
    out = torch.from_numpy(u.copy()).cuda()
    _run(P, lambda: P.laplace3d_f64(torch.from_numpy(u).cuda(), out, nz, ny, nx, 0.125, **cfg))
    assert np.array_equal(bits(out.cpu().numpy()), bits(ref)), cfg


@settings(max_examples=120, deadline=None, derandomize=True)
@given(int_csr(), st.integers(1, 8), st.sampled_from([1, 2, 4, 8, 32]),
       st.sampled_from(["spmd", "generic_smem", "generic_shfl"]), st.booleans(), st.booleans())
def test_xpeer_random_virtual_ranks(P, m, nranks, S, mode, vec, blocked):
    # NEXT-4 on virtual ranks: every rank's rows, gathering x from the owners' slices,
    # bit-exact against the oracle (integer data)
    rp, col, val, x = m
    n = rp.size - 1
    ncols = x.size
    yref, _ = oracle.spmv_csr_f64(rp, col, val, x)
    xc = P.x_chunk(ncols, nranks)
    sl = []
    for r in range(nranks):
        s = torch.zeros(max(xc, 1), dtype=torch.float64, device="cuda")
        b, k = P.local_x_range(ncols, nranks, r)
        if k > 0:
            s[:k] = torch.from_numpy(x[b:b + k]).cuda()
        sl.append(s)
    for r in range(nranks):
        _, rb, nloc = P.shard_rows(n, nranks, r)
        lrp = rp[rb:rb + nloc + 1] - rp[rb]
        t = [torch.from_numpy(np.ascontiguousarray(a)).cuda()
             for a in (lrp, col[rp[rb]:rp[rb + nloc]], val[rp[rb]:rp[rb + nloc]])]
        xp = P.XPeer(ncols, nranks=nranks, rank=r, local_slices=sl)
        try:
            y = _run(P, lambda: xp.spmv_csr_f64(n, *t, simdlen=S, mode=mode, vec128=vec, blocked=blocked))
        finally:
            xp.close()
        assert np.array_equal(bits(y.cpu().numpy()), bits(yref[rb:rb + nloc])), (nranks, r, S, mode, vec)


@settings(max_examples=80, deadline=None, derandomize=True)
@given(int_csr(), st.integers(1, 8), launch())
def test_xsym_random_virtual_ranks(P, m, nranks, cfg):
    # NEXT-4b: every shard's rows on the symmetric x (any variant), bit-exact vs the oracle
    rp, col, val, x = m
    n = rp.size - 1
    yref, _ = oracle.spmv_csr_f64(rp, col, val, x)
    xs = P.XSym(x.size, nranks=nranks)
    try:
        for r in range(nranks):
            lo = r * xs.xchunk
            if lo < x.size:
                xs.set_x(torch.from_numpy(x[lo:lo + xs.xchunk].copy()).cuda(), rank=r)
        torch.cuda.synchronize()
        for r in range(nranks):
            _, rb, nloc = P.shard_rows(n, nranks, r)
            lrp = rp[rb:rb + nloc + 1] - rp[rb]
            t = [torch.from_numpy(np.ascontiguousarray(a)).cuda()
                 for a in (lrp, col[rp[rb]:rp[rb + nloc]], val[rp[rb]:rp[rb + nloc]])]
            y = _run(P, lambda: xs.spmv_csr_f64(*t, **cfg))
            assert np.array_equal(bits(y.cpu().numpy()), bits(yref[rb:rb + nloc])), (nranks, r, cfg)
    finally:
        xs.close()
