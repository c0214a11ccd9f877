"""NEXT-4b on one GPU: the symmetric x (every rank's slice mapped into one virtual
range with CUDA virtual memory), so the row-partitioned SpMV is the ordinary kernel on
a contiguous x.

* single process, P slices (nest_xsym_create_local): every shard's y is bit-identical
  to the single-GPU SpMV's rows for every variant (same kernel, same x values) and
  bit-exact against the oracle on integer data;
* two processes on the same GPU exchanging the slices' POSIX file descriptors over a
  unix socket (the multi-GPU code path, minus NVLink), x rewritten between iterations
  (sync + process barrier order the writes and the gathers)."""
import os
import socket

import numpy as np
import pytest

import oracle
from nestgen import recipes as R

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def P():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_icpp_wrightdtcc23_b200 as P
    return P


def bits(a):
    return np.ascontiguousarray(a).view(np.int64)


def fill(P, xs, x):
    for r in range(xs.nranks):
        lo = r * xs.xchunk
        if lo < x.size:
            xs.set_x(torch.from_numpy(x[lo:lo + xs.xchunk].copy()).cuda(), rank=r)
    torch.cuda.synchronize()


def test_xsym_slices_of_any_size(P):
    # slice sizes that are not powers of two (the reservation is granule-aligned)
    for ncols, nranks in ((12_500_000, 8), (3 * (1 << 18) + 5, 3), (1, 1)):
        xs = P.XSym(ncols, nranks=nranks)
        assert xs.xchunk * nranks >= ncols and xs.x_ptr() % 256 == 0
        xs.close()


@pytest.mark.parametrize("nranks", [1, 2, 3, 8])
def test_xsym_local_slices_match_single_gpu(P, nranks):
    spec = R.SpmvSpec("xs", 781, 300_007, 300_007, 0, 17, band_w=3000, far_den=4, values="int")
    rp, col, val, x = R.spmv_inputs(spec)
    yref, _ = oracle.spmv_csr_f64(rp, col, val, x)
    d = [torch.from_numpy(a).cuda() for a in (rp, col, val, x)]
    xs = P.XSym(spec.ncols, nranks=nranks)
    assert xs.xchunk * nranks >= spec.ncols
    fill(P, xs, x)
    for cfg in (dict(simdlen=2, quad=True, blocked=True, threads_per_team=1024, x_l2_persist=True),
                dict(simdlen=8, mode="generic_smem"), dict(simdlen=1, vec128=True, blocked=True),
                dict(simdlen=4, x_halo=700, threads_per_team=512)):
        y1 = P.spmv_csr_f64(*d, **cfg).cpu().numpy()
        for r in range(nranks):
            _, rb, nloc = P.shard_rows(spec.nrows, nranks, r)
            lrp, lcol, lval = R.spmv_matrix(spec, row_begin=rb, nrows=nloc)
            t = [torch.from_numpy(a).cuda() for a in (lrp, lcol, lval)]
            y = xs.spmv_csr_f64(*t, **cfg).cpu().numpy()
            tup = 4 if cfg.get("quad") else 2 if cfg.get("vec128") else 1
            if rp[rb] % tup == 0:   # tuples follow the local nonzero numbering (R16)
                assert np.array_equal(bits(y), bits(y1[rb:rb + nloc])), (cfg, r)
            assert np.array_equal(bits(y), bits(yref[rb:rb + nloc])), (cfg, r)
    xs.close()


def test_xsym_rejects_bad_arguments(P):
    from paper_conf_icpp_wrightdtcc23_b200 import _nest as N
    import ctypes
    h = ctypes.c_void_p()
    assert N.nest_xsym_create_local(0, 100, ctypes.byref(h)) == N.NEST_ERR_INVALID_ARG
    fd = ctypes.c_int32()
    assert N.nest_xsym_create(2, 2, 100, ctypes.byref(h), ctypes.byref(fd)) == N.NEST_ERR_INVALID_ARG
    assert N.nest_xsym_x(None) is None and N.nest_xsym_xchunk(None) == 0
    xs = P.XSym(1000, nranks=2)
    with pytest.raises(P.NestError):   # a local object is already mapped: no FD import
        P.check(N.nest_xsym_open(xs._h, (ctypes.c_int32 * 2)(0, 0)), "nest_xsym_open")
    xs.close()


def _port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, nranks, port, q):
    import torch.distributed as dist

    import paper_conf_icpp_wrightdtcc23_b200 as P
    try:
        torch.cuda.set_device(0)
        os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
        dist.init_process_group("gloo", rank=rank, world_size=nranks)
        spec = R.SpmvSpec("xs2", 783, 600_011, 600_011, 0, 12, band_w=2_000, far_den=3)
        x = R.spmv_x(spec)
        _, rb, nloc = P.shard_rows(spec.nrows, nranks, rank)
        lrp, lcol, lval = R.spmv_matrix(spec, row_begin=rb, nrows=nloc)
        xs = P.XSym(spec.ncols, tag=f"t{port}")
        lo = rank * xs.xchunk
        t = [torch.from_numpy(a).cuda() for a in (lrp, lcol, lval)]
        full = [torch.from_numpy(a).cuda() for a in R.spmv_matrix(spec)]
        for it in range(3):   # x changes between iterations
            xv = x * (it + 1)
            if lo < xv.size:
                xs.set_x(torch.from_numpy(xv[lo:lo + xs.xchunk].copy()).cuda())
            torch.cuda.synchronize()
            dist.barrier()   # every slice written before any rank gathers
            y = xs.spmv_csr_f64(*t, simdlen=2, quad=True, blocked=True, threads_per_team=1024).cpu().numpy()
            y1 = P.spmv_csr_f64(*full, torch.from_numpy(xv).cuda(), simdlen=8).cpu().numpy()
            yr, ar = oracle.spmv_csr_f64(lrp, lcol, lval, xv)
            assert np.all(np.abs(y - yr) <= 1e-12 * ar), (rank, it)
            assert np.all(np.abs(y - y1[rb:rb + nloc]) <= 2e-12 * ar), (rank, it)
            torch.cuda.synchronize()
            dist.barrier()   # every rank done gathering before the slices are rewritten
        xs.close()
        dist.destroy_process_group()
        q.put((rank, "ok"))
    except Exception as e:  # reported to the parent
        q.put((rank, repr(e)))


def test_xsym_two_processes_one_gpu(P):
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=240) for _ in procs)
    for p in procs:
        p.join(timeout=60)
    assert res == {0: "ok", 1: "ok"}, res
