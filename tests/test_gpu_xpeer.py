"""NEXT-4 on one GPU: the comm-free row-partitioned SpMV (x gathered from the
owning rank's slice, no all-gather).

* single process, P "ranks" whose x slices are separate device buffers
  (nest_xpeer_create_local): every rank's y_local is bit-identical to the
  single-GPU SpMV's rows at the same (simdlen, mode, variant) (R16)
  and within the R3 bound of the oracle;
* two processes on the same GPU exchanging CUDA IPC handles over a gloo
  process group, with the peer-memory flag barrier (the multi-GPU code path,
  minus NVLink)."""
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


def slices_of(P, x, ncols, nranks):
    xc = P.x_chunk(ncols, nranks)
    out = []
    for r in range(nranks):
        s = torch.zeros(max(xc, 1), dtype=torch.float64, device="cuda")
        b, n = P.local_x_range(ncols, nranks, r)
        if n > 0:
            s[:n] = torch.from_numpy(x[b:b + n]).cuda()
        out.append(s)
    return out


@pytest.mark.parametrize("values", ["int", "real"])
@pytest.mark.parametrize("nranks", [1, 2, 3, 8])
def test_xpeer_virtual_ranks_match_single_gpu(P, values, nranks):
    spec = R.SpmvSpec("xp", 777, 30_011, 30_011, 0, 17, band_w=300, far_den=4, values=values)
    rp, col, val, x = R.spmv_inputs(spec)
    yref, aref = oracle.spmv_csr_f64(rp, col, val, x)
    d = [torch.from_numpy(a).cuda() for a in (rp, col, val, x)]
    sl = slices_of(P, x, spec.ncols, nranks)
    for S, mode, fl in ((1, "spmd", {}), (2, "spmd", dict(vec128=True, blocked=True, threads_per_team=1024)),
                        (8, "generic_smem", {}), (4, "generic_shfl", dict(blocked=True, team_chunk=700)),
                        (32, "spmd", dict(vec128=True)), (16, "generic_smem", dict(outer_unroll=2))):
        y1 = P.spmv_csr_f64(*d, simdlen=S, mode=mode, **fl).cpu().numpy()
        for r in range(nranks):
            _, rb, nloc = P.shard_rows(spec.nrows, nranks, r)
            lrp, lcol, lval = R.spmv_matrix(spec, row_begin=rb, nrows=nloc)
            xp = P.XPeer(spec.ncols, nranks=nranks, rank=r, local_slices=sl)
            t = [torch.from_numpy(a).cuda() for a in (lrp, lcol, lval)]
            y = xp.spmv_csr_f64(spec.nrows, *t, simdlen=S, mode=mode, **fl).cpu().numpy()
            xp.close()
            # R16: bit-identical to the single-GPU rows -- except that the 128-bit
            # pair tuples follow the LOCAL nonzero numbering, so a shard starting at
            # an odd global nonzero offset pairs differently (rounding order only)
            if not fl.get("vec128") or rp[rb] % 2 == 0 or values == "int":
                assert np.array_equal(bits(y), bits(y1[rb:rb + nloc])), (S, mode, fl, r)
            if values == "int":
                assert np.array_equal(bits(y), bits(yref[rb:rb + nloc]))
            else:
                assert np.all(np.abs(y - yref[rb:rb + nloc]) <= 1e-12 * aref[rb:rb + nloc])


def test_xpeer_odd_chunks_and_errors(P):
    # ncols not a multiple of nranks (short tail slice), chunk sizes that are not powers of two
    spec = R.SpmvSpec("xp2", 778, 1_000_003, 1_000_003, 1, 9, band_w=50_000, far_den=2)
    rp, col, val, x = R.spmv_inputs(spec)
    d = [torch.from_numpy(a).cuda() for a in (rp, col, val, x)]
    y1 = P.spmv_csr_f64(*d, simdlen=4).cpu().numpy()
    nranks = 7
    sl = slices_of(P, x, spec.ncols, nranks)
    for r in (0, 6):
        _, rb, nloc = P.shard_rows(spec.nrows, nranks, r)
        lrp, lcol, lval = R.spmv_matrix(spec, row_begin=rb, nrows=nloc)
        t = [torch.from_numpy(a).cuda() for a in (lrp, lcol, lval)]
        xp = P.XPeer(spec.ncols, nranks=nranks, rank=r, local_slices=sl)
        y = xp.spmv_csr_f64(spec.nrows, *t, simdlen=4).cpu().numpy()
        assert np.array_equal(bits(y), bits(y1[rb:rb + nloc]))
        with pytest.raises(P.NestError):          # wrong local row count
            xp.spmv_csr_f64(spec.nrows + 50, *t)
        with pytest.raises(P.NestError):          # the x ring is not offered here
            xp.spmv_csr_f64(spec.nrows, *t, x_halo=100, threads_per_team=256)
        with pytest.raises(P.NestError) as e:     # nor the persisting window (x is distributed)
            xp.spmv_csr_f64(spec.nrows, *t, x_l2_persist=True)
        assert e.value.status == P._nest.NEST_ERR_UNSUPPORTED
        xp.close()


def _port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _ipc_worker(rank, nranks, port, q):
    import torch.distributed as dist

    import paper_conf_icpp_wrightdtcc23_b200 as P
    try:
        torch.cuda.set_device(0)
        os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
        dist.init_process_group("gloo", rank=rank, world_size=nranks)
        spec = R.SpmvSpec("xp3", 779, 40_000, 40_000, 0, 12, band_w=2_000, far_den=3)
        x = R.spmv_x(spec)
        _, rb, nloc = P.shard_rows(spec.nrows, nranks, rank)
        lrp, lcol, lval = R.spmv_matrix(spec, row_begin=rb, nrows=nloc)
        xp = P.XPeer(spec.ncols)
        b, n = P.local_x_range(spec.ncols, nranks, rank)
        for it in range(3):   # x changes between iterations: the barriers order writes and gathers
            xs = x * (it + 1)
            xp.set_local_x(torch.from_numpy(xs[b:b + n].copy()).cuda())
            t = [torch.from_numpy(a).cuda() for a in (lrp, lcol, lval)]
            y = xp.spmv_csr_f64(spec.nrows, *t, simdlen=8, mode="generic_smem").cpu().numpy()
            full = [torch.from_numpy(a).cuda() for a in R.spmv_matrix(spec)] + [torch.from_numpy(xs).cuda()]
            y1 = P.spmv_csr_f64(*full, simdlen=8, mode="generic_smem").cpu().numpy()
            assert np.array_equal(bits(y), bits(y1[rb:rb + nloc])), (rank, it)
        torch.cuda.synchronize()
        dist.barrier()
        xp.close()
        dist.destroy_process_group()
        q.put((rank, "ok"))
    except Exception as e:  # reported to the parent
        q.put((rank, repr(e)))


def test_xpeer_ipc_two_processes_one_gpu(P):
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    procs = [ctx.Process(target=_ipc_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=240) for _ in procs)
    for p in procs:
        p.join(timeout=60)
    assert res == {0: "ok", 1: "ok"}, res
