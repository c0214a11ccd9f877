"""a12 on one GPU: the NCCL path of the row-partitioned SpMV with a single
rank (the all-gather degenerates to a copy through NCCL), against the oracle,
and bit-identical to the single-GPU SpMV (R16)."""
import os
import socket

import numpy as np
import pytest

import oracle
from nestgen import recipes as R

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


def _port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def test_dist_spmv_single_rank_nccl():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import torch.distributed as dist

    import paper_conf_icpp_wrightdtcc23_b200 as P
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(_port()))
    dist.init_process_group("gloo", rank=0, world_size=1)
    try:
        comm = P.Comm()
        spec = R.SpmvSpec("d1", 91, 20011, 20011, 0, 15, band_w=500, far_den=8)
        rp, col, val, x = R.spmv_inputs(spec)
        yref, aref = oracle.spmv_csr_f64(rp, col, val, x)
        d = [torch.from_numpy(a).cuda() for a in (rp, col, val, x)]
        xf = torch.empty(P.x_chunk(spec.ncols, 1), dtype=torch.float64, device="cuda")
        for S, mode, halo in ((1, "spmd", 0), (8, "generic_smem", 0), (4, "spmd", 500), (32, "generic_shfl", 0)):
            y = comm.spmv_csr_f64(spec.nrows, spec.ncols, d[0], d[1], d[2], d[3], xf,
                                  simdlen=S, mode=mode, x_halo=halo).cpu().numpy()
            assert np.all(np.abs(y - yref) <= 1e-12 * aref)
            y1 = P.spmv_csr_f64(*d, simdlen=S, mode=mode, x_halo=halo).cpu().numpy()
            assert np.array_equal(y.view(np.int64), y1.view(np.int64))
        # x_full under the persisting-L2 window: the same bits
        y = comm.spmv_csr_f64(spec.nrows, spec.ncols, d[0], d[1], d[2], d[3], xf, simdlen=2, quad=True, blocked=True,
                              threads_per_team=1024, x_l2_persist=True).cpu().numpy()
        y1 = P.spmv_csr_f64(*d, simdlen=2, quad=True, blocked=True, threads_per_team=1024).cpu().numpy()
        assert np.array_equal(y.view(np.int64), y1.view(np.int64))
        with pytest.raises(P.NestError):   # wrong local row count for the rank
            comm.spmv_csr_f64(spec.nrows + 5, spec.ncols, d[0], d[1], d[2], d[3], xf)
        # the exchange step alone, and the host-buffer entry point
        xf2 = torch.zeros_like(xf)
        comm.allgather_x(d[3], xf2, spec.ncols)
        assert torch.equal(xf2[:spec.ncols], d[3])
        pin = lambda a: torch.from_numpy(np.ascontiguousarray(a)).pin_memory()
        hy = torch.empty(spec.nrows, dtype=torch.float64).pin_memory()
        ws = torch.empty(comm.hostio_workspace_bytes(spec.nrows, val.size, spec.ncols), dtype=torch.uint8,
                         device="cuda")
        for cfg in (dict(simdlen=2, quad=True, blocked=True, threads_per_team=1024), dict(simdlen=8),
                    dict(simdlen=2, quad=True, blocked=True, threads_per_team=1024, x_l2_persist=True)):
            comm.spmv_csr_f64_hostio(spec.nrows, spec.ncols, pin(rp), pin(col), pin(val), pin(x), hy, ws, **cfg)
            torch.cuda.synchronize()
            y1 = P.spmv_csr_f64(*d, **cfg).cpu().numpy()
            assert np.array_equal(hy.numpy().view(np.int64), y1.view(np.int64)), cfg
        with pytest.raises(ValueError):    # short host buffer: refused before the C call
            comm.spmv_csr_f64_hostio(spec.nrows, spec.ncols, pin(rp), pin(col[:-1]), pin(val), pin(x), hy, ws)
        comm.close()
    finally:
        dist.destroy_process_group()


def _nccl_worker(rank, world, port, q):
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    torch.cuda.set_device(rank)
    dist.init_process_group("nccl", rank=rank, world_size=world)
    try:
        import paper_conf_icpp_wrightdtcc23_b200 as P
        spec = R.SpmvSpec("d2", 93, 40_009, 40_009, 0, 21, band_w=700, far_den=4)
        chunk, rb, nloc = P.shard_rows(spec.nrows, world, rank)
        rp, col, val = R.spmv_matrix(spec, row_begin=rb, nrows=nloc)
        xc = P.x_chunk(spec.ncols, world)
        xb, xn = P.local_x_range(spec.ncols, world, rank)
        xl = torch.zeros(xc, dtype=torch.float64)
        xl[:xn] = torch.from_numpy(R.spmv_x(spec, begin=xb, n=xn))
        d = [torch.from_numpy(a).cuda() for a in (rp, col, val)]
        dxl = xl.cuda()
        xf = torch.empty(xc * world, dtype=torch.float64, device="cuda")
        comm = P.Comm()
        out = {}
        for S, mode, vec in ((2, "spmd", True), (8, "generic_smem", False), (1, "spmd", False)):
            y = comm.spmv_csr_f64(spec.nrows, spec.ncols, *d, dxl, xf, simdlen=S, mode=mode, vec128=vec,
                                  threads_per_team=1024, blocked=True)
            out[(S, mode, vec)] = y.cpu().numpy()
        # the exchange step alone and the host-buffer entry point
        xf2 = torch.zeros_like(xf)
        comm.allgather_x(dxl, xf2, spec.ncols)
        same_x = bool(torch.equal(xf, xf2))
        ws = torch.empty(comm.hostio_workspace_bytes(nloc, val.size, spec.ncols), dtype=torch.uint8, device="cuda")
        hy = torch.empty(nloc, dtype=torch.float64).pin_memory()
        pin = lambda a: torch.from_numpy(a).pin_memory()
        comm.spmv_csr_f64_hostio(spec.nrows, spec.ncols, pin(rp), pin(col), pin(val), xl.pin_memory(), hy, ws,
                                 simdlen=2, vec128=True, threads_per_team=1024, blocked=True)
        torch.cuda.synchronize()
        q.put((rank, rb, out, same_x, hy.numpy().copy()))
        comm.close()
    finally:
        dist.destroy_process_group()


def test_dist_spmv_two_ranks_nccl():
    """a12 with a real exchange: 2 ranks, one GPU each, ncclAllGather of x over
    NVLink; every rank's rows against the oracle, bit-identical to the 1-GPU
    kernel at the same variant (R16).  Skips on a one-GPU box."""
    if not torch.cuda.is_available() or torch.cuda.device_count() < 2:
        pytest.skip("needs two GPUs")
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    procs = [ctx.Process(target=_nccl_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = [q.get(timeout=600) for _ in range(2)]
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    import paper_conf_icpp_wrightdtcc23_b200 as P
    spec = R.SpmvSpec("d2", 93, 40_009, 40_009, 0, 21, band_w=700, far_den=4)
    rp, col, val, x = R.spmv_inputs(spec)
    yref, aref = oracle.spmv_csr_f64(rp, col, val, x)
    d = [torch.from_numpy(a).cuda() for a in (rp, col, val, x)]
    for rank, rb, out, same_x, hy in res:
        assert same_x
        for (S, mode, vec), y in out.items():
            sl = slice(rb, rb + y.size)
            assert np.all(np.abs(y - yref[sl]) <= 1e-12 * aref[sl])
            y1 = P.spmv_csr_f64(*d, simdlen=S, mode=mode, vec128=vec, threads_per_team=1024,
                                blocked=True).cpu().numpy()
            # R16: bit-identical to the 1-GPU kernel; 128-bit pairs need the shard's
            # nonzero offset to be even (the same tuple boundaries)
            if not vec or rp[rb] % 2 == 0:
                assert np.array_equal(y.view(np.int64), y1[sl].view(np.int64)), (rank, S, mode, vec)
        assert np.array_equal(hy.view(np.int64), out[(2, "spmd", True)].view(np.int64))
