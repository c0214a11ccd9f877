"""Multi-process (world_size 2, gloo, CPU) checks of the row-partitioned SpMV's
host logic (a12): the NCCL-id bootstrap through the torch
process group, the equal-row / equal-x-chunk decomposition, and that the
per-rank pieces -- local rows against the all-gathered x -- reproduce the
single-process oracle bit for bit (R16).  The device all-gather itself runs
under NCCL on GPUs (tests/test_gpu_dist.py, bench.py --gpus N)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
from nestgen import recipes as R


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import paper_conf_icpp_wrightdtcc23_b200 as P
        uid = P.broadcast_unique_id()
        ids = [None] * world
        dist.all_gather_object(ids, uid)
        spec = R.SpmvSpec("dist", 77, 3001, 2999, 0, 17, band_w=300, far_den=4, values="int")
        chunk, rb, nloc = P.shard_rows(spec.nrows, world, rank)
        rp, col, val = R.spmv_matrix(spec, row_begin=rb, nrows=nloc)
        xc = P.x_chunk(spec.ncols, world)
        xb, xn = P.local_x_range(spec.ncols, world, rank)
        xl = np.zeros(xc)
        xl[:xn] = R.spmv_x(spec, begin=xb, n=xn)
        parts = [torch.zeros(xc, dtype=torch.float64) for _ in range(world)]
        dist.all_gather(parts, torch.from_numpy(xl))       # the exchange step, gloo here
        x_full = torch.cat(parts).numpy()
        y_local, _ = oracle.spmv_csr_f64(rp, col, val, x_full)
        ys = [None] * world
        dist.all_gather_object(ys, (rb, y_local))
        q.put((rank, ids, chunk, ys, x_full.size))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2])
def test_row_partitioned_spmv_gloo(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    spec = R.SpmvSpec("dist", 77, 3001, 2999, 0, 17, band_w=300, far_den=4, values="int")
    rp, col, val, x = R.spmv_inputs(spec)
    yref, _ = oracle.spmv_csr_f64(rp, col, val, x)
    for rank, ids, chunk, ys, nfull in res:
        assert len(set(ids)) == 1 and len(ids[0]) == 128      # one NCCL id everywhere
        assert chunk == -(-spec.nrows // world)
        assert nfull == world * -(-spec.ncols // world)
        y = np.concatenate([y for _, y in sorted(ys, key=lambda t: t[0])])
        assert np.array_equal(y.view(np.int64), yref.view(np.int64))


def _fd_worker(rank, world, port, tmpdir, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_icpp_wrightdtcc23_b200.dist import _exchange_fds
        # each rank opens its own file holding its rank number and passes the descriptor
        path = os.path.join(tmpdir, f"r{rank}")
        with open(path, "w") as f:
            f.write(f"rank {rank}")
        fd = os.open(path, os.O_RDONLY)
        fds = _exchange_fds(fd, rank, world, f"gloo{port}")
        got = []
        for r, f in enumerate(fds):
            os.lseek(f, 0, os.SEEK_SET)
            got.append(os.read(f, 64).decode())
            os.close(f)
        q.put((rank, got))
    except Exception as e:
        q.put((rank, repr(e)))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_symmetric_x_fd_exchange_gloo(world, tmp_path):
    # NEXT-4b host logic: every rank receives every other rank's file descriptor (SCM_RIGHTS
    # over unix sockets, ordered by the process group) and it refers to the sender's object
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_fd_worker, args=(r, world, port, str(tmp_path), q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=120) for _ in procs)
    for p in procs:
        p.join(timeout=30)
    for r in range(world):
        assert res[r] == [f"rank {k}" for k in range(world)], res
