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
        with pytest.raises(P.NestError):   # wrong local row count for the rank
            comm.spmv_csr_f64(spec.nrows + 5, spec.ncols, d[0], d[1], d[2], d[3], xf)
        comm.close()
    finally:
        dist.destroy_process_group()
