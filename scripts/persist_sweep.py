"""NEST_F_X_L2_PERSIST set-aside sweep (developer tool): the library raises the
device's persisting-L2 limit to half of L2 and uses max(limit, that); here the
limit is raised further by hand and the headline quads timed on cfg2 and G100
(median of 10 launches, L2 flushed and persisting lines reset before each)."""
import os
import statistics
import sys

import torch
from cuda.bindings import runtime as rt

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
import paper_conf_icpp_wrightdtcc23_b200 as P  # noqa: E402
from nestgen import recipes as R  # noqa: E402

flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
for spec in (R.CFG2, R.G100):
    drp, dcol, dval, nnz, _, _ = bench.gen_to_device(torch, spec, torch.device("cuda"))
    t = [drp, dcol, dval, torch.from_numpy(R.spmv_x(spec)).cuda()]
    y = torch.empty(spec.nrows, dtype=torch.float64, device="cuda")
    B = bench.alg_bytes(spec.nrows, spec.ncols, nnz)
    for S, fl in ((2, "bq"), (2, "bqp"), (1, "bqp")):
        for mb in ((0,) if "p" not in fl else (0, 72)):
            if mb:
                rt.cudaDeviceSetLimit(rt.cudaLimit.cudaLimitPersistingL2CacheSize, mb << 20)
            c = (S, "spmd", 1, 1024, 0, fl)
            ms = statistics.median(bench.time_steps(torch, lambda: P.spmv_csr_f64(*t, y, **bench.cfg_of(c)),
                                                    flush, P, 10))
            info = P.spmv_plan(spec.nrows, spec.ncols, nnz, **bench.cfg_of(c))
            print(f"{spec.name} S{S} {fl:4s} limit {mb:3d} MB setaside {info['l2_setaside_bytes'] >> 20} MB "
                  f"window {info['l2_window_bytes'] >> 20} MB: {ms:.4f} ms {B / ms / 1e6:.0f} GB/s", flush=True)
        rt.cudaDeviceSetLimit(rt.cudaLimit.cudaLimitPersistingL2CacheSize, 0)
    del t, drp, dcol, dval
    torch.cuda.empty_cache()
