"""configs[4] rank-0 shard at P = 2 / 4 / 8 on one GPU (x = the full 800 MB, as after the
all-gather): which local SpMV configuration is fastest per shard size (developer tool).
Median of 10 launches, L2 flushed before each."""
import os
import statistics
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
import paper_conf_icpp_wrightdtcc23_b200 as P  # noqa: E402
from nestgen import recipes as R  # noqa: E402

spec = R.CFG5
dx = torch.from_numpy(R.spmv_x(spec)).cuda()
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
CANDS = [(8, "spmd", 1, 1024, 0, "bv"), (8, "spmd", 1, 1024, 0, "bq"), (4, "spmd", 1, 1024, 0, "bq"),
         (2, "spmd", 1, 1024, 0, "bq"), (2, "spmd", 1, 1024, 0, "bqp"), (2, "spmd", 1, 1024, 0, "bv"),
         (1, "spmd", 1, 1024, 0, "bqp")]
for nranks in (2, 4, 8):
    _, rb, nloc = P.shard_rows(spec.nrows, nranks, 0)
    drp, dcol, dval, nnz, _, _ = bench.gen_to_device(torch, spec, torch.device("cuda"), row_begin=rb, nrows=nloc)
    y = torch.empty(nloc, dtype=torch.float64, device="cuda")
    B = nnz * 12 + (nloc + 1) * 8 + nloc * 8 + spec.ncols * 8
    res = []
    for c in CANDS:
        fn = lambda: P.spmv_csr_f64(drp, dcol, dval, dx, y, ncols=spec.ncols, **bench.cfg_of(c))
        fn()
        ms = statistics.median(bench.time_steps(torch, fn, flush, P, 10))
        res.append((ms, c))
    res.sort()
    print(f"P={nranks} shard {nloc} rows:", "  ".join(f"{c[0]}{c[5]} {ms:.3f}" for ms, c in res), flush=True)
    del drp, dcol, dval
    torch.cuda.empty_cache()
