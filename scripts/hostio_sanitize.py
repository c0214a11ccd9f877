"""compute-sanitizer workload for the chunked end-to-end SpMV (run with
NEST_HOSTIO_CHUNKS set): small ragged matrices, the headline and quad configs."""
import os
import sys
from dataclasses import replace

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_icpp_wrightdtcc23_b200 as P  # noqa: E402
from nestgen import recipes as R  # noqa: E402

pin = lambda a: torch.from_numpy(np.ascontiguousarray(a)).pin_memory()
for nrows, lo, hi in ((7, 0, 3), (5001, 0, 9)):
    spec = replace(R.CFG1, name="hio", seed=R.seed(9) + nrows, nrows=nrows, ncols=max(nrows, 64),
                   nnz_min=lo, nnz_max=hi)
    rp, col, val = R.spmv_matrix(spec)
    x = R.spmv_x(spec)
    for cfg in (dict(simdlen=2, threads_per_team=1024, blocked=True, vec128=True),
                dict(simdlen=1, threads_per_team=1024, blocked=True, quad=True)):
        hy = torch.empty(nrows, dtype=torch.float64).pin_memory()
        ws = torch.empty(P.hostio_workspace_bytes(nrows, x.size, val.size), dtype=torch.uint8, device="cuda")
        P.spmv_csr_f64_hostio(pin(rp), pin(col), pin(val), pin(x), hy, ws, **cfg)
        torch.cuda.synchronize()
print("hostio sanitize workload done")
