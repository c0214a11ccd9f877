"""Library comparison point (not a product path): cuSPARSE CSR SpMV through
torch.sparse on the cfg2 matrix, timed like bench.py (CUDA events, L2 flushed
between iterations).  Prints one JSON line."""
import json
import os
import statistics
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_wrightdtcc23_b200 as P  # noqa: E402
from nestgen import recipes as R  # noqa: E402

spec = getattr(R, sys.argv[1] if len(sys.argv) > 1 else "CFG2")
rp, col, val = R.spmv_matrix(spec)
x = R.spmv_x(spec)
d = torch.device("cuda")
# cuSPARSE needs one index type for row offsets and columns: int32 for both (fits; fewer bytes)
A = torch.sparse_csr_tensor(torch.from_numpy(rp.astype("int32")).to(d), torch.from_numpy(col).to(d),
                            torch.from_numpy(val).to(d), size=(spec.nrows, spec.ncols))
xd = torch.from_numpy(x).to(d)
flush = torch.empty(512 << 20, dtype=torch.uint8, device=d)
y = torch.mv(A, xd)
yn = P.spmv_csr_f64(*(torch.from_numpy(a).to(d) for a in (rp, col, val)), xd, simdlen=2, blocked=True,
                    threads_per_team=1024, vec128=True)
err = (y - yn).abs().max().item()
ts = []
for _ in range(20):
    P.l2_flush(flush)
    e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
    e0.record()
    torch.mv(A, xd)
    e1.record()
    e1.synchronize()
    ts.append(e0.elapsed_time(e1))
nnz = val.size
B = nnz * 12 + (spec.nrows + 1) * 8 + spec.nrows * 8 + spec.ncols * 8
ms = statistics.median(ts)
print(json.dumps({"impl": "cuSPARSE via torch.mv(sparse_csr)", "spec": spec.name, "ms": ms, "GBs": B / ms / 1e6,
                  "max_abs_diff_vs_nest": err}))
