"""End-to-end SpMV (nest_spmv_csr_f64_hostio, pinned host buffers) on cfg2 in the bench
headline's configuration: ms per call and the H2D rate, for the chunk count in
NEST_HOSTIO_CHUNKS (developer tool; one process per chunk count)."""
import os, sys, time, torch
sys.path.insert(0, "/root/repo")
import bench
import paper_conf_icpp_wrightdtcc23_b200 as P
from nestgen import recipes as R
spec = R.CFG2
rp, col, val = R.spmv_matrix(spec); x = R.spmv_x(spec)
pin = lambda a: torch.from_numpy(a).pin_memory()
h = [pin(rp), pin(col), pin(val), pin(x)]
hy = torch.empty(spec.nrows, dtype=torch.float64).pin_memory()
ws = torch.empty(P.hostio_workspace_bytes(spec.nrows, spec.ncols, val.size), dtype=torch.uint8, device="cuda")
cfg = bench.cfg_of(bench.HEADLINE)
f = lambda: P.spmv_csr_f64_hostio(*h, hy, ws, **cfg)
f(); torch.cuda.synchronize()
ts = []
for _ in range(8):
    e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
    e0.record(); f(); e1.record(); e1.synchronize(); ts.append(e0.elapsed_time(e1))
B = bench.alg_bytes(spec.nrows, spec.ncols, val.size)
ms = sorted(ts)[len(ts)//2]
print(os.environ.get("NEST_HOSTIO_CHUNKS", "default"), f"{ms:.3f} ms  e2e {B/ms/1e6:.1f} GB/s  h2d {(val.size*12+(spec.nrows+1)*8+spec.ncols*8)/ms/1e6:.1f} GB/s")
