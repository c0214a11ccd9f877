"""Run one SpMV variant a few times (for ncu captures).  The matrix is generated
in row chunks straight into device memory (bench.gen_to_device), so configs[4]
(100M rows) fits.  Usage:
python scripts/one_spmv.py --spec CFG2 --S 2 --T 1024 --blocked 1 --vec 1 --iters 3"""
import argparse
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402
import paper_conf_icpp_wrightdtcc23_b200 as P  # noqa: E402
from nestgen import recipes as R  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--spec", default="CFG2")
ap.add_argument("--S", type=int, default=8)
ap.add_argument("--mode", default="spmd")
ap.add_argument("--U", type=int, default=1)
ap.add_argument("--T", type=int, default=256)
ap.add_argument("--hints", type=int, default=0)
ap.add_argument("--persistent", type=int, default=0)
ap.add_argument("--iters", type=int, default=3)
ap.add_argument("--halo", type=int, default=0)
ap.add_argument("--tps", type=int, default=0)
ap.add_argument("--blocked", type=int, default=0)
ap.add_argument("--vec", type=int, default=0)
ap.add_argument("--chunk", type=int, default=0)
ap.add_argument("--persist", type=int, default=0, help="NEST_F_X_L2_PERSIST (x under a persisting-L2 window)")
ap.add_argument("--far_den", type=int, default=0, help="override the spec's far-column odds (1/far_den)")
ap.add_argument("--l2fetch", type=int, default=0, help="cudaLimitMaxL2FetchGranularity in bytes (0: default)")
a = ap.parse_args()
spec = getattr(R, a.spec)
if a.far_den:
    import dataclasses
    spec = dataclasses.replace(spec, name=f"{spec.name}_far{a.far_den}", far_den=a.far_den)
if a.l2fetch:
    torch.cuda.init()
    from cuda.bindings import runtime as rt
    print("set l2 fetch", rt.cudaDeviceSetLimit(rt.cudaLimit.cudaLimitMaxL2FetchGranularity, a.l2fetch),
          rt.cudaDeviceGetLimit(rt.cudaLimit.cudaLimitMaxL2FetchGranularity))
drp, dcol, dval, nnz, _, _ = bench.gen_to_device(torch, spec, torch.device("cuda"))
t = [drp, dcol, dval, torch.from_numpy(R.spmv_x(spec)).cuda()]
y = torch.empty(spec.nrows, dtype=torch.float64, device="cuda")
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
for _ in range(a.iters):
    torch.cuda.synchronize()
    P.l2_flush(flush)
    P.spmv_csr_f64(*t, y, simdlen=a.S, mode=a.mode, outer_unroll=a.U, stream_hints=bool(a.hints),
                   threads_per_team=a.T, persistent=bool(a.persistent), x_halo=a.halo, teams_per_sm=a.tps,
                   blocked=bool(a.blocked), vec128=a.vec >= 1, quad=a.vec == 2, team_chunk=a.chunk,
                   x_l2_persist=bool(a.persist))
torch.cuda.synchronize()
print("done")
