"""Run laplace3d 256^3 a few times (for ncu captures).
python scripts/one_laplace.py --S 32 --T 1024 --blocked 1 --vec 1 --iters 3"""
import argparse
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_wrightdtcc23_b200 as P  # noqa: E402
from nestgen import recipes as R  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--S", type=int, default=32)
ap.add_argument("--T", type=int, default=1024)
ap.add_argument("--blocked", type=int, default=1)
ap.add_argument("--vec", type=int, default=1)
ap.add_argument("--iters", type=int, default=3)
a = ap.parse_args()
nz, ny, nx = R.LAPLACE_SHAPE
u = torch.from_numpy(R.laplace_inputs(nz, ny, nx)).cuda()
o = u.clone()
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
for _ in range(a.iters):
    P.l2_flush(flush)
    P.laplace3d_f64(u, o, nz, ny, nx, 0.1, simdlen=a.S, threads_per_team=a.T, blocked=bool(a.blocked),
                    vec128=bool(a.vec))
torch.cuda.synchronize()
print("done")
