"""Run the cfg4 batched matvec a few times (for ncu captures).
python scripts/one_batched.py --S 4 --U 1 --T 256 --iters 3"""
import argparse
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_wrightdtcc23_b200 as P  # noqa: E402
from nestgen import recipes as R  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--S", type=int, default=4)
ap.add_argument("--U", type=int, default=1)
ap.add_argument("--T", type=int, default=256)
ap.add_argument("--mode", default="spmd")
ap.add_argument("--iters", type=int, default=3)
a = ap.parse_args()
B = 500_000
A, x = (torch.from_numpy(v).cuda() for v in R.batched_inputs(B))
y = torch.empty(B * 64, dtype=torch.float32, device="cuda")
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
for _ in range(a.iters):
    P.l2_flush(flush)
    P.batched_matvec_f32(A, x, B, y=y, simdlen=a.S, mode=a.mode, outer_unroll=a.U, threads_per_team=a.T,
                         vec128=True)
torch.cuda.synchronize()
print("done")
