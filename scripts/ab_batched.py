"""A/B timing of batched 64x64 matvec configurations on cfg4 (developer experiment)."""
import os
import statistics
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_wrightdtcc23_b200 as P  # noqa: E402
from nestgen import recipes as R  # noqa: E402

B = 500_000
A, x = (torch.from_numpy(a).cuda() for a in R.batched_inputs(B))
y = torch.empty(B * 64, dtype=torch.float32, device="cuda")
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
alg = B * 16896
for S, U, T in ((4, 1, 256), (4, 2, 256), (8, 1, 256), (8, 2, 256), (4, 1, 512), (2, 1, 256), (16, 1, 256)):
    ts = []
    for _ in range(8):
        P.l2_flush(flush)
        e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
        e0.record()
        P.batched_matvec_f32(A, x, B, y=y, simdlen=S, outer_unroll=U, threads_per_team=T, vec128=True)
        e1.record()
        ts.append((e0, e1))
    torch.cuda.synchronize()
    ms = statistics.median([a.elapsed_time(b) for a, b in ts][2:])
    print(f"S={S:2d} U={U} T={T:4d}  {ms:.4f} ms  {alg / ms / 1e6:.0f} GB/s")
