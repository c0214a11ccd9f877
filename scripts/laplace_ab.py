"""laplace3d 256^3, pair body, SPMD: flushed timing over (simdlen, T, schedule)
(developer tool; run once per library build).  Prints the best configuration."""
import os
import statistics
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_wrightdtcc23_b200 as P  # noqa: E402
from nestgen import recipes as R  # noqa: E402

nz, ny, nx = R.LAPLACE_SHAPE
u = torch.from_numpy(R.laplace_inputs(nz, ny, nx)).cuda()
o = u.clone()
B = 8 * nz * ny * nx + 8 * (nz - 2) * (ny - 2) * (nx - 2)
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
res = []
for S in (8, 16, 32):
    for T in (256, 512, 768, 1024):
        for blocked in (False, True):
            cfg = dict(simdlen=S, mode="spmd", blocked=blocked, threads_per_team=T, vec128=True)
            try:
                P.laplace3d_f64(u, o, nz, ny, nx, 0.1, **cfg)
            except P.NestError:
                continue
            ts = []
            for _ in range(15):
                P.l2_flush(flush)
                e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
                e0.record()
                P.laplace3d_f64(u, o, nz, ny, nx, 0.1, **cfg)
                e1.record()
                ts.append((e0, e1))
            torch.cuda.synchronize()
            ms = statistics.median(a.elapsed_time(b) for a, b in ts)
            res.append((ms, S, T, blocked))
res.sort()
for ms, S, T, blocked in res[:5]:
    print(f"  {ms:.4f} ms {B / ms / 1e6:7.1f} GB/s  S={S} T={T} blocked={blocked}")
