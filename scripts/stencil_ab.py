"""cfg3 nested stencil: flushed single-launch timing of a configuration grid
(developer tool).  python scripts/stencil_ab.py [--Ls 4,8,16,32,64] [--json out]
Each configuration: median of `iters` launches, one per event pair, L2 flushed
(and left clean) before each -- the HBM number.  Prints the best per L overall,
per simd unit (scalar / pairs) and the best simdlen 1."""
import argparse
import json
import os
import statistics
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_wrightdtcc23_b200 as P  # noqa: E402
from nestgen import recipes as R  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--Ls", default="4,8,16,32,64")
ap.add_argument("--iters", type=int, default=15)
ap.add_argument("--json", default="")
ap.add_argument("--U", default="1", help="outer_unroll values (SPMD transpose-reduce), e.g. 1,2,4")
a = ap.parse_args()
N = 1 << 20
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
res = []
for L in map(int, a.Ls.split(",")):
    inp, coef, w = R.stencil_inputs(N, L)
    t = [torch.from_numpy(v).cuda() for v in (inp, coef, w)]
    o = torch.empty(N, dtype=torch.float64, device="cuda")
    B = 8 * (N * L + 2) + 16 * N + 8 * L
    for S in (1, 2, 4, 8, 16):
        for unit in ("scalar", "pairs"):
            for T, blocked, U in ((T, b, U) for T in (256, 512, 1024) for b in (False, True)
                                  for U in map(int, a.U.split(","))):
                if True:
                    cfg = dict(simdlen=S, mode="spmd", threads_per_team=T, blocked=blocked,
                               vec128=unit != "scalar", outer_unroll=U)
                    try:
                        P.nested_stencil_f64(*t, N, L, o, **cfg)
                    except P.NestError:
                        continue
                    ts = []
                    for _ in range(a.iters):
                        P.l2_flush(flush)
                        e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
                        e0.record()
                        P.nested_stencil_f64(*t, N, L, o, **cfg)
                        e1.record()
                        ts.append((e0, e1))
                    torch.cuda.synchronize()
                    ms = statistics.median(x.elapsed_time(y) for x, y in ts)
                    res.append(dict(L=L, unit=unit, ms=ms, GBs=B / ms / 1e6, **cfg))
    rows = [r for r in res if r["L"] == L]
    best = min(rows, key=lambda r: r["ms"])
    s1 = min((r for r in rows if r["simdlen"] == 1), key=lambda r: r["ms"])
    print(f"L={L:3d} best {best['GBs']:7.1f} GB/s ({best['GBs'] / 6446:.3f}) S={best['simdlen']} {best['unit']} "
          f"T={best['threads_per_team']} blocked={best['blocked']} U={best['outer_unroll']}  | simdlen1 {s1['GBs']:7.1f} ({s1['unit']} "
          f"T={s1['threads_per_team']})  speedup {s1['ms'] / best['ms']:.2f}", flush=True)
    for unit in ("scalar", "pairs"):
        ur = [r for r in rows if r["unit"] == unit]
        if ur:
            b = min(ur, key=lambda r: r["ms"])
            print(f"       {unit:6s} {b['GBs']:7.1f} GB/s S={b['simdlen']} T={b['threads_per_team']} "
                  f"blocked={b['blocked']}", flush=True)
if a.json:
    with open(a.json, "w") as f:
        json.dump(res, f)
