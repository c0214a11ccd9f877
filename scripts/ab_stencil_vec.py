"""A/B: nested stencil (cfg3, N = 2^20) scalar simd unit vs 128-bit pairs
(NEST_F_VEC128).  Per (L, S, mode): median of 20 launches, L2 flushed before
each, CUDA events on the launching stream.  GB/s = (8 (N L + 2) + 16 N + 8 L) / t
(DESIGN.md §6).  python scripts/ab_stencil_vec.py > out.json"""
import json
import os
import statistics
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_wrightdtcc23_b200 as P  # noqa: E402
from nestgen import recipes as R  # noqa: E402

N = 1 << 20
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
res = {}
for L in R.STENCIL_LS:
    inp, coef, w = R.stencil_inputs(N, L)
    t = [torch.from_numpy(a).cuda() for a in (inp, coef, w)]
    out = torch.empty(N, dtype=torch.float64, device="cuda")
    B = 8 * (N * L + 2) + 16 * N + 8 * L
    for S in (1, 2, 4, 8, 16, 32):
        for mode in ("spmd", "generic_smem"):
            if S == 1 and mode != "spmd":
                continue
            for vec in (False, True):
                cfg = dict(simdlen=S, mode=mode, vec128=vec, threads_per_team=256)
                P.nested_stencil_f64(*t, N, L, out, **cfg)
                ev = []
                for _ in range(20):
                    P.l2_flush(flush)
                    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    e0.record()
                    P.nested_stencil_f64(*t, N, L, out, **cfg)
                    e1.record()
                    ev.append((e0, e1))
                torch.cuda.synchronize()
                ms = statistics.median(a.elapsed_time(b) for a, b in ev)
                res[f"L{L} S{S} {mode} {'vec' if vec else 'scalar'}"] = {"ms": round(ms, 5), "GBs": round(B / ms / 1e6, 1)}
    del t
print(json.dumps(res, indent=1))
