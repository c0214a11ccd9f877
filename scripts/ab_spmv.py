"""A/B timing of SpMV configurations on cfg2 (developer experiment, not the bench):
alternates L2-flush modes (NEST_FLUSH_CLEAN) and configurations in one process.
python scripts/ab_spmv.py [rounds]"""
import os
import statistics
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_wrightdtcc23_b200 as P  # noqa: E402
from nestgen import recipes as R  # noqa: E402

spec = R.CFG2
rp, col, val = R.spmv_matrix(spec)
x = R.spmv_x(spec)
t = [torch.from_numpy(v).cuda() for v in (rp, col, val, x)]
y = torch.empty(spec.nrows, dtype=torch.float64, device="cuda")
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
CFGS = {
    "S2 bv": dict(simdlen=2, threads_per_team=1024, blocked=True, vec128=True),
    "S1 bv": dict(simdlen=1, threads_per_team=1024, blocked=True, vec128=True),
    "S2 b": dict(simdlen=2, threads_per_team=1024, blocked=True),
    "S2 bvh": dict(simdlen=2, threads_per_team=1024, blocked=True, vec128=True, stream_hints=True),
    "S1 bvh": dict(simdlen=1, threads_per_team=1024, blocked=True, vec128=True, stream_hints=True),
    "S4 bvh": dict(simdlen=4, threads_per_team=1024, blocked=True, vec128=True, stream_hints=True),
    "S1 cyc256": dict(simdlen=1, threads_per_team=256),
    "S2 bv T768": dict(simdlen=2, threads_per_team=768, blocked=True, vec128=True),
    "S1 bv T768": dict(simdlen=1, threads_per_team=768, blocked=True, vec128=True),
    "S2 bv T512": dict(simdlen=2, threads_per_team=512, blocked=True, vec128=True),
    "S2 v xwin4096 T1024": dict(simdlen=2, threads_per_team=1024, vec128=True, x_halo=4096),
    "S2 v xwin3072 T1024": dict(simdlen=2, threads_per_team=1024, vec128=True, x_halo=3072),
    "S2 v xwin4096 T512": dict(simdlen=2, threads_per_team=512, vec128=True, x_halo=4096),
    "S4 v xwin4096 T1024": dict(simdlen=4, threads_per_team=1024, vec128=True, x_halo=4096),
    "S1 v xwin4096 T1024": dict(simdlen=1, threads_per_team=1024, vec128=True, x_halo=4096),
    "S2 b gsmem": dict(simdlen=2, mode="generic_smem", threads_per_team=1024, blocked=True),
    "S2 b gshfl": dict(simdlen=2, mode="generic_shfl", threads_per_team=1024, blocked=True),
    "S4 b": dict(simdlen=4, threads_per_team=1024, blocked=True),
    "S8 b": dict(simdlen=8, threads_per_team=1024, blocked=True),
    "S8 b gsmem": dict(simdlen=8, mode="generic_smem", threads_per_team=1024, blocked=True),
    "S1 b": dict(simdlen=1, threads_per_team=1024, blocked=True),
    "S2 v xwin4096 U2": dict(simdlen=2, threads_per_team=1024, vec128=True, x_halo=4096, outer_unroll=2),
    "S2 v xwin4096 U4": dict(simdlen=2, threads_per_team=1024, vec128=True, x_halo=4096, outer_unroll=4),
    "S4 v xwin4096 U2": dict(simdlen=4, threads_per_team=1024, vec128=True, x_halo=4096, outer_unroll=2),
}
if os.environ.get("AB_ONLY"):
    CFGS = {k: v for k, v in CFGS.items() if k in os.environ["AB_ONLY"].split(",")}
rounds = int(sys.argv[1]) if len(sys.argv) > 1 else 3
res = {}
for r in range(rounds):
    for clean in ("1",):
        os.environ["NEST_FLUSH_CLEAN"] = clean
        for name, cfg in CFGS.items():
            ts = []
            for _ in range(12):
                P.l2_flush(flush)
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record()
                P.spmv_csr_f64(*t, y, **cfg)
                e1.record()
                ts.append((e0, e1))
            torch.cuda.synchronize()
            ms = [a.elapsed_time(b) for a, b in ts][2:]
            res.setdefault((name, clean), []).append(statistics.median(ms))
for (name, clean), v in sorted(res.items()):
    print(f"{name:12s} clean={clean}  medians {' '.join(f'{m:.4f}' for m in v)}")
