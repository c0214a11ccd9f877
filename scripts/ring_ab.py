"""A/B timing of SpMV launch configurations on one matrix (developer tool).

python scripts/ring_ab.py --spec CFG2 [--check]
Each configuration: median of 10 CUDA-event-timed launches, L2 flushed before
each.  --check compares every configuration's y with the first one bitwise
where the lane order is the same, else within R3 against the oracle on a sample.
"""
import argparse
import json
import os
import statistics
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_wrightdtcc23_b200 as P  # noqa: E402
from nestgen import recipes as R  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--spec", default="CFG2")
ap.add_argument("--iters", type=int, default=10)
ap.add_argument("--check", action="store_true")
ap.add_argument("--configs", default="default")
a = ap.parse_args()
spec = getattr(R, a.spec)
import bench  # noqa: E402
x = R.spmv_x(spec)
drp, dcol, dval, nnz, _, _ = bench.gen_to_device(torch, spec, torch.device("cuda"))
B = nnz * 12 + (spec.nrows + 1) * 8 + spec.nrows * 8 + spec.ncols * 8
t = [drp, dcol, dval, torch.from_numpy(x).cuda()]
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")

base = dict(threads_per_team=1024, blocked=True)
CONFIGS = {
    "default": [
        ("nest S2 pairs (r1 headline)", dict(simdlen=2, vec128=True, **base)),
        ("nest S1 pairs", dict(simdlen=1, vec128=True, **base)),
        ("ring S2 pairs T768 tps2", dict(simdlen=2, vec128=True, x_halo=4096, teams_per_sm=2, threads_per_team=768)),
        ("ring S2 pairs T768 tps2 kb2", dict(simdlen=2, vec128=True, x_halo=4096, teams_per_sm=2, outer_unroll=2,
                                             threads_per_team=768)),
        ("ring S2 scalar T768 tps2", dict(simdlen=2, x_halo=4096, teams_per_sm=2, threads_per_team=768)),
        ("ring S2 pairs T1024 tps1", dict(simdlen=2, vec128=True, x_halo=4096, teams_per_sm=1, threads_per_team=1024)),
        ("ring S4 pairs T768 tps2", dict(simdlen=4, vec128=True, x_halo=4096, teams_per_sm=2, threads_per_team=768)),
        ("ring S1 pairs T768 tps2", dict(simdlen=1, vec128=True, x_halo=4096, teams_per_sm=2, threads_per_team=768)),
        ("ring S8 pairs T768 tps2", dict(simdlen=8, vec128=True, x_halo=4096, teams_per_sm=2, threads_per_team=768)),
        ("ring S2 pairs T768 gsmem", dict(simdlen=2, vec128=True, x_halo=4096, teams_per_sm=2, mode="generic_smem",
                                          threads_per_team=768)),
    ],
    "chunks": [(f"S{S} {'pairs' if v else 'scalar'} chunk {c}",
                dict(simdlen=S, vec128=v, team_chunk=c, **base))
               for S, v in ((8, True), (4, True), (2, True), (1, True), (8, False))
               for c in (0, 512, 2048, 8192, 32768)],
    "pshape": [(f"S{S} {'quads' if q else 'pairs'} T{T} persist", dict(simdlen=S, vec128=True, quad=q, blocked=True,
                                                                      threads_per_team=T, x_l2_persist=True))
               for S in (2, 4) for q in (True, False) for T in (512, 640, 768, 1024)],
    "generic": [(f"S{S} {m} {fl} T{T}", dict(simdlen=S, mode=m, blocked=True, threads_per_team=T,
                                               vec128=fl != "scalar", quad=fl == "quads", x_l2_persist=True))
                for S in (2, 4, 8) for m in ("generic_smem", "generic_shfl") for fl in ("scalar", "pairs", "quads")
                for T in (768, 1024)],
    "ringp": [(f"ring S2 pairs T768 kb2{' persist' if pe else ''}", dict(simdlen=2, vec128=True, x_halo=4096,
                teams_per_sm=2, outer_unroll=2, threads_per_team=768, x_l2_persist=pe)) for pe in (False, True)],
    "waves": [(f"S2 quads persist teams {nt}", dict(simdlen=2, quad=True, blocked=True, threads_per_team=1024,
                                                    x_l2_persist=True, num_teams=nt))
              for nt in (0, 592, 888, 1184, 2368, 4736)],
    "cfg5ab": [(f"S8 {nm} rep{r}", dict(simdlen=8, vec128=True, quad=q, blocked=True, threads_per_team=1024))
               for r in range(3) for nm, q in (("pairs", False), ("quads", True))],
    "cfg5": [(f"S{S} {'quads' if q else 'pairs'} U{U}{' persist' if pe else ''}",
              dict(simdlen=S, vec128=True, quad=q, blocked=True, threads_per_team=1024, outer_unroll=U,
                   x_l2_persist=pe))
             for S in (4, 8, 16) for q in (True, False) for U in (1, 2) for pe in (False, True)],
    "xpol": [("S8 pairs", dict(simdlen=8, vec128=True, **base)),
             ("S8 pairs persist", dict(simdlen=8, vec128=True, x_l2_persist=True, **base)),
             ("S2 quads", dict(simdlen=2, quad=True, **base)),
             ("S2 quads persist", dict(simdlen=2, quad=True, x_l2_persist=True, **base)),
             ("S4 quads", dict(simdlen=4, quad=True, **base)),
             ("S1 pairs", dict(simdlen=1, vec128=True, **base))],
    "hint": [("S8 pairs", dict(simdlen=8, vec128=True, **base)), ("S2 pairs", dict(simdlen=2, vec128=True, **base)),
             ("S4 pairs", dict(simdlen=4, vec128=True, **base)), ("S1 pairs", dict(simdlen=1, vec128=True, **base))],
    "unroll": [(f"S{S} {'pairs' if v else 'scalar'} U{U} T{T}", dict(simdlen=S, vec128=v, outer_unroll=U,
                                                                    threads_per_team=T, blocked=True))
               for S in (2, 4, 8, 16) for v in (True, False) for U in (1, 2, 4) for T in (512, 1024)],
    "teams": [(f"S{S} pairs teams {nt}", dict(simdlen=S, vec128=True, num_teams=nt, **base))
              for S in (8, 2) for nt in (0, 148, 444, 592)],
    "quads": [(f"S{S} {'quads' if q else 'pairs'}", dict(simdlen=S, vec128=True, quad=q, **base))
              for S in (1, 2, 4, 8) for q in (False, True)],
    "ringq": [("nest S2 quads", dict(simdlen=2, vec128=True, quad=True, **base)),
              ("ring S2 quads T768 tps2", dict(simdlen=2, vec128=True, quad=True, x_halo=4096, teams_per_sm=2,
                                               threads_per_team=768)),
              ("ring S2 quads T1024 tps1", dict(simdlen=2, vec128=True, quad=True, x_halo=4096, teams_per_sm=1,
                                                threads_per_team=1024)),
              ("ring S4 quads T768 tps2", dict(simdlen=4, vec128=True, quad=True, x_halo=4096, teams_per_sm=2,
                                               threads_per_team=768)),
              ("ring S2 pairs T768 tps2", dict(simdlen=2, vec128=True, x_halo=4096, teams_per_sm=2,
                                               threads_per_team=768))],
    "shape": [(f"S{S} {'quads' if q else 'pairs'} T{T}", dict(simdlen=S, vec128=True, quad=q, threads_per_team=T,
                                                                blocked=True))
              for S in (2, 4) for q in (True, False) for T in (256, 512, 1024)],
    "diag": [
        ("nest S2 pairs (r1 headline)", dict(simdlen=2, vec128=True, **base)),
        ("ring S2 pairs T768 H1", dict(simdlen=2, vec128=True, x_halo=1, teams_per_sm=2, threads_per_team=768)),
        ("ring S2 pairs T768 H4096", dict(simdlen=2, vec128=True, x_halo=4096, teams_per_sm=2, threads_per_team=768)),
        ("ring S2 pairs T768 H1 kb4", dict(simdlen=2, vec128=True, x_halo=1, teams_per_sm=2, threads_per_team=768,
                                           outer_unroll=4)),
        ("ring S2 pairs T768 H4096 kb4", dict(simdlen=2, vec128=True, x_halo=4096, teams_per_sm=2,
                                              threads_per_team=768, outer_unroll=4)),
        ("ring S2 pairs T1024 H1 tps1", dict(simdlen=2, vec128=True, x_halo=1, teams_per_sm=1, threads_per_team=1024)),
        ("nest S2 pairs T768", dict(simdlen=2, vec128=True, threads_per_team=768, blocked=True)),
    ],
}[a.configs]

out = {}
ys = {}
for name, cfg in CONFIGS:
    y = torch.empty(spec.nrows, dtype=torch.float64, device="cuda")
    try:
        P.spmv_csr_f64(*t, y, **cfg)
        torch.cuda.synchronize()
        plan = P.spmv_plan(spec.nrows, spec.ncols, nnz, **cfg)
    except P.NestError as e:
        print(f"{name}: {e}", flush=True)
        continue
    ts = []
    for _ in range(a.iters):
        P.l2_flush(flush)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        P.spmv_csr_f64(*t, y, **cfg)
        e1.record()
        ts.append((e0, e1))
    torch.cuda.synchronize()
    ms = statistics.median(a.elapsed_time(b) for a, b in ts)
    out[name] = {"ms": ms, "GBs": B / ms / 1e6, "plan": plan}
    ys[name] = y
    print(f"{name:34s} {ms:.4f} ms  {B / ms / 1e6:7.1f} GB/s  grid {plan['grid']} smem {plan['smem_bytes']} "
          f"segs {plan['ring_segments']} rowslots {plan['ring_row_slots']}", flush=True)

if a.check:
    import oracle
    rng = np.random.default_rng(3)
    starts = np.concatenate([[0, spec.nrows - 256], rng.integers(0, spec.nrows - 256, 40)])
    for s in starts:
        rpl, cl, vl = R.spmv_matrix(spec, row_begin=int(s), nrows=256)
        yr, ar = oracle.spmv_csr_f64(rpl, cl, vl, x)
        for name, y in ys.items():
            yy = y[s:s + 256].cpu().numpy()
            err = np.abs(yy - yr)
            assert np.all(err <= 1e-12 * ar), (name, s, float(np.max(err / np.maximum(ar, 1e-300))))
    # same lane order -> same bits
    pairs = [k for k in ys if "pairs" in k and "S2" in k]
    for k in pairs[1:]:
        assert torch.equal(ys[pairs[0]], ys[k]), (pairs[0], k)
    print("check ok", flush=True)
print(json.dumps(out))
