"""Developer sweep: time the CSR SpMV over (simdlen, mode, U, hints, T) on one
workload with CUDA events, L2 flushed between iterations.  Prints one line per
variant.  Not the bench contract (see bench.py)."""
import argparse
import json
import os
import sys
import time

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_wrightdtcc23_b200 as P  # noqa: E402
from nestgen import recipes as R  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--spec", default="CFG2")
    ap.add_argument("--iters", type=int, default=10)
    ap.add_argument("--simdlens", default="1,2,4,8,16,32")
    ap.add_argument("--modes", default="spmd,generic_smem,generic_shfl")
    ap.add_argument("--unrolls", default="1,2,4")
    ap.add_argument("--hints", default="0,1")
    ap.add_argument("--threads", default="256")
    ap.add_argument("--halos", default="0")
    ap.add_argument("--staged", default="0")
    ap.add_argument("--blocked", default="0")
    ap.add_argument("--vec", default="0")
    ap.add_argument("--chunks", default="0")
    ap.add_argument("--tag", default="")
    ap.add_argument("--out", default=None)
    a = ap.parse_args()
    spec = getattr(R, a.spec)
    t0 = time.time()
    rp, col, val = R.spmv_matrix(spec)
    x = R.spmv_x(spec)
    print(f"gen {time.time()-t0:.1f}s nnz={val.size}", flush=True)
    t = [torch.from_numpy(v).cuda() for v in (rp, col, val, x)]
    y = torch.empty(spec.nrows, dtype=torch.float64, device="cuda")
    nnz = val.size
    B = nnz * 12 + (spec.nrows + 1) * 8 + spec.nrows * 8 + spec.ncols * 8
    flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
    res = []
    for T in map(int, a.threads.split(",")):
        for S in map(int, a.simdlens.split(",")):
            for mode in a.modes.split(","):
                if S == 1 and mode != "spmd":
                    continue
                for U in map(int, a.unrolls.split(",")):
                    for h, xh, sg, bl, vc, ck in [(h, xh, sg, bl, vc, ck) for h in map(int, a.hints.split(","))
                                              for xh in map(int, a.halos.split(","))
                                              for sg in map(int, a.staged.split(","))
                                              for bl in map(int, a.blocked.split(","))
                                              for vc in map(int, a.vec.split(","))
                                              for ck in map(int, a.chunks.split(","))]:
                        if vc == 2 and xh:
                            continue
                        cfg = dict(simdlen=S, mode=mode, outer_unroll=U, stream_hints=bool(h), threads_per_team=T,
                                   x_halo=xh, staged=bool(sg), blocked=bool(bl), vec128=vc >= 1, quad=vc == 2, team_chunk=ck if bl else 0)
                        try:
                            P.spmv_csr_f64(*t, y, **cfg)
                        except P.NestError as e:
                            print("skip", cfg, e)
                            continue
                        for _ in range(3):
                            P.spmv_csr_f64(*t, y, **cfg)
                        ts = []
                        for _ in range(a.iters):
                            P.l2_flush(flush)
                            e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
                            e0.record()
                            P.spmv_csr_f64(*t, y, **cfg)
                            e1.record()
                            e1.synchronize()
                            ts.append(e0.elapsed_time(e1))
                        ms = float(np.median(ts))
                        r = dict(T=T, S=S, mode=mode, U=U, hints=h, halo=xh, staged=sg, blocked=bl, vec=vc, chunk=ck, tag=a.tag, ms=ms, min_ms=min(ts), GBs=B / ms / 1e6)
                        res.append(r)
                        print(json.dumps(r), flush=True)
    best = min(res, key=lambda r: r["ms"])
    s1 = min((r for r in res if r["S"] == 1), key=lambda r: r["ms"], default=None)
    print("BEST", json.dumps(best))
    if s1:
        print("S1", json.dumps(s1), "speedup", s1["ms"] / best["ms"])
    if a.out:
        with open(a.out, "w") as f:
            json.dump(res, f, indent=1)


if __name__ == "__main__":
    main()
