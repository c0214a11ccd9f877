"""Secondary measurements for SURVEY.md §8(d): the other configs' sweeps.

  cfg3  nested stencil loop, N = 2^20, L in {4..64}: simdlen x mode, GB/s and
        the generic/SPMD time ratio (the paper's Fig 10 question)
  cfg4  batched 64x64 fp32 matvec, 500k batches: simdlen x mode x unroll, GB/s
  g100  CSR SpMV on the 100M-nnz matrix (north_star 70% gate), best variants

CUDA events on the current stream, L2 flushed before each timed launch
(cfg3 launches are us-scale: 20 back-to-back launches per event pair, no
flush between them -- stated in the output).  Writes one JSON document.
"""
import argparse
import json
import os
import statistics
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_wrightdtcc23_b200 as P  # noqa: E402
from nestgen import recipes as R  # noqa: E402

MODES = ("spmd", "generic_smem", "generic_shfl")
flush = None


def timed(fn, iters=5, reps=1, do_flush=True):
    ts = []
    fn()
    torch.cuda.synchronize()
    for _ in range(iters):
        if do_flush:
            P.l2_flush(flush)
        e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
        e0.record()
        for _ in range(reps):
            fn()
        e1.record()
        e1.synchronize()
        ts.append(e0.elapsed_time(e1) / reps)
    return statistics.median(ts)


def timed_graph(fn, iters=5, reps=20):
    """us-scale launches: `reps` launches captured once in a CUDA graph and replayed,
    so host launch overhead does not enter the per-launch time (no flush)."""
    fn()
    torch.cuda.synchronize()
    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())
    g = torch.cuda.CUDAGraph()
    with torch.cuda.stream(s):
        fn()   # warm on the capture stream
        torch.cuda.synchronize()
        with torch.cuda.graph(g, stream=s):
            for _ in range(reps):
                fn()
    torch.cuda.synchronize()
    g.replay()
    torch.cuda.synchronize()
    ts = []
    for _ in range(iters):
        e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
        e0.record()
        g.replay()
        e1.record()
        e1.synchronize()
        ts.append(e0.elapsed_time(e1) / reps)
    return statistics.median(ts)


def cfg3(out):
    N = 1 << 20
    res = []
    for L in R.STENCIL_LS:
        inp, coef, w = R.stencil_inputs(N, L)
        t = [torch.from_numpy(a).cuda() for a in (inp, coef, w)]
        o = torch.empty(N, dtype=torch.float64, device="cuda")
        B = 8 * (N * L + 2) + 16 * N + 8 * L
        for S in (1, 2, 4, 8, 16, 32):
            for mode in MODES:
                if S == 1 and mode != "spmd":
                    continue
                for blocked in (False, True):
                    for vec in (False, True):   # scalar simd unit / 128-bit pairs (StencilVecBody)
                        # SPMD at S >= 8: also 2 / 4 outer iterations per group in flight,
                        # reduced together (transpose-reduce)
                        for U in ((1, 2, 4) if mode == "spmd" and S >= 8 else (1,)):
                            try:
                                ms = timed_graph(lambda: P.nested_stencil_f64(*t, N, L, o, simdlen=S, mode=mode,
                                                                              blocked=blocked, threads_per_team=256,
                                                                              vec128=vec, outer_unroll=U))
                            except P.NestError:
                                continue
                            res.append(dict(L=L, S=S, mode=mode, blocked=blocked, vec=vec, U=U, ms=ms,
                                            GBs=B / ms / 1e6))
        print("cfg3 L", L, "done", flush=True)
    summary = {}
    for L in R.STENCIL_LS:
        allrows = [r for r in res if r["L"] == L]
        best = min(allrows, key=lambda r: r["ms"])
        s1 = min((r for r in allrows if r["S"] == 1), key=lambda r: r["ms"])
        # the mode study (generic / SPMD at each simdlen) on the scalar simd unit
        rows = [r for r in allrows if not r["vec"]]
        best_scalar = min(rows, key=lambda r: r["ms"])
        s1_scalar = min((r for r in rows if r["S"] == 1), key=lambda r: r["ms"])
        ratios = {}
        for S in (2, 4, 8, 16, 32):
            sp = min((r["ms"] for r in rows if r["S"] == S and r["mode"] == "spmd" and r["U"] == 1))
            ratios[S] = {m: min(r["ms"] for r in rows if r["S"] == S and r["mode"] == m) / sp
                         for m in ("generic_smem", "generic_shfl")}
        # honest HBM numbers: the best and the best simdlen-1 configuration again, one launch
        # per event pair with L2 flushed (and left clean) before it -- at L = 4 / 8 the whole
        # working set (50 / 84 MB) otherwise stays in the 126 MB L2 between graph replays
        inp, coef, w = R.stencil_inputs(N, L)
        t = [torch.from_numpy(a).cuda() for a in (inp, coef, w)]
        o = torch.empty(N, dtype=torch.float64, device="cuda")
        B = 8 * (N * L + 2) + 16 * N + 8 * L
        for r in (best, s1):
            r["ms_flushed"] = timed(lambda: P.nested_stencil_f64(*t, N, L, o, simdlen=r["S"], mode=r["mode"],
                                                                 blocked=r["blocked"], threads_per_team=256,
                                                                 vec128=r["vec"], outer_unroll=r["U"]), iters=20)
            r["GBs_flushed"] = B / r["ms_flushed"] / 1e6
        summary[L] = dict(best=best, simdlen1=s1, speedup_vs_simdlen1=s1["ms"] / best["ms"],
                          speedup_vs_simdlen1_flushed=s1["ms_flushed"] / best["ms_flushed"],
                          best_scalar=best_scalar,
                          scalar_speedup_vs_simdlen1=s1_scalar["ms"] / best_scalar["ms"],
                          generic_over_spmd=ratios)
    out["cfg3"] = dict(note="N=2^20 outer iterations; ms: 20 launches captured in a CUDA graph, replayed per event "
                            "pair (no flush, no host launch overhead -- L = 4/8 run from L2); ms_flushed: one launch "
                            "per event pair after a 512 MiB L2 flush (the HBM number)",
                       results=res, summary=summary)


def cfg4(out):
    Bn = 500_000
    A, x = R.batched_inputs(Bn)
    tA, tx = torch.from_numpy(A).cuda(), torch.from_numpy(x).cuda()
    y = torch.empty(Bn * 64, dtype=torch.float32, device="cuda")
    Bytes = Bn * (64 * 64 * 4 + 64 * 4 + 64 * 4)
    res = []
    for S in (1, 2, 4, 8, 16, 32):
        for mode in MODES:
            if S == 1 and mode != "spmd":
                continue
            for U in (1, 2, 4):
                for T in (256, 1024):
                    for vec in (False, True):
                        try:
                            ms = timed(lambda: P.batched_matvec_f32(tA, tx, Bn, 64, 64, y, simdlen=S, mode=mode,
                                                                    outer_unroll=U, threads_per_team=T,
                                                                    vec128=vec))
                        except P.NestError as e:
                            print("skip", S, mode, U, T, vec, str(e)[:80])
                            continue
                        res.append(dict(S=S, mode=mode, U=U, T=T, vec128=vec, ms=ms, GBs=Bytes / ms / 1e6))
    best = min(res, key=lambda r: r["ms"])
    s1 = min((r for r in res if r["S"] == 1), key=lambda r: r["ms"])
    out["cfg4"] = dict(alg_bytes=Bytes, results=res, best=best, simdlen1=s1,
                       speedup_vs_simdlen1=s1["ms"] / best["ms"])
    print("cfg4 done", flush=True)


def laplace(out):
    nz, ny, nx = R.LAPLACE_SHAPE
    u = torch.from_numpy(R.laplace_inputs(nz, ny, nx)).cuda()
    o = u.clone()
    B = 8 * nz * ny * nx + 8 * (nz - 2) * (ny - 2) * (nx - 2)   # u read once, interior written
    res = []
    for S in (1, 2, 4, 8, 16, 32):
        for mode in MODES:
            if S == 1 and mode != "spmd":
                continue
            for blocked in (False, True):
                for T in (256, 1024):
                    for vec in (False, True):   # scalar points / aligned pairs (LaplaceVecBody)
                        try:
                            ms = timed(lambda: P.laplace3d_f64(u, o, nz, ny, nx, 0.1, simdlen=S, mode=mode,
                                                               blocked=blocked, threads_per_team=T, vec128=vec),
                                       iters=7)
                        except P.NestError as e:   # e.g. T above the variant's register limit
                            print("skip laplace", S, mode, blocked, T, vec, str(e)[:60])
                            continue
                        res.append(dict(S=S, mode=mode, blocked=blocked, T=T, vec=vec, ms=ms, GBs=B / ms / 1e6))
    # Fig 10 (time over No-SIMD at S = 32) on the scalar simd unit, as in the paper
    sc = [r for r in res if not r["vec"]]
    s1 = min((r for r in sc if r["S"] == 1), key=lambda r: r["ms"])
    fig10 = {m: min(r["ms"] for r in sc if r["S"] == 32 and r["mode"] == m) / s1["ms"] for m in MODES}
    out["laplace"] = dict(shape=[nz, ny, nx], alg_bytes=B, results=res, best=min(res, key=lambda r: r["ms"]),
                          best_scalar=min(sc, key=lambda r: r["ms"]),
                          best_vec=min((r for r in res if r["vec"]), key=lambda r: r["ms"]),
                          no_simd=s1, fig10_time_over_no_simd_at_S32=fig10)
    print("laplace done", flush=True)


def g100(out):
    spec = R.G100
    rp, col, val = R.spmv_matrix(spec)
    x = R.spmv_x(spec)
    t = [torch.from_numpy(a).cuda() for a in (rp, col, val, x)]
    y = torch.empty(spec.nrows, dtype=torch.float64, device="cuda")
    B = val.size * 12 + (spec.nrows + 1) * 8 + spec.nrows * 8 + spec.ncols * 8
    res = []
    for S, mode, U, T, blocked, vec in ((1, "spmd", 1, 256, False, False), (1, "spmd", 1, 1024, True, True),
                                        (2, "spmd", 1, 1024, True, True), (2, "spmd", 1, 1024, True, False),
                                        (4, "spmd", 1, 1024, True, True), (2, "generic_smem", 1, 1024, True, True),
                                        (8, "spmd", 1, 1024, True, False)):
        ms = timed(lambda: P.spmv_csr_f64(*t, y, simdlen=S, mode=mode, outer_unroll=U, threads_per_team=T,
                                          blocked=blocked, vec128=vec), iters=10)
        res.append(dict(S=S, mode=mode, U=U, T=T, blocked=blocked, vec128=vec, ms=ms, GBs=B / ms / 1e6,
                        frac_of_8TBs=B / ms / 1e6 / 8000.0))
    # warm-x variant: L2 flushed, then x read once (x.sum()) before each timed launch
    best = min(res, key=lambda r: r["ms"])
    bcfg = dict(simdlen=best["S"], mode=best["mode"], outer_unroll=best["U"], threads_per_team=best["T"],
                blocked=best["blocked"], vec128=best["vec128"])
    ts = []
    for _ in range(10):
        P.l2_flush(flush)
        t[3].sum()
        e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
        e0.record()
        P.spmv_csr_f64(*t, y, **bcfg)
        e1.record()
        e1.synchronize()
        ts.append(e0.elapsed_time(e1))
    wms = statistics.median(ts)
    warm = dict(bcfg, ms=wms, GBs=B / wms / 1e6, note="x read into L2 before each launch (x is 100 MB: "
                "beyond the ~72-80 MB effective L2 for gathers, so only partly resident)")
    out["g100"] = dict(nnz=int(val.size), alg_bytes=B, results=res, best=best, warm_x=warm)
    print("g100 done", flush=True)


def cfg5(out):
    """BASELINE configs[4] (100M x 100M, U{8..24} nnz/row, 1.6G nonzeros) on ONE GPU:
    the headline and simdlen-1 configurations over the whole matrix, sampled
    parity against the oracle, and a single-GPU emulation of the P-rank row
    partition (each rank's rows as its own launch through the peer-gather
    kernel, every x slice on this GPU: NVLink traffic is not exercised)."""
    import numpy as np

    import oracle  # test infrastructure: the checker (bench-side use, not the product path)
    spec = R.CFG5
    rp, col, val = R.spmv_matrix(spec)
    x = R.spmv_x(spec)
    nnz = int(val.size)
    B = nnz * 12 + (spec.nrows + 1) * 8 + spec.nrows * 8 + spec.ncols * 8
    t = [torch.from_numpy(a).cuda() for a in (rp, col, val, x)]
    del col, val
    y = torch.empty(spec.nrows, dtype=torch.float64, device="cuda")
    res = []
    for S, flags in ((2, "bv"), (4, "bv"), (8, "bv"), (2, "bq"), (4, "bq"), (1, "bv"), (1, "bq"), (2, "b"), (4, "b"),
                     (1, "b"), (1, "")):
        cfg = dict(simdlen=S, threads_per_team=1024 if "b" in flags else 256, blocked="b" in flags,
                   vec128="v" in flags or "q" in flags, quad="q" in flags)
        ms = timed(lambda: P.spmv_csr_f64(*t, y, **cfg), iters=5)
        res.append(dict(cfg, ms=ms, GBs=B / ms / 1e6, frac_of_8TBs=B / ms / 1e6 / 8000.0))
    # sampled parity of the headline configuration (R3 tolerance)
    bcfg = {k: v for k, v in min(res, key=lambda r: r["ms"]).items() if k not in ("ms", "GBs", "frac_of_8TBs")}
    P.spmv_csr_f64(*t, y, **bcfg)
    yh = y.cpu().numpy()
    rng = np.random.default_rng(5)
    worst = 0.0
    for s0 in np.concatenate([[0, spec.nrows - 64], rng.integers(0, spec.nrows - 64, 6)]):
        rpl, cl, vl = R.spmv_matrix(spec, row_begin=int(s0), nrows=64)
        yr, ar = oracle.spmv_csr_f64(rpl, cl, vl, x)
        err = np.abs(yh[s0:s0 + 64] - yr)
        assert np.all(err <= 1e-12 * ar), f"cfg5 parity at rows {s0}"
        worst = max(worst, float(np.max(err / np.maximum(ar, 1e-300))))
    # row partition emulated on one GPU: rank r's rows and CSR slice, x split in P slices
    part = []
    y_pairs = torch.empty_like(y)
    best = min(res, key=lambda r: r["ms"])
    hcfg = {k: best[k] for k in ("simdlen", "threads_per_team", "blocked", "vec128")}
    P.spmv_csr_f64(*t, y_pairs, **hcfg)   # whole-matrix reference for the bitwise check (pairs)
    for Pn in (2, 4, 8):
        chunk = -(-spec.nrows // Pn)
        xc = -(-spec.ncols // Pn)
        xpad = torch.zeros(xc * Pn, dtype=torch.float64, device="cuda")
        xpad[:spec.ncols] = t[3]
        slices = [xpad[r * xc:(r + 1) * xc] for r in range(Pn)]
        for r in (0, Pn - 1):
            rb, re_ = r * chunk, min((r + 1) * chunk, spec.nrows)
            k0, k1 = int(rp[rb]), int(rp[re_])
            lrp = (t[0][rb:re_ + 1] - k0).contiguous()
            lcol, lval = t[1][k0:k1].clone(), t[2][k0:k1].clone()
            xp = P.XPeer(spec.ncols, nranks=Pn, rank=r, local_slices=slices)
            yl = torch.empty(re_ - rb, dtype=torch.float64, device="cuda")
            ms = timed(lambda: xp.spmv_csr_f64(spec.nrows, lrp, lcol, lval, yl, **hcfg), iters=5)
            same = bool(torch.equal(yl, y_pairs[rb:re_]))
            xp.close()
            Br = (k1 - k0) * 12 + (re_ - rb + 1) * 8 + (re_ - rb) * 8 + spec.ncols * 8
            part.append(dict(P=Pn, rank=r, rows=re_ - rb, nnz=k1 - k0, ms=ms, GBs=Br / ms / 1e6,
                             bitwise_equal_whole=same))
            del lrp, lcol, lval, yl
        del xpad, slices
    out["cfg5"] = dict(nnz=nnz, alg_bytes=B, results=res, best=min(res, key=lambda r: r["ms"]),
                       parity_worst_rel_err=worst, partition_emulation=part)
    del t
    torch.cuda.empty_cache()
    print("cfg5 done", json.dumps(out["cfg5"]["best"]), json.dumps(part), flush=True)


def fig9(out):
    """Fig 9 analogue: CSR SpMV time per simdlen and mode on the
    short-row cfg2 matrix and its all-far variant, best variant per (S, mode)
    among blocked teams of 1024 with scalar / 128-bit pair / quad loads, each with
    and without x persisting in L2 (NEST_F_X_L2_PERSIST)."""
    res = {}
    for spec in (R.CFG2, R.CFG2_UNIFORM):
        rp, col, val = R.spmv_matrix(spec)
        x = R.spmv_x(spec)
        t = [torch.from_numpy(a).cuda() for a in (rp, col, val, x)]
        y = torch.empty(spec.nrows, dtype=torch.float64, device="cuda")
        B = val.size * 12 + (spec.nrows + 1) * 8 + spec.nrows * 8 + spec.ncols * 8
        rows = []
        for S in (1, 2, 4, 8, 16, 32):
            for mode in (("spmd",) if S == 1 else MODES):
                best = None
                # U > 1 in SPMD: U rows per group in flight, reduced together (transpose-reduce)
                variants = [(f, 1, 1024) for f in ("b", "bv", "bq", "bp", "bvp", "bqp")]
                if mode == "spmd" and S > 1:
                    variants += [(f, U, T) for f in ("b", "bv", "bvp") for U in (2, 4) for T in (512, 1024)]
                for flags, U, T in variants:
                    cfg = dict(simdlen=S, mode=mode, threads_per_team=T, blocked=True, vec128="v" in flags or
                               "q" in flags, quad="q" in flags, outer_unroll=U, x_l2_persist="p" in flags)
                    try:
                        ms = timed(lambda: P.spmv_csr_f64(*t, y, **cfg), iters=5)
                    except P.NestError:
                        continue
                    if best is None or ms < best["ms"]:
                        best = dict(S=S, mode=mode, variant=flags, U=U, T=T, ms=ms, GBs=B / ms / 1e6)
                rows.append(best)
        s1 = rows[0]["ms"]
        for r in rows:
            r["speedup_vs_simdlen1"] = s1 / r["ms"]
        res[spec.name] = dict(alg_bytes=B, results=rows)
        del t
        torch.cuda.empty_cache()
    out["fig9"] = res
    print("fig9 done", flush=True)


def teams(out):
    """NEXT-1: the paper's two-level baseline (teams distribute in generic mode +
    parallel for) against the three-level path, CFG2 matrix."""
    spec = R.CFG2
    rp, col, val = R.spmv_matrix(spec)
    x = R.spmv_x(spec)
    t = [torch.from_numpy(a).cuda() for a in (rp, col, val, x)]
    y = torch.empty(spec.nrows, dtype=torch.float64, device="cuda")
    B = val.size * 12 + (spec.nrows + 1) * 8 + spec.nrows * 8 + spec.ncols * 8
    res = []
    for T in (32, 64, 128, 256):
        for teams_ in (0, 148 * 4, 148 * 16):
            try:
                ms = timed(lambda: P.spmv_csr_f64(*t, y, simdlen=1, mode="teams_generic", threads_per_team=T,
                                                  num_teams=teams_), iters=5)
            except P.NestError as e:
                print("skip", T, teams_, str(e)[:80])
                continue
            res.append(dict(level=2, T=T, num_teams=teams_, ms=ms, GBs=B / ms / 1e6))
    for S, mode, T, blocked, vec in ((1, "spmd", 1024, True, True), (2, "spmd", 1024, True, True),
                                     (2, "generic_smem", 1024, True, True), (4, "spmd", 1024, True, True),
                                     (8, "generic_smem", 256, False, False)):
        ms = timed(lambda: P.spmv_csr_f64(*t, y, simdlen=S, mode=mode, threads_per_team=T, blocked=blocked,
                                          vec128=vec), iters=10)
        res.append(dict(level=3, S=S, mode=mode, T=T, blocked=blocked, vec128=vec, ms=ms, GBs=B / ms / 1e6))
    two = min((r for r in res if r["level"] == 2), key=lambda r: r["ms"])
    three = min((r for r in res if r["level"] == 3), key=lambda r: r["ms"])
    out["teams"] = dict(alg_bytes=B, results=res, best_two_level=two, best_three_level=three,
                        speedup_three_over_two=two["ms"] / three["ms"])
    print("teams done", flush=True)


def main():
    global flush
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default="gpurun_out/suite.json")
    ap.add_argument("--only", default="cfg3,cfg4,g100,laplace,teams")
    a = ap.parse_args()
    flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
    out = {}
    for name in a.only.split(","):
        globals()[name](out)
    os.makedirs(os.path.dirname(a.out) or ".", exist_ok=True)
    with open(a.out, "w") as f:
        json.dump(out, f, indent=1)
    if "teams" in out:
        print("teams 3-level/2-level speedup", out["teams"]["speedup_three_over_two"], out["teams"]["best_two_level"])
    for k in ("cfg3", "cfg4", "g100", "laplace"):
        if k in out:
            v = out[k]
            print(k, json.dumps(v.get("summary", v.get("best")), default=str)[:2000])
            if k == "laplace":
                print("fig10", v["fig10_time_over_no_simd_at_S32"])


if __name__ == "__main__":
    main()
