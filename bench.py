"""Benchmark: the three-level CSR SpMV hot path on B200 (BASELINE.json metric
"3-level SpMV GB/s vs HBM peak; speedup over simd-folded 2-level mapping").

One step = one y = A x over BASELINE.json configs[1] (10M x 10M CSR, nnz/row
U{4..12} banded+far, fp64) through the C ABI, in the best (simdlen, mode,
variant) found by a short untimed autotune; the simd-folded two-level mapping
(simdlen = 1) is timed the same way for the speedup.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]

N > 1 (torchrun, one rank per GPU): the row-partitioned SpMV with the NCCL
all-gather of x (BASELINE.json configs[4] scheme), weak scaling with 10M rows
per rank.  --impl reference times the CPU oracle (the only reference this
paper-only tier has) on the same workload.  Prints ONE JSON line on rank 0.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

from nestgen import recipes as R  # noqa: E402

METRIC = "3-level SpMV GB/s vs HBM peak; speedup over simd-folded 2-level mapping"
UNIT = "GB/s"
SPEC = R.CFG2


def alg_bytes(nrows: int, ncols: int, nnz: int) -> int:
    """Algorithmic bytes of one SpMV: the CSR arrays once,
    x once, y written once."""
    return nnz * (8 + 4) + (nrows + 1) * 8 + nrows * 8 + ncols * 8


def peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            p = json.load(f)
        return float(p["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md)"


class ClockSampler:
    """nvidia-smi-equivalent clock / throttle sampling through NVML, run during
    the timed region."""

    def __init__(self, index: int, period: float = 0.002):
        self.samples, self.reasons = [], set()
        self.max_mhz = None
        self._stop = threading.Event()
        self._period = period
        try:
            import pynvml
            pynvml.nvmlInit()
            self._nv = pynvml
            self._h = pynvml.nvmlDeviceGetHandleByIndex(index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self._h, pynvml.NVML_CLOCK_SM)
        except Exception:
            self._nv = None
        self._t = threading.Thread(target=self._run, daemon=True)

    def _run(self):
        nv = self._nv
        names = {}
        if nv is not None:
            for k in ("HwSlowdown", "HwThermalSlowdown", "SwThermalSlowdown", "SwPowerCap",
                      "HwPowerBrakeSlowdown", "SyncBoost", "ApplicationsClocksSetting", "GpuIdle"):
                v = getattr(nv, "nvmlClocksEventReason" + k, None) or getattr(nv, "nvmlClocksThrottleReason" + k, None)
                if v is not None:
                    names[k] = v
        while not self._stop.is_set():
            if nv is not None:
                try:
                    self.samples.append(nv.nvmlDeviceGetClockInfo(self._h, nv.NVML_CLOCK_SM))
                    r = nv.nvmlDeviceGetCurrentClocksEventReasons(self._h)
                    for k, bit in names.items():
                        if r & bit and k != "GpuIdle":
                            self.reasons.add(k)
                except Exception:
                    pass
            time.sleep(self._period)

    def __enter__(self):
        self._t.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        self._t.join()

    def summary(self):
        return {"sm_mhz": statistics.median(self.samples) if self.samples else None,
                "sm_max_mhz": self.max_mhz, "samples": len(self.samples),
                "reasons": sorted(self.reasons)}


# ---------------------------------------------------------------- CPU oracle
def cpu_baseline(spec, min_seconds=10.0, max_seconds=30.0):
    """The oracle as it stands (plain sequential C, 1 thread) on a bounded
    sample: whole passes of the same matrix until >= min_seconds."""
    import oracle
    rp, col, val = R.spmv_matrix(spec)
    x = R.spmv_x(spec)
    B = alg_bytes(spec.nrows, spec.ncols, val.size)
    passes, t_total = 0, 0.0
    while t_total < min_seconds and (passes == 0 or t_total + t_total / passes < max_seconds):
        t0 = time.perf_counter()
        oracle.spmv_csr_f64(rp, col, val, x)
        t_total += time.perf_counter() - t0
        passes += 1
    return {"value": B * passes / t_total / 1e9, "unit": UNIT, "cores": 1, "kind": "oracle",
            "sample": f"{passes} full passes of {spec.name} ({spec.nrows} rows, {val.size} nnz), "
                      f"{t_total:.1f} s single-threaded C (oracle/oracle.c)",
            "host": host_cpu()}


def host_cpu():
    """The box's CPU model and logical core count (context for cpu_baseline)."""
    model = "unknown"
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    model = line.split(":", 1)[1].strip()
                    break
    except OSError:
        pass
    return {"model": model, "logical_cores": os.cpu_count()}


def run_reference(args, rank, world):
    """--impl reference: the oracle on the box's host cores, rank 0 only."""
    if rank != 0:
        return
    import oracle
    spec = SPEC
    rp, col, val = R.spmv_matrix(spec)
    x = R.spmv_x(spec)
    B = alg_bytes(spec.nrows, spec.ncols, val.size)
    for _ in range(args.warmup):
        oracle.spmv_csr_f64(rp, col, val, x)
    ts = []
    for _ in range(args.steps):
        t0 = time.perf_counter()
        oracle.spmv_csr_f64(rp, col, val, x)
        ts.append(time.perf_counter() - t0)
    ms = 1e3 * sum(ts) / len(ts)
    value = B / (ms / 1e3) / 1e9
    line = {"metric": METRIC, "value": value, "unit": UNIT, "impl": "reference", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": f"{spec.name}: CSR SpMV fp64 {spec.nrows}x{spec.ncols}, nnz/row "
                                   f"U{{{spec.nnz_min}..{spec.nnz_max}}} banded+far (W={spec.band_w}, "
                                   f"far 1/{spec.far_den})", "nnz": int(val.size), "alg_bytes": B},
            "cpu_baseline": {"value": value, "unit": UNIT, "cores": 1, "kind": "oracle",
                             "sample": f"the full {spec.name} matrix per step, single-threaded C oracle", "host": host_cpu()},
            "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ---------------------------------------------------------------- GPU arm
# (simdlen, mode, outer_unroll, threads_per_team, x_halo, flags) -- flags: "b" blocked
# team schedule, "s" staged pipeline, "h" streaming cache hints, "v" 128-bit pair
# loads, "q" 128-bit quad loads
CANDIDATES = [
    (1, "spmd", 1, 256, 0, ""),
    (1, "spmd", 1, 1024, 0, "b"),
    (1, "spmd", 1, 1024, 0, "bv"),
    (1, "spmd", 1, 1024, 0, "bq"),
    (2, "spmd", 1, 1024, 0, "b"),
    (2, "spmd", 1, 1024, 0, "bv"),
    (2, "generic_smem", 1, 1024, 0, "b"),
    (2, "generic_shfl", 1, 1024, 0, "b"),
    (2, "generic_smem", 1, 1024, 0, "bq"),
    (4, "spmd", 1, 1024, 0, "b"),
    (4, "spmd", 1, 1024, 0, "bv"),
    (2, "spmd", 1, 1024, 0, "bq"),
    (4, "spmd", 1, 1024, 0, "bq"),
    (4, "generic_smem", 1, 1024, 0, "b"),
    (4, "generic_shfl", 1, 1024, 0, "b"),
    (8, "spmd", 1, 1024, 0, "b"),
    (8, "generic_smem", 1, 1024, 0, "b"),
    (16, "spmd", 1, 1024, 0, "b"),
    (32, "spmd", 1, 1024, 0, "b"),
    (4, "spmd", 1, 512, 4096, "s"),
]

# The headline: the best measured THREE-level configuration (simdlen >= 2; the
# metric is the 3-level mapping's GB/s): simdlen 2, SPMD, blocked teams of 1024,
# 128-bit pair loads.  The 2-level comparison point is the best simdlen-1 candidate.
HEADLINE = (2, "spmd", 1, 1024, 0, "bv")


def cfg_of(c):
    S, mode, U, T, halo, fl = c
    return dict(simdlen=S, mode=mode, outer_unroll=U, threads_per_team=T, x_halo=halo,
                stream_hints="h" in fl, staged="s" in fl, blocked="b" in fl, vec128="v" in fl or "q" in fl,
                quad="q" in fl)


def time_steps(torch, fn, flush, P, iters, events_out=None):
    """Per-step CUDA-event times (ms) on the current stream, L2 flushed between steps."""
    ts = []
    for _ in range(iters):
        P.l2_flush(flush)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        fn()
        e1.record()
        ts.append((e0, e1))
    torch.cuda.synchronize()
    return [a.elapsed_time(b) for a, b in ts]


def run_gpu(args, rank, world, local_rank):
    import torch
    import torch.distributed as dist

    import paper_conf_icpp_wrightdtcc23_b200 as P

    torch.cuda.set_device(local_rank)
    dev = torch.device("cuda", local_rank)
    spec = SPEC
    if world > 1:
        gspec = R.SpmvSpec(f"{spec.name}x{world}", spec.seed, spec.nrows * world, spec.ncols * world,
                           spec.nnz_min, spec.nnz_max, spec.structure, spec.band_w, spec.far_den)
        chunk, rb, nloc = P.shard_rows(gspec.nrows, world, rank)
    else:
        gspec, rb, nloc = spec, 0, spec.nrows
    rp, col, val = R.spmv_matrix(gspec, row_begin=rb, nrows=nloc)
    nnz = int(val.size)
    pin = lambda a: torch.from_numpy(a).pin_memory()
    h_rp, h_col, h_val = pin(rp), pin(col), pin(val)
    d_rp, d_col, d_val = (h_rp.to(dev), h_col.to(dev), h_val.to(dev))
    flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)   # 4x the 126 MB L2
    peak, peak_src = peaks()

    if world == 1:
        x = R.spmv_x(spec)
        h_x = pin(x)
        d_x = h_x.to(dev)
        d_y = torch.empty(spec.nrows, dtype=torch.float64, device=dev)
        B = alg_bytes(spec.nrows, spec.ncols, nnz)

        # untimed autotune over the candidate (simdlen, mode, variant) set
        sweep = []
        for c in CANDIDATES:
            cfg = cfg_of(c)
            fn = lambda cfg=cfg: P.spmv_csr_f64(d_rp, d_col, d_val, d_x, d_y, **cfg)
            try:
                fn()
            except P.NestError as e:
                print(f"skip {c}: {e}", file=sys.stderr)
                continue
            ts = time_steps(torch, fn, flush, P, 5)
            sweep.append((statistics.median(ts), c))
        sweep.sort(key=lambda t: t[0])
        # the timed configuration is fixed (reproducible under a profiler); --autotune
        # times the fastest candidate of this run's sweep instead
        best = min((t for t in sweep if t[1][0] >= 2), key=lambda t: t[0])[1] if args.autotune else HEADLINE
        s1 = min((t for t in sweep if t[1][0] == 1), key=lambda t: t[0])   # best 2-level (simdlen 1)
        cfg = cfg_of(best)
        step = lambda: P.spmv_csr_f64(d_rp, d_col, d_val, d_x, d_y, **cfg)

        for _ in range(args.warmup):
            step()
        torch.cuda.synchronize()
        # timed region: K steps, L2 flushed between steps (flush outside the events)
        with ClockSampler(local_rank) as clk:
            torch.cuda.synchronize()
            ts = time_steps(torch, step, flush, P, args.steps)
            torch.cuda.synchronize()
        ms = sum(ts) / len(ts)
        value = B / (ms / 1e3) / 1e9
        # simd-folded two-level mapping (simdlen = 1), same protocol
        s1_cfg = cfg_of(s1[1])
        ts1 = time_steps(torch, lambda: P.spmv_csr_f64(d_rp, d_col, d_val, d_x, d_y, **s1_cfg), flush, P,
                         max(3, args.steps // 2))
        ms1 = sum(ts1) / len(ts1)

        # e2e through the C ABI with HOST buffers: H2D of A and x, the SpMV, D2H of y
        h_y = torch.empty(spec.nrows, dtype=torch.float64).pin_memory()
        ws = torch.empty(P.hostio_workspace_bytes(spec.nrows, spec.ncols, nnz), dtype=torch.uint8, device=dev)
        e2e_step = lambda: P.spmv_csr_f64_hostio(h_rp, h_col, h_val, h_x, h_y, ws, **cfg)
        e2e_step()
        torch.cuda.synchronize()
        n_e2e = max(3, min(args.steps, 10))
        te = []
        for _ in range(n_e2e):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            e2e_step()
            e1.record()
            e1.synchronize()
            te.append(e0.elapsed_time(e1))
        ms_e2e = sum(te) / len(te)
        h2d = (spec.nrows + 1) * 8 + nnz * 12 + spec.ncols * 8
        d2h = spec.nrows * 8

        body = ("SpmvVecBody<0,4>" if "q" in best[5] else "SpmvVecBody<0,2>" if "v" in best[5]
                else f"SpmvBody<{int('h' in best[5])},0>")
        kname = ("nest_kernel_2pm" if ("v" in best[5] or "q" in best[5]) and best[2] == 1
                 and not ("q" in best[5] and best[0] == 1) else "nest_kernel")
        kernel_name = (f"spmv_staged_kernel<S={best[0]},{best[1]},SUM,U={best[2]}>" if "s" in best[5] else
                       f"{kname}<S={best[0]},{best[1]},SUM,U={best[2]},{body}>")
        traffic = None
        try:
            with open(os.path.join(ROOT, "profiles", "traffic.json")) as f:
                traffic = json.load(f).get(json.dumps(list(best)))

        except Exception:
            pass
        line = {
            "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": 1, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": f"{spec.name}: CSR SpMV fp64 {spec.nrows}x{spec.ncols}, nnz/row "
                                   f"U{{{spec.nnz_min}..{spec.nnz_max}}} banded+far (W={spec.band_w}, far "
                                   f"1/{spec.far_den}), seed {spec.seed} (BASELINE.json configs[1])",
                       "nnz": nnz, "alg_bytes": B, "simdlen": best[0], "mode": best[1],
                       "outer_unroll": best[2], "threads_per_team": best[3], "x_halo": best[4],
                       "variant": " + ".join({"b": "blocked teams", "s": "staged pipeline", "h": "stream hints",
                                              "v": "128-bit pair loads", "q": "128-bit quad loads"}[f]
                                             for f in best[5]) or "cyclic teams",
                       "l2": "flushed between timed steps (512 MiB write, then a 256 MiB read so L2 holds only clean lines)",
                       "parallelism": "1 GPU"},
            "speedup_vs_simdlen1": ms1 / ms,
            "simdlen1": {"ms_per_step": ms1, "GBs": B / (ms1 / 1e3) / 1e9, "config": cfg_of(s1[1])},
            "sweep_ms": {json.dumps(list(c)): round(t, 4) for t, c in sweep},
            "roofline": {"bound": "hbm", "achieved": value, "peak": peak, "unit": "GB/s",
                         "frac": value / peak, "traffic": traffic, "peak_source": peak_src,
                         "traffic_source": "profiles/traffic.json: dram read+write bytes per launch, ncu --set full",
                         "traffic_over_alg_bytes": (traffic / B) if traffic else None,
                         "kernel": kernel_name, "frac_of_8TBs_spec": value / 8000.0},
            "e2e": {"value": B / (ms_e2e / 1e3) / 1e9, "unit": UNIT, "h2d_bytes_per_step": h2d,
                    "d2h_bytes_per_step": d2h, "ms_per_step": ms_e2e,
                    "h2d_gbs": h2d / (ms_e2e / 1e3) / 1e9,
                    "pipeline": (f"{int(os.environ['NEST_HOSTIO_CHUNKS'])} row chunks (forced)"
                                 if os.environ.get("NEST_HOSTIO_CHUNKS") else
                                 f"{min(32, max(1, -(-nnz // (8 << 20))))} row chunks of ~8 Mi nonzeros")
                    + ": chunk c's SpMV and y copy overlap the H2D of chunks > c"},
            "gpu_launches": 3 * args.steps,
            "gpu_launches_detail": "per step: 1 SpMV kernel + 2 l2 flush kernels (write, clean-read; outside the step events)",
            "clocks": clk.summary(),
        }
        if not args.no_cpu_baseline:
            line["cpu_baseline"] = cpu_baseline(spec)
        print(json.dumps(line), flush=True)
        return

    # ---- N > 1: row-partitioned SpMV (weak scaling: spec.nrows rows per rank).
    # Two exchange strategies, both timed: "xpeer" (NEXT-4, the headline) -- x
    # stays distributed and the SpMV's simd lanes gather remote x from the
    # owner's slice over NVLink, bracketed by peer-memory barriers -- and
    # "allgather" (a12) -- NCCL all-gather of x into x_full, then the local SpMV.
    cfg = cfg_of(HEADLINE)
    xchunk = -(-gspec.ncols // world)
    xb = min(rank * xchunk, gspec.ncols)
    xl = R.spmv_x(gspec, begin=xb, n=min(xchunk, gspec.ncols - xb))
    h_xl = torch.zeros(xchunk, dtype=torch.float64).pin_memory()
    h_xl[:xl.size] = torch.from_numpy(xl)
    d_xl = h_xl.to(dev)
    d_y = torch.empty(nloc, dtype=torch.float64, device=dev)
    nnz_t = torch.tensor([nnz], dtype=torch.int64, device=dev)
    dist.all_reduce(nnz_t)
    B = alg_bytes(gspec.nrows, gspec.ncols, int(nnz_t.item()))

    def timed(step, iters):
        for _ in range(args.warmup):
            step()
        torch.cuda.synchronize()
        dist.barrier()
        with ClockSampler(local_rank) as clk:
            torch.cuda.synchronize()
            ts = time_steps(torch, step, flush, P, iters)
            torch.cuda.synchronize()
        dist.barrier()
        t = torch.tensor([sum(ts) / len(ts)], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)   # max over ranks
        return float(t.item()), clk.summary()

    res = {}
    comm = None
    y_ag = None
    if not SHARE_GPU:   # NCCL needs one GPU per rank
        comm = P.Comm()
        d_xf = torch.empty(xchunk * world, dtype=torch.float64, device=dev)
        res["allgather"] = timed(lambda: comm.spmv_csr_f64(gspec.nrows, gspec.ncols, d_rp, d_col, d_val, d_xl,
                                                           d_xf, d_y, **cfg), args.steps)
        y_ag = d_y.clone()
    xp_err = None
    try:
        xp = P.XPeer(gspec.ncols)
        xp.set_local_x(d_xl)
        res["xpeer"] = timed(lambda: xp.spmv_csr_f64(gspec.nrows, d_rp, d_col, d_val, d_y, **cfg), args.steps)
        # R16: same rows, same variant -> same bits (even nnz offsets)
        same = bool(torch.equal(d_y, y_ag)) if y_ag is not None else None
        # e2e through the public API: H2D of the local CSR and x slice from pinned
        # memory, the peer-gather SpMV, D2H of y_local -- all inside the timed region
        h_y = torch.empty(nloc, dtype=torch.float64).pin_memory()

        def e2e_step():
            a = h_rp.to(dev, non_blocking=True)
            c = h_col.to(dev, non_blocking=True)
            v = h_val.to(dev, non_blocking=True)
            xl_d = h_xl.to(dev, non_blocking=True)
            xp.set_local_x(xl_d)
            h_y.copy_(xp.spmv_csr_f64(gspec.nrows, a, c, v, **cfg), non_blocking=True)
        ms_e2e, _ = timed(e2e_step, max(3, args.steps // 20))
        e2e = {"value": B / (ms_e2e / 1e3) / 1e9, "unit": UNIT, "ms_per_step": ms_e2e,
               "h2d_bytes_per_step": (h_rp.numel() + h_col.numel() // 2 + h_val.numel() + h_xl.numel()) * 8,
               "d2h_bytes_per_step": nloc * 8}
    except P.NestError as e:   # reported, and the all-gather number stands in
        xp_err, same, e2e = str(e), None, None
    head = "xpeer" if "xpeer" in res else "allgather"
    ms, clocks = res[head]
    if rank == 0:
        line = {"metric": METRIC, "value": B / (ms / 1e3) / 1e9, "unit": UNIT, "n_gpus": world,
                "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True,
                "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
                "config": {"workload": f"row-partitioned CSR SpMV fp64, {spec.nrows} rows per rank "
                                       f"(global {gspec.nrows}), nnz/row U{{{spec.nnz_min}..{spec.nnz_max}}}, "
                                       f"banded+far; x exchange: {head}", "parallelism": f"rows/{world}",
                           "l2": "flushed between timed steps", "variant": "blocked teams + 128-bit pair loads",
                           **cfg},
                "exchange": {k: {"ms_per_step": v[0], "GBs": B / (v[0] / 1e3) / 1e9} for k, v in res.items()},
                "xpeer_error": xp_err, "xpeer_bitwise_equal_allgather": same,
                "gpu_launches": args.steps * (3 if head == "xpeer" else 1),
                "gpu_launches_detail": ("per step: barrier + SpMV + barrier kernels (+ l2_flush outside the events)"
                                        if head == "xpeer" else "per step: SpMV kernel + NCCL all-gather"),
                "clocks": clocks, "e2e": e2e}
        peak, peak_src = peaks()
        per_gpu = line["value"] / world
        line["roofline"] = {"bound": "hbm", "achieved": per_gpu, "peak": peak, "unit": "GB/s",
                            "frac": per_gpu / peak, "traffic": None, "peak_source": peak_src,
                            "kernel": f"nest_kernel_2pm<S={cfg['simdlen']},{cfg['mode']},SUM,U=1,SpmvVecBody<0,2,int,"
                                      f"{'XPeer' if head == 'xpeer' else 'XLocal'}>>",
                            "note": "per GPU: algorithmic bytes of all ranks / world / max-over-ranks step time"}
        print(json.dumps(line), flush=True)
    if "xpeer" in res:
        xp.close()
    if comm is not None:
        comm.close()


# Developer check of the N > 1 code path on a one-GPU box: every rank on cuda:0,
# gloo process group, the NCCL all-gather leg skipped (timings are meaningless).
SHARE_GPU = os.environ.get("NEST_BENCH_SHARE_GPU") == "1"


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--autotune", action="store_true", help="time the fastest candidate of the sweep")
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3)
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = 0 if SHARE_GPU else int(os.environ.get("LOCAL_RANK", "0"))
    if world > 1:
        import torch.distributed as dist
        backend = "gloo" if args.impl == "reference" or SHARE_GPU else "nccl"
        if backend == "nccl":
            import torch
            torch.cuda.set_device(local_rank)
        dist.init_process_group(backend)
    try:
        if args.impl == "reference":
            run_reference(args, rank, world)
        else:
            run_gpu(args, rank, world, local_rank)
    finally:
        if world > 1:
            import torch.distributed as dist
            dist.destroy_process_group()


if __name__ == "__main__":
    main()
