"""Benchmark: the three-level CSR SpMV hot path on B200 (BASELINE.json metric
"3-level SpMV GB/s vs HBM peak; speedup over simd-folded 2-level mapping").

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]

N = 1: one step = one y = A x over BASELINE.json configs[1] (10M x 10M CSR,
nnz/row U{4..12} banded+far, fp64) through the C ABI in the headline
configuration (simdlen 2, SPMD, blocked teams, quad tuples); ``value`` is its
algorithmic GB/s.  The same line carries the simd-folded two-level mapping
(simdlen 1) timed the same way, a short sweep of (simdlen, mode, variant), the
north_star's 100M-nnz gate matrix (G100) and configs[4] on one GPU (100M rows,
1.6G nonzeros) as extra legs with their own roofline, the end-to-end call from
pinned host buffers, and the CPU oracle (1 thread and all cores).

N > 1 (torchrun, one rank per GPU): configs[4] -- 100M rows, U{8..24} nnz/row --
row-partitioned over the ranks at FIXED total size (strong scaling); each rank
generates only its own rows.  A step is the NCCL all-gather of x plus the local
SpMV (a12); the all-gather and the local SpMV are also timed alone, the peer-
gather variant (NEXT-4) beside them, every rank's rows are checked against the
oracle, and the line carries the end-to-end host-buffer call.

--impl reference: the CPU oracle (this paper-only tier has no installable
reference implementation) on the same workload, rank 0 only.
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
SPEC_MULTI = R.CFG5
FLUSH_BYTES = 512 << 20   # 4x the 126 MB L2


def alg_bytes(nrows: int, ncols: int, nnz: int) -> int:
    """Algorithmic bytes of one SpMV: the CSR arrays once,
    x once, y written once."""
    return nnz * (8 + 4) + (nrows + 1) * 8 + nrows * 8 + ncols * 8


def workload(spec, which: str = "configs[1]") -> str:
    """The workload string -- identical in both arms (--impl ours / reference)."""
    return (f"{spec.name}: CSR SpMV fp64 {spec.nrows}x{spec.ncols}, nnz/row U{{{spec.nnz_min}..{spec.nnz_max}}} "
            f"banded+far (W={spec.band_w}, far 1/{spec.far_den}), seed {spec.seed} (BASELINE.json {which})")


def peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            p = json.load(f)
        return float(p["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md)"


def traffic_of(key: str):
    """ncu dram read+write bytes per launch for a (workload, config) key, from the
    committed capture summary profiles/traffic.json (None if not captured)."""
    try:
        with open(os.path.join(ROOT, "profiles", "traffic.json")) as f:
            return json.load(f).get(key)
    except Exception:
        return None


class ClockSampler:
    """nvidia-smi-equivalent clock / throttle sampling through NVML, run during
    the timed region."""

    def __init__(self, index: int, period: float = 0.001):
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

    def _sample_once(self):
        nv = self._nv
        if nv is not None:
            try:
                self.samples.append(nv.nvmlDeviceGetClockInfo(self._h, nv.NVML_CLOCK_SM))
            except Exception:
                pass

    def __enter__(self):
        # short thread switch interval so the sampler runs while the main thread
        # enqueues steps (the timed region is tens of ms); one sample on each edge
        self._switch = sys.getswitchinterval()
        sys.setswitchinterval(2e-4)
        self._t.start()
        return self

    def __exit__(self, *a):
        self._sample_once()
        self._stop.set()
        self._t.join()
        sys.setswitchinterval(self._switch)

    def summary(self):
        return {"sm_mhz": statistics.median(self.samples) if self.samples else None,
                "sm_max_mhz": self.max_mhz, "samples": len(self.samples),
                "reasons": sorted(self.reasons)}


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


# ---------------------------------------------------------------- CPU oracle
def cpu_baseline(spec, rp, col, val, x, min_seconds=8.0, max_seconds=20.0):
    """The oracle as it stands on a bounded sample: whole passes of the same
    matrix for >= min_seconds on ONE thread (the baseline of record), then the
    same per-row loop on all host cores (OpenMP over rows, bit-identical)."""
    import oracle
    B = alg_bytes(spec.nrows, spec.ncols, val.size)

    def timed(fn):
        passes, t_total = 0, 0.0
        while t_total < min_seconds and (passes == 0 or t_total + t_total / passes < max_seconds):
            t0 = time.perf_counter()
            fn()
            t_total += time.perf_counter() - t0
            passes += 1
        return passes, t_total

    p1, t1 = timed(lambda: oracle.spmv_csr_f64(rp, col, val, x))
    ncores = os.cpu_count() or 1
    used = [1]

    def allcores():
        used[0] = oracle.spmv_csr_f64_threads(rp, col, val, x, ncores)[2]
    pn, tn = timed(allcores)
    return {"value": B * p1 / t1 / 1e9, "unit": UNIT, "cores": 1, "kind": "oracle",
            "sample": f"{p1} full passes of {spec.name} ({spec.nrows} rows, {val.size} nnz), {t1:.1f} s, "
                      "single-threaded C (oracle/oracle.c)",
            "all_cores": {"value": B * pn / tn / 1e9, "unit": UNIT, "cores": used[0], "kind": "oracle",
                          "sample": f"{pn} full passes, {tn:.1f} s, the same per-row loop on {used[0]} threads "
                                    "(OpenMP over rows, bit-identical to 1 thread)"},
            "host": host_cpu()}


def run_reference(args, rank, world):
    """--impl reference: the oracle on the box's host cores, rank 0 only; the
    workload string, metric and unit are the GPU arm's.  N = 1: the whole
    configs[1] matrix per step; N > 1: configs[4] (the GPU arm's workload there)
    on a bounded sample per step (its first 5M rows), so the run stays short."""
    if rank != 0:
        return
    import oracle
    if world == 1:
        spec, which, nrows = SPEC, "configs[1]", SPEC.nrows
    else:
        spec, which, nrows = SPEC_MULTI, "configs[4], row-partitioned at fixed total size", 5_000_000
    rp, col, val = R.spmv_matrix(spec, row_begin=0, nrows=nrows)
    x = R.spmv_x(spec)
    B = alg_bytes(nrows, spec.ncols, val.size)
    for _ in range(args.warmup):
        oracle.spmv_csr_f64(rp, col, val, x)
    ts = []
    for _ in range(args.steps):
        t0 = time.perf_counter()
        oracle.spmv_csr_f64(rp, col, val, x)
        ts.append(time.perf_counter() - t0)
    ms = 1e3 * sum(ts) / len(ts)
    value = B / (ms / 1e3) / 1e9
    sample = (f"the full {spec.name} matrix per step" if nrows == spec.nrows else
              f"rows [0, {nrows}) of {spec.name} ({val.size} nnz) per step")
    line = {"metric": METRIC, "value": value, "unit": UNIT, "impl": "reference", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True,
            "scaling": "weak" if world == 1 else "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": workload(spec, which), "nnz_per_step": int(val.size), "alg_bytes_per_step": B},
            "cpu_baseline": {"value": value, "unit": UNIT, "cores": 1, "kind": "oracle",
                             "sample": f"{sample}, single-threaded C oracle", "host": host_cpu()},
            "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ---------------------------------------------------------------- GPU arm
# (simdlen, mode, outer_unroll, threads_per_team, x_halo, flags) -- flags: "b" blocked
# team schedule, "v" 128-bit pair loads, "q" 128-bit quad loads, "h" streaming cache
# hints, "p" x under a persisting-L2 access-policy window (NEST_F_X_L2_PERSIST); x_halo
# > 0 is the x ring (teams_per_sm chosen by the planner); SPMD with outer_unroll > 1
# reduces its U rows together (transpose-reduce)
CANDIDATES = [
    (1, "spmd", 1, 256, 0, ""),
    (1, "spmd", 1, 1024, 0, "bv"),
    (1, "spmd", 1, 1024, 0, "bq"),
    (1, "spmd", 1, 1024, 0, "bvp"),
    (1, "spmd", 1, 1024, 0, "bqp"),
    (2, "spmd", 1, 1024, 0, "b"),
    (2, "spmd", 1, 1024, 0, "bv"),
    (2, "spmd", 1, 1024, 0, "bq"),
    (2, "spmd", 1, 1024, 0, "bvp"),
    (2, "spmd", 1, 1024, 0, "bqp"),
    (2, "generic_smem", 1, 1024, 0, "b"),
    (2, "generic_shfl", 1, 1024, 0, "b"),
    (2, "generic_smem", 1, 1024, 0, "bqp"),
    (2, "generic_shfl", 1, 1024, 0, "bqp"),
    (4, "spmd", 1, 1024, 0, "bv"),
    (4, "spmd", 1, 1024, 0, "bq"),
    (4, "spmd", 1, 1024, 0, "bqp"),
    (4, "generic_smem", 1, 1024, 0, "b"),
    (8, "spmd", 1, 1024, 0, "bv"),
    (8, "spmd", 2, 1024, 0, "bv"),
    (8, "spmd", 1, 1024, 0, "bvp"),
    (8, "generic_smem", 1, 1024, 0, "b"),
    (16, "spmd", 2, 1024, 0, "b"),
    (32, "spmd", 4, 1024, 0, "b"),
    (2, "spmd", 2, 768, 4096, "v"),
]

# The headline: the best measured THREE-level configuration (simdlen >= 2; the
# metric is the 3-level mapping's GB/s): simdlen 2, SPMD, blocked teams of 1024,
# quads of nonzeros (one 128-bit colind + one 256-bit val load per lane).  The
# 2-level comparison point is the best simdlen-1 candidate.
HEADLINE = (2, "spmd", 1, 1024, 0, "bqp")
SIMDLEN1 = [c for c in CANDIDATES if c[0] == 1]
# configs[4] (16 nnz/row): wider groups pay (DESIGN.md Fig 9 analogue / cfg5 table)
HEADLINE_CFG5 = (8, "spmd", 1, 1024, 0, "bv")
# the local SpMV of a rank's configs[4] shard at N > 1: fastest per shard size on one B200
# (profiles/r02s3/shard_configs.txt: S = 8 quads at N = 2, S = 4 quads from N = 4 on)
SHARD_HEADLINE = {2: (8, "spmd", 1, 1024, 0, "bq")}
SHARD_HEADLINE_DEFAULT = (4, "spmd", 1, 1024, 0, "bq")


def cfg_of(c):
    S, mode, U, T, halo, fl = c
    return dict(simdlen=S, mode=mode, outer_unroll=U, threads_per_team=T, x_halo=halo,
                stream_hints="h" in fl, blocked="b" in fl, vec128="v" in fl or "q" in fl, quad="q" in fl,
                x_l2_persist="p" in fl)


def cfg_key(spec, c) -> str:
    return f"{spec.name}:{json.dumps(list(c))}"


def kernel_name(c) -> str:
    S, mode, U, T, halo, fl = c
    if halo:
        return f"spmv_ring_kernel<S={S},{mode},SUM,SpmvVecBody<0,2,int,XRing>>" if "v" in fl else \
            f"spmv_ring_kernel<S={S},{mode},SUM,SpmvBody<0,int,XRing>>"
    body = ("SpmvVecBody<0,4,int>" if "q" in fl else "SpmvVecBody<0,2,int>" if "v" in fl
            else f"SpmvBody<{int('h' in fl)},int>")
    two_pm = ("v" in fl or "q" in fl) and U == 1 and not ("q" in fl and S == 1)
    name = f"{'nest_kernel_2pm' if two_pm else 'nest_kernel'}<S={S},{mode},SUM,U={U},{body}>"
    return name + (" + x persisting-L2 window" if "p" in fl else "")


def time_steps(torch, fn, flush, P, iters):
    """Per-step CUDA-event times (ms) on the current stream (the launching
    stream), L2 flushed (and left clean) before every step, outside the events."""
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


def roofline(B, ms, peak, peak_src, c, spec):
    achieved = B / (ms / 1e3) / 1e9
    traffic = traffic_of(cfg_key(spec, c))
    return {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
            "traffic": traffic, "peak_source": peak_src,
            "traffic_source": "profiles/traffic.json: ncu --set full dram__bytes_read.sum + dram__bytes_write.sum "
                              "per launch (cold L2)",
            "traffic_over_alg_bytes": (traffic / B) if traffic else None,
            **({"traffic_note": "ncu neutralises the persisting-L2 window (profiles/r02s3_x_l2_persist.md): this is "
                                "the kernel's DRAM traffic WITHOUT x persisting; with it the kernel runs 5-7% faster"}
               if "p" in c[5] else {}),
            "alg_bytes_per_launch": B,
            "alg_bytes_rule": "12 B per nonzero + 16 B per row (rowptr, y) + 8 B per column (x once)",
            "kernel": kernel_name(c), "frac_of_8TBs_spec": achieved / 8000.0}


def gen_to_device(torch, spec, dev, row_begin=0, nrows=None, chunk=10_000_000, with_oracle=False, x=None,
                  threads=None):
    """The CSR rows [row_begin, row_begin + nrows) of spec straight into device
    memory, generated in row chunks (bounded host memory); rowptr is 0-based for
    the block.  with_oracle: also the oracle's (y, abs) of every row (x given),
    computed chunk by chunk as it is generated (threaded oracle, bit-identical)."""
    import oracle
    n = spec.nrows - row_begin if nrows is None else nrows
    bounds, total = [], 0
    for r0 in range(0, n, chunk):
        m = min(chunk, n - r0)
        rp = R.spmv_matrix(spec, row_begin=row_begin + r0, nrows=m)[0]   # row lengths only
        bounds.append((r0, m, total))
        total += int(rp[-1])
    drp = torch.empty(n + 1, dtype=torch.int64, device=dev)
    dcol = torch.empty(total, dtype=torch.int32, device=dev)
    dval = torch.empty(total, dtype=torch.float64, device=dev)
    yref = np.empty(n) if with_oracle else None
    aref = np.empty(n) if with_oracle else None
    for r0, m, z0 in bounds:
        rp, col, val = R.spmv_matrix(spec, row_begin=row_begin + r0, nrows=m)
        if with_oracle:
            yref[r0:r0 + m], aref[r0:r0 + m], _ = oracle.spmv_csr_f64_threads(rp, col, val, x, threads or
                                                                              (os.cpu_count() or 1))
        drp[r0:r0 + m + 1] = torch.from_numpy(rp + z0)
        dcol[z0:z0 + col.size] = torch.from_numpy(col)
        dval[z0:z0 + val.size] = torch.from_numpy(val)
    return drp, dcol, dval, total, yref, aref


def parity(y, yref, aref):
    """R3 on every row: |y - ref| <= 1e-12 * sum|terms|, +0.0 where sum|terms| == 0."""
    y = np.asarray(y, np.float64)
    zero = aref == 0
    err = np.abs(y - yref)
    rel = np.where(zero, np.where((y == 0) & ~np.signbit(y), 0.0, np.inf), err / np.where(zero, 1.0, aref))
    worst = float(rel.max()) if rel.size else 0.0
    return {"rows_checked": int(y.size), "rows_total": int(y.size), "tol": 1e-12, "worst_rel_to_abs": worst,
            "ok": bool(worst <= 1e-12)}


def time_leg(torch, P, spec, c, t, y, flush, iters):
    fn = lambda: P.spmv_csr_f64(*t, y, **cfg_of(c))
    fn()
    ts = time_steps(torch, fn, flush, P, iters)
    return sum(ts) / len(ts)


def run_gpu_single(args, local_rank):
    import torch

    import oracle
    import paper_conf_icpp_wrightdtcc23_b200 as P

    torch.cuda.set_device(local_rank)
    dev = torch.device("cuda", local_rank)
    spec = SPEC
    peak, peak_src = peaks()
    flush = torch.empty(FLUSH_BYTES, dtype=torch.uint8, device=dev)
    rp, col, val = R.spmv_matrix(spec)
    x = R.spmv_x(spec)
    nnz = int(val.size)
    pin = lambda a: torch.from_numpy(a).pin_memory()
    h_rp, h_col, h_val, h_x = pin(rp), pin(col), pin(val), pin(x)
    t = [h_rp.to(dev), h_col.to(dev), h_val.to(dev), h_x.to(dev)]
    d_y = torch.empty(spec.nrows, dtype=torch.float64, device=dev)
    B = alg_bytes(spec.nrows, spec.ncols, nnz)

    # untimed sweep over the candidate (simdlen, mode, variant) set
    sweep = []
    for c in CANDIDATES:
        try:
            ms_c = time_leg(torch, P, spec, c, t, d_y, flush, 5)
        except P.NestError as e:
            print(f"skip {c}: {e}", file=sys.stderr)
            continue
        sweep.append((ms_c, c))
    sweep.sort(key=lambda q: q[0])
    ran = {c for _, c in sweep}
    # the fixed headline, unless this device cannot run it (then the best 3-level candidate)
    best = HEADLINE if HEADLINE in ran and not args.autotune else \
        min((q for q in sweep if q[1][0] >= 2), key=lambda q: q[0])[1]
    s1 = min((q for q in sweep if q[1][0] == 1), key=lambda q: q[0])[1]
    cfg = cfg_of(best)
    step = lambda: P.spmv_csr_f64(*t, d_y, **cfg)

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
    # parity of the timed configuration: every row against the oracle
    yref, aref = oracle.spmv_csr_f64(rp, col, val, x)
    par = parity(d_y.cpu().numpy(), yref, aref)
    y_head = d_y.clone()
    # simd-folded two-level mapping (simdlen = 1), same protocol
    ms1 = time_leg(torch, P, spec, s1, t, d_y, flush, max(5, args.steps // 2))
    # the paper's own comparison (Fig 9): the LLVM-style TWO-level mapping -- teams
    # distribute in generic mode (extra team-main warp, block state machine) + parallel
    # for over a row's nonzeros on 32-thread blocks (NEXT-1)
    tg = []
    for nt in (0, 2368):
        c_tg = dict(simdlen=1, mode="teams_generic", threads_per_team=32, num_teams=nt)
        P.spmv_csr_f64(*t, d_y, **c_tg)
        tg.append((statistics.median(time_steps(torch, lambda: P.spmv_csr_f64(*t, d_y, **c_tg), flush, P, 5)),
                   nt))
    ms_tg, nt_tg = min(tg)
    P.spmv_csr_f64(*t, d_y, simdlen=1, mode="teams_generic", threads_per_team=32, num_teams=nt_tg)
    par_tg = parity(d_y.cpu().numpy(), yref, aref)["ok"]

    # e2e through the C ABI with HOST buffers: H2D of A and x, the SpMV, D2H of y
    h_y = torch.empty(spec.nrows, dtype=torch.float64).pin_memory()
    ws = torch.empty(P.hostio_workspace_bytes(spec.nrows, spec.ncols, nnz), dtype=torch.uint8, device=dev)
    e2e_step = lambda: P.spmv_csr_f64_hostio(h_rp, h_col, h_val, h_x, h_y, ws, **cfg)
    e2e_step()
    torch.cuda.synchronize()
    te = []
    for _ in range(max(3, min(args.steps, 10))):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        e2e_step()
        e1.record()
        e1.synchronize()
        te.append(e0.elapsed_time(e1))
    ms_e2e = sum(te) / len(te)
    e2e_ok = bool(np.array_equal(h_y.numpy().view(np.int64), y_head.cpu().numpy().view(np.int64)))
    h2d = (spec.nrows + 1) * 8 + nnz * 12 + spec.ncols * 8
    d2h = spec.nrows * 8
    cpu = None if args.no_cpu_baseline else cpu_baseline(spec, rp, col, val, x)
    del t, ws, h_rp, h_col, h_val, h_x, h_y, rp, col, val, y_head
    torch.cuda.empty_cache()

    # ---- extra legs: the 100M-nnz gate matrix and configs[4] on one GPU
    legs = {}
    for lspec, heads, which in ((R.G100, [best, s1], "north_star 70% gate, SURVEY.md §8(d) G100"),
                                (R.CFG5, [HEADLINE_CFG5, s1], "configs[4] on one GPU")):
        lx = R.spmv_x(lspec)
        drp, dcol, dval, lnnz, lyref, laref = gen_to_device(torch, lspec, dev, with_oracle=True, x=lx)
        lt = [drp, dcol, dval, torch.from_numpy(lx).to(dev)]
        ly = torch.empty(lspec.nrows, dtype=torch.float64, device=dev)
        LB = alg_bytes(lspec.nrows, lspec.ncols, lnnz)
        leg = {"workload": workload(lspec, which), "nnz": lnnz, "alg_bytes": LB, "configs": {}}
        for c in heads:
            lms = time_leg(torch, P, lspec, c, lt, ly, flush, 10)
            leg["configs"][json.dumps(list(c))] = {"ms": lms, "GBs": LB / (lms / 1e3) / 1e9,
                                                   "gflops": 2 * lnnz / (lms / 1e3) / 1e9,
                                                   "roofline": roofline(LB, lms, peak, peak_src, c, lspec),
                                                   "parity": parity(ly.cpu().numpy(), lyref, laref)}
        h3 = leg["configs"][json.dumps(list(heads[0]))]
        if lspec is R.G100:
            # SURVEY.md §8(d) "warm-x" variant: L2 flushed, then x read once (a torch reduction,
            # outside the events) so the launch starts with as much of x in L2 as it holds
            cfg_h = cfg_of(heads[0])
            wts = []
            for _ in range(10):
                P.l2_flush(flush)
                lt[3].sum()
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record()
                P.spmv_csr_f64(*lt, ly, **cfg_h)
                e1.record()
                wts.append((e0, e1))
            torch.cuda.synchronize()
            wms = statistics.median(a.elapsed_time(b) for a, b in wts)
            h3["warm_x"] = {"ms": wms, "GBs": LB / (wms / 1e3) / 1e9,
                            "note": "x read into L2 (outside the events) after the flush; not a bench value"}
        leg["headline"] = heads[0]
        leg["speedup_vs_simdlen1"] = leg["configs"][json.dumps(list(s1))]["ms"] / h3["ms"]
        legs[lspec.name] = leg
        del lt, drp, dcol, dval, ly
        torch.cuda.empty_cache()

    line = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": 1, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms, "ms_median": statistics.median(ts), "ms_min": min(ts),
        "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": workload(spec), "nnz": nnz, "alg_bytes": B, "simdlen": best[0], "mode": best[1],
                   "outer_unroll": best[2], "threads_per_team": best[3], "x_halo": best[4],
                   "variant": " + ".join({"b": "blocked teams", "h": "stream hints", "v": "128-bit pair loads",
                                          "q": "128-bit quad loads", "p": "x persisting in L2 (access-policy window)"}[f]
                                         for f in best[5]) or "cyclic teams",
                   "l2": "flushed between timed steps (512 MiB write, then a 256 MiB read so L2 holds only clean "
                         "lines)",
                   "parallelism": "1 GPU"},
        "parity": par,
        "gflops": 2 * nnz / (ms / 1e3) / 1e9,
        "gflops_rule": "2 flops (multiply + add) per nonzero",
        "paper_comparison": {"baseline": "teams-generic two-level mapping (teams distribute generic + parallel for, "
                                         "32-thread blocks; NEXT-1, PAPER.md:886-889)",
                             "baseline_ms": ms_tg, "baseline_GBs": B / (ms_tg / 1e3) / 1e9,
                             "baseline_num_teams": nt_tg, "baseline_parity_ok": par_tg,
                             "speedup_of_headline": ms_tg / ms,
                             "paper_reported": "up to 3.5x (simdlen 8) for sparse_matvec on one A100 40 GB "
                                               "(PAPER.md:811-817, 922-928): context, not the target"},
        "speedup_vs_simdlen1": ms1 / ms,
        "simdlen1": {"ms_per_step": ms1, "GBs": B / (ms1 / 1e3) / 1e9, "config": cfg_of(s1)},
        "sweep_ms": {json.dumps(list(c)): round(m, 4) for m, c in sweep},
        "roofline": roofline(B, ms, peak, peak_src, best, spec),
        "legs": legs,
        "e2e": {"value": B / (ms_e2e / 1e3) / 1e9, "unit": UNIT, "h2d_bytes_per_step": h2d,
                "d2h_bytes_per_step": d2h, "ms_per_step": ms_e2e, "h2d_gbs": h2d / (ms_e2e / 1e3) / 1e9,
                "bitwise_equal_device_call": e2e_ok,
                "pipeline": f"{min(32, max(1, -(-nnz // (8 << 20))))} row chunks of ~8 Mi nonzeros: chunk c's "
                            "SpMV and y copy overlap the H2D of chunks > c (nest_spmv_csr_f64_hostio)"},
        "gpu_launches": 3 * args.steps,
        "gpu_launches_detail": "per step: 1 SpMV kernel + 2 l2 flush kernels (write, clean-read; outside the "
                               "step events)",
        "clocks": clk.summary(),
    }
    if cpu is not None:
        line["cpu_baseline"] = cpu
    print(json.dumps(line), flush=True)


def run_gpu_multi(args, rank, world, local_rank):
    """configs[4] row-partitioned over the ranks at fixed total size."""
    import torch
    import torch.distributed as dist

    import paper_conf_icpp_wrightdtcc23_b200 as P

    torch.cuda.set_device(local_rank)
    dev = torch.device("cuda", local_rank)
    spec = SPEC_MULTI
    peak, peak_src = peaks()
    flush = torch.empty(FLUSH_BYTES, dtype=torch.uint8, device=dev)
    chunk, rb, nloc = P.shard_rows(spec.nrows, world, rank)
    xb, xn = P.local_x_range(spec.ncols, world, rank)
    xc = P.x_chunk(spec.ncols, world)
    x_full_host = R.spmv_x(spec)                      # the oracle reads global columns
    h_xl = torch.zeros(xc, dtype=torch.float64).pin_memory()
    h_xl[:xn] = torch.from_numpy(x_full_host[xb:xb + xn])
    d_xl = h_xl.to(dev)
    threads = max(1, (os.cpu_count() or 1) // world)
    drp, dcol, dval, nnz, yref, aref = gen_to_device(torch, spec, dev, row_begin=rb, nrows=nloc, with_oracle=True,
                                                     x=x_full_host, threads=threads)
    d_y = torch.empty(nloc, dtype=torch.float64, device=dev)
    nnz_t = torch.tensor([nnz], dtype=torch.int64, device=dev if not SHARE_GPU else "cpu")
    dist.all_reduce(nnz_t)
    B = alg_bytes(spec.nrows, spec.ncols, int(nnz_t.item()))
    B_local = nnz * 12 + (nloc + 1) * 8 + nloc * 8 + spec.ncols * 8
    local_c = SHARD_HEADLINE.get(world, SHARD_HEADLINE_DEFAULT)
    cfg = cfg_of(local_c)

    def maxr(v):
        tt = torch.tensor([v], dtype=torch.float64, device=dev if not SHARE_GPU else "cpu")
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        return float(tt.item())

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
        return maxr(sum(ts) / len(ts)), clk.summary()   # max over ranks

    res, checks = {}, {}
    comm = None
    if not SHARE_GPU:   # NCCL needs one GPU per rank
        comm = P.Comm()
        d_xf = torch.empty(xc * world, dtype=torch.float64, device=dev)
        res["step_allgather_spmv"] = timed(lambda: comm.spmv_csr_f64(spec.nrows, spec.ncols, drp, dcol, dval, d_xl,
                                                                     d_xf, d_y, **cfg), args.steps)
        checks["allgather"] = parity(d_y.cpu().numpy(), yref, aref)
        res["allgather_alone"] = timed(lambda: comm.allgather_x(d_xl, d_xf, spec.ncols), args.steps)
        res["local_spmv_alone"] = timed(lambda: P.spmv_csr_f64(drp, dcol, dval, d_xf, d_y, ncols=spec.ncols,
                                                               **cfg), args.steps)
    xp_err = None
    cfg_xp = dict(cfg, quad=False)   # the peer-gather kernel takes scalar or pair loads
    try:
        xp = P.XPeer(spec.ncols)
        xp.set_local_x(d_xl)
        res["step_peer_gather"] = timed(lambda: xp.spmv_csr_f64(spec.nrows, drp, dcol, dval, d_y, **cfg_xp),
                                        args.steps)
        checks["peer_gather"] = parity(d_y.cpu().numpy(), yref, aref)
    except Exception as e:   # an optional leg must not take the bench down
        xp, xp_err = None, repr(e)
    # NEXT-4b: x as one virtual range over every rank's slice (CUDA virtual memory, file
    # descriptors over a unix socket): the plain kernel on a contiguous x, remote columns
    # read over NVLink; x written once (the timed step is the SpMV alone)
    xsym_err = None
    try:
        xsym = P.XSym(spec.ncols, tag=f"bench{os.getppid()}")
        lo = rank * xsym.xchunk
        if lo < spec.ncols:
            xsym.set_x(torch.from_numpy(x_full_host[lo:lo + xsym.xchunk].copy()).to(dev))
        torch.cuda.synchronize()
        dist.barrier()
        res["step_symmetric_x"] = timed(lambda: xsym.spmv_csr_f64(drp, dcol, dval, d_y, **cfg), args.steps)
        checks["symmetric_x"] = parity(d_y.cpu().numpy(), yref, aref)
    except Exception as e:   # an optional leg must not take the bench down
        xsym, xsym_err = None, repr(e)
    head = next(k for k in ("step_allgather_spmv", "step_symmetric_x", "step_peer_gather") if k in res)
    ms, clocks = res[head]
    worst = maxr(max(c["worst_rel_to_abs"] for c in checks.values()))

    # e2e through the public API with HOST buffers: the shard and x slice cross PCIe,
    # all-gather + local SpMV, y_local back (a12 hostio entry point)
    e2e = None
    if comm is not None:
        cpu = lambda a: a.cpu().pin_memory()
        h_rp, h_col, h_val, h_y = cpu(drp), cpu(dcol), cpu(dval), torch.empty(nloc, dtype=torch.float64).pin_memory()
        ws = torch.empty(comm.hostio_workspace_bytes(nloc, nnz, spec.ncols), dtype=torch.uint8, device=dev)
        del drp, dcol, dval
        torch.cuda.empty_cache()
        ms_e2e, _ = timed(lambda: comm.spmv_csr_f64_hostio(spec.nrows, spec.ncols, h_rp, h_col, h_val, h_xl, h_y,
                                                            ws, **cfg), max(3, min(args.steps, 5)))
        e2e = {"value": B / (ms_e2e / 1e3) / 1e9, "unit": UNIT, "ms_per_step": ms_e2e,
               "h2d_bytes_per_step": (nloc + 1) * 8 + nnz * 12 + xc * 8, "d2h_bytes_per_step": nloc * 8,
               "note": "per rank; nest_spmv_csr_f64_dist_hostio, max over ranks"}
    if rank == 0:
        ag_bytes = (world - 1) * xc * 8
        line = {"metric": METRIC, "value": B / (ms / 1e3) / 1e9, "unit": UNIT, "n_gpus": world,
                "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True,
                "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
                "config": {"workload": workload(spec, "configs[4], row-partitioned at fixed total size"),
                           "alg_bytes": B, "parallelism": f"rows/{world}", "x_exchange": head,
                           "l2": "flushed between timed steps", **cfg},
                "gflops": 2 * int(nnz_t.item()) / (ms / 1e3) / 1e9,
                "parts_ms": {k: v[0] for k, v in res.items()},
                "local_spmv_GBs_per_gpu": (B_local / (res["local_spmv_alone"][0] / 1e3) / 1e9
                                           if "local_spmv_alone" in res else None),
                "allgather_busbw_GBs": (ag_bytes / (res["allgather_alone"][0] / 1e3) / 1e9
                                        if "allgather_alone" in res else None),
                "parity": {"rows_checked": spec.nrows, "worst_rel_to_abs_over_ranks": worst,
                           "ok": bool(worst <= 1e-12), "per_variant_rank0": checks},
                "xpeer_error": xp_err, "xsym_error": xsym_err,
                "gpu_launches": args.steps * (5 if head == "step_peer_gather" else 3),
                "gpu_launches_detail": {"step_allgather_spmv": "per step: NCCL all-gather (NCCL's kernel) + our SpMV "
                                                               "kernel + 2 l2_flush kernels (outside the events)",
                                        "step_symmetric_x": "per step: the SpMV kernel on the symmetric x + 2 l2_flush",
                                        "step_peer_gather": "per step: barrier + SpMV + barrier + 2 l2_flush"}[head],
                "clocks": clocks, "e2e": e2e}
        per_gpu = line["value"] / world
        line["roofline"] = {"bound": "hbm", "achieved": per_gpu, "peak": peak, "unit": "GB/s",
                            "frac": per_gpu / peak, "traffic": None, "peak_source": peak_src,
                            "kernel": kernel_name(local_c),
                            "note": "per GPU: algorithmic bytes of all ranks / world / max-over-ranks step time"}
        if not args.no_cpu_baseline:
            line["cpu_baseline"] = cpu_sample_multi(spec)
        print(json.dumps(line), flush=True)
    if xp is not None:
        xp.close()
    if xsym is not None:
        xsym.close()
    if comm is not None:
        comm.close()


def cpu_sample_multi(spec):
    """N > 1: the oracle (1 thread) on a bounded sample of configs[4]: its first
    5M rows (about 80M nonzeros), repeated for ~10 s."""
    import oracle
    n = 5_000_000
    rp, col, val = R.spmv_matrix(spec, row_begin=0, nrows=n)
    x = R.spmv_x(spec)
    Bs = val.size * 12 + (n + 1) * 8 + n * 8 + spec.ncols * 8
    passes, t_total = 0, 0.0
    while t_total < 10.0:
        t0 = time.perf_counter()
        oracle.spmv_csr_f64(rp, col, val, x)
        t_total += time.perf_counter() - t0
        passes += 1
    return {"value": Bs * passes / t_total / 1e9, "unit": UNIT, "cores": 1, "kind": "oracle",
            "sample": f"{passes} passes over rows [0, {n}) of {spec.name} ({val.size} nnz), single-threaded C",
            "host": host_cpu()}


# Developer check of the N > 1 code path on a one-GPU box: every rank on cuda:0,
# gloo process group, the NCCL legs skipped (timings are meaningless).
SHARE_GPU = os.environ.get("NEST_BENCH_SHARE_GPU") == "1"


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=50)
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
            # NCCL's communicator lines (one per rank, for the torch group and for
            # libnest's own communicator) go to stderr, so the rank count is visible
            os.environ.setdefault("NCCL_DEBUG", "INFO")
            os.environ.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
        if backend == "nccl":
            import torch
            torch.cuda.set_device(local_rank)
        dist.init_process_group(backend)
    try:
        if args.impl == "reference":
            run_reference(args, rank, world)
        elif world == 1:
            run_gpu_single(args, local_rank)
        else:
            run_gpu_multi(args, rank, world, local_rank)
    finally:
        if world > 1:
            import torch.distributed as dist
            dist.destroy_process_group()


if __name__ == "__main__":
    main()
