"""Torch-tensor wrappers over the C ABI (argument marshalling only).

Every step of the path runs in libnest.so's CUDA kernels; these functions only
check tensor dtypes/devices/sizes, build the ``nest_desc`` and translate a
non-OK status into ``NestError``.  PyTorch provides device memory and streams.
"""
from __future__ import annotations

import ctypes

from . import _nest as N

MODES = {"spmd": N.NEST_MODE_SPMD, "generic_smem": N.NEST_MODE_GENERIC_SMEM,
         "generic_shfl": N.NEST_MODE_GENERIC_SHFL, "teams_generic": N.NEST_MODE_TEAMS_GENERIC}
REDUCES = {"sum": N.NEST_REDUCE_SUM, "max": N.NEST_REDUCE_MAX, "min": N.NEST_REDUCE_MIN}
SIMDLENS = (1, 2, 4, 8, 16, 32)


class NestError(RuntimeError):
    def __init__(self, status: int, where: str):
        self.status = status
        msg = N.nest_last_error().decode(errors="replace")
        name = N.nest_status_str(status).decode()
        super().__init__(f"{where}: {name}: {msg}")


def check(status: int, where: str) -> None:
    if status != N.NEST_OK:
        raise NestError(status, where)


def make_desc(simdlen: int = 8, mode: str | int = "spmd", reduce: str | int = "sum",
              threads_per_team: int = 256, num_teams: int = 0, sharing_bytes: int = 0,
              outer_unroll: int = 1, persistent: bool = False, stream_hints: bool = False,
              x_halo: int = 0, blocked: bool = False,
              vec128: bool = False, quad: bool = False, team_chunk: int = 0, teams_per_sm: int = 0,
              x_l2_persist: bool = False, flags: int = 0) -> N.nest_desc:
    """A nest_desc (include/nest.h) from keyword arguments: the integer fields by name
    (simdlen, threads_per_team, num_teams, sharing_bytes, outer_unroll, x_halo,
    team_chunk, teams_per_sm), mode "spmd" / "generic_smem" / "generic_shfl" /
    "teams_generic", reduce "sum" / "max" / "min", and the flags: persistent ->
    NEST_F_PERSISTENT_GRID, stream_hints -> NEST_F_STREAM_HINTS, blocked -> NEST_F_BLOCKED,
    vec128 -> NEST_F_VEC128, quad -> NEST_F_VEC128 | NEST_F_VEC_QUAD, x_l2_persist ->
    NEST_F_X_L2_PERSIST (plus any raw bits in `flags`)."""
    d = N.nest_desc()
    d.abi_version = N.NEST_ABI_VERSION
    d.num_teams = num_teams
    d.threads_per_team = threads_per_team
    d.simdlen = simdlen
    d.mode = MODES[mode] if isinstance(mode, str) else int(mode)
    d.reduce = REDUCES[reduce] if isinstance(reduce, str) else int(reduce)
    d.sharing_bytes = sharing_bytes
    d.outer_unroll = outer_unroll
    d.x_halo = x_halo
    d.team_chunk = team_chunk
    d.teams_per_sm = teams_per_sm
    d.flags = flags | (N.NEST_F_PERSISTENT_GRID if persistent else 0) | (
        N.NEST_F_STREAM_HINTS if stream_hints else 0) | (
        N.NEST_F_BLOCKED if blocked else 0) | (N.NEST_F_VEC128 if vec128 or quad else 0) | (
        N.NEST_F_VEC_QUAD if quad else 0) | (N.NEST_F_X_L2_PERSIST if x_l2_persist else 0)
    return d


def plan(outer_iters: int, payload_bytes: int = 0, **cfg) -> dict:
    info = N.nest_plan_info()
    check(N.nest_plan(ctypes.byref(make_desc(**cfg)), outer_iters, payload_bytes,
                      ctypes.byref(info)), "nest_plan")
    return {f: getattr(info, f) for f, _ in N.nest_plan_info._fields_}


def spmv_plan(nrows: int, ncols: int, nnz: int, **cfg) -> dict:
    """a1 for a8: the plan nest_spmv_csr_f64 launches for this matrix shape."""
    info = N.nest_plan_info()
    check(N.nest_spmv_plan(ctypes.byref(make_desc(**cfg)), nrows, ncols, nnz, ctypes.byref(info)),
          "nest_spmv_plan")
    return {f: getattr(info, f) for f, _ in N.nest_plan_info._fields_}


def _torch():
    import torch
    return torch


def _stream(stream):
    torch = _torch()
    s = torch.cuda.current_stream() if stream is None else stream
    return ctypes.c_void_p(s.cuda_stream)


def _dev(t, dtype, n, name):
    torch = _torch()
    if not isinstance(t, torch.Tensor) or not t.is_cuda:
        raise TypeError(f"{name} must be a CUDA tensor")
    if t.dtype != dtype:
        raise TypeError(f"{name} must be {dtype}, got {t.dtype}")
    if not t.is_contiguous():
        raise ValueError(f"{name} must be contiguous")
    if n is not None and t.numel() < n:
        raise ValueError(f"{name} has {t.numel()} elements, needs {n}")
    return ctypes.c_void_p(t.data_ptr()) if t.numel() else None


def spmv_csr_f64(rowptr, colind, val, x, y=None, *, ncols=None, stream=None, **cfg):
    """a8: y = A x for CSR A (rowptr int64, colind int32, val f64), x f64."""
    torch = _torch()
    nrows = rowptr.numel() - 1
    ncols = x.numel() if ncols is None else ncols
    nnz = val.numel()
    if y is None:
        y = torch.empty(nrows, dtype=torch.float64, device=val.device)
    d = make_desc(**cfg)
    check(N.nest_spmv_csr_f64(ctypes.byref(d), nrows, ncols, nnz,
                              _dev(rowptr, torch.int64, nrows + 1, "rowptr"),
                              _dev(colind, torch.int32, nnz, "colind"),
                              _dev(val, torch.float64, nnz, "val"),
                              _dev(x, torch.float64, ncols, "x"),
                              _dev(y, torch.float64, nrows, "y"), _stream(stream)),
          "nest_spmv_csr_f64")
    return y


def hostio_workspace_bytes(nrows: int, ncols: int, nnz: int) -> int:
    return int(N.nest_spmv_hostio_workspace_bytes(nrows, ncols, nnz))


def spmv_csr_f64_hostio(h_rowptr, h_colind, h_val, h_x, h_y, workspace, *, stream=None, **cfg):
    """a8 end to end: HOST (pinned) tensors in and out, device workspace."""
    torch = _torch()
    nrows = h_rowptr.numel() - 1
    ncols, nnz = h_x.numel(), h_val.numel()
    for t, dt, name, n in ((h_rowptr, torch.int64, "h_rowptr", nrows + 1), (h_colind, torch.int32, "h_colind", nnz),
                           (h_val, torch.float64, "h_val", nnz), (h_x, torch.float64, "h_x", ncols),
                           (h_y, torch.float64, "h_y", nrows)):
        if t.is_cuda or t.dtype != dt or not t.is_contiguous():
            raise TypeError(f"{name} must be a contiguous host {dt} tensor")
        if t.numel() < n:   # the C side copies n elements from / into it
            raise ValueError(f"{name} has {t.numel()} elements, needs {n}")
    d = make_desc(**cfg)
    check(N.nest_spmv_csr_f64_hostio(ctypes.byref(d), nrows, ncols, nnz,
                                     ctypes.c_void_p(h_rowptr.data_ptr()),
                                     ctypes.c_void_p(h_colind.data_ptr()),
                                     ctypes.c_void_p(h_val.data_ptr()),
                                     ctypes.c_void_p(h_x.data_ptr()),
                                     ctypes.c_void_p(h_y.data_ptr()),
                                     _dev(workspace, torch.uint8, None, "workspace"),
                                     workspace.numel(), _stream(stream)),
          "nest_spmv_csr_f64_hostio")
    return h_y


def batched_matvec_f32(A, x, batch, m=64, n=64, y=None, *, stream=None, **cfg):
    """a9: y[b] = A[b] @ x[b] for batch small dense fp32 matrices."""
    torch = _torch()
    if y is None:
        y = torch.empty(batch * m, dtype=torch.float32, device=A.device)
    d = make_desc(**cfg)
    check(N.nest_batched_matvec_f32(ctypes.byref(d), batch, m, n,
                                    _dev(A, torch.float32, batch * m * n, "A"),
                                    _dev(x, torch.float32, batch * n, "x"),
                                    _dev(y, torch.float32, batch * m, "y"), _stream(stream)),
          "nest_batched_matvec_f32")
    return y


def nested_stencil_f64(inp, coef, w, nouter, L, out=None, visits=None, *, stream=None, **cfg):
    """a10: nested loop with a sequential, side-effecting prologue."""
    torch = _torch()
    if out is None:
        out = torch.empty(nouter, dtype=torch.float64, device=w.device)
    d = make_desc(**cfg)
    check(N.nest_nested_stencil_f64(ctypes.byref(d), nouter, L,
                                    _dev(inp, torch.float64, nouter * L + 2, "in"),
                                    _dev(coef, torch.float64, L, "coef"),
                                    _dev(w, torch.float64, nouter, "w"),
                                    _dev(out, torch.float64, nouter, "out"),
                                    None if visits is None else _dev(visits, torch.int64, 1, "visits"),
                                    _stream(stream)),
          "nest_nested_stencil_f64")
    return out


def laplace3d_f64(u, out, nz, ny, nx, alpha, *, stream=None, **cfg):
    """NEXT-2: one Jacobi heat-diffusion step on the interior (non-reducing simd loop)."""
    torch = _torch()
    d = make_desc(**cfg)
    n = nz * ny * nx
    check(N.nest_laplace3d_f64(ctypes.byref(d), nz, ny, nx, float(alpha), _dev(u, torch.float64, n, "u"),
                               _dev(out, torch.float64, n, "out"), _stream(stream)), "nest_laplace3d_f64")
    return out


def probe_mapping(num_teams, trip, *, with_map=True, stream=None, **cfg):
    """a2/a5/a6 probe: returns (map[grid*T,5], hits[trip], owner[trip], totals[grid*G])."""
    torch = _torch()
    T = cfg.get("threads_per_team", 256) or 256
    S = cfg.get("simdlen", 8)
    dev = torch.device("cuda", torch.cuda.current_device())
    mp = torch.full((num_teams * T, 5), -7, dtype=torch.int32, device=dev) if with_map else None
    hits = torch.zeros(max(trip, 0), dtype=torch.int32, device=dev)
    owner = torch.full((max(trip, 0),), -1, dtype=torch.int32, device=dev)
    totals = torch.full((num_teams * (T // S),), -1.0, dtype=torch.float64, device=dev)
    d = make_desc(num_teams=num_teams, **cfg)
    check(N.nest_probe_mapping(ctypes.byref(d), _dev(mp, torch.int32, None, "map") if mp is not None else None,
                               trip, _dev(hits, torch.int32, None, "hits"),
                               _dev(owner, torch.int32, None, "owner"),
                               _dev(totals, torch.float64, None, "totals"), _stream(stream)),
          "nest_probe_mapping")
    return mp, hits, owner, totals


def csr_validate(rowptr, colind, ncols, *, stream=None) -> int:
    """Device check of the CSR preconditions; returns the violation bits (syncs)."""
    torch = _torch()
    bad = torch.zeros(1, dtype=torch.int32, device=rowptr.device)
    nrows, nnz = rowptr.numel() - 1, colind.numel()
    check(N.nest_csr_validate(nrows, ncols, nnz, _dev(rowptr, torch.int64, nrows + 1, "rowptr"),
                              _dev(colind, torch.int32, nnz, "colind"),
                              _dev(bad, torch.int32, 1, "bad"), _stream(stream)), "nest_csr_validate")
    return int(bad.item())


def l2_flush(buf, *, stream=None) -> None:
    torch = _torch()
    check(N.nest_util_l2_flush(_dev(buf, torch.uint8, None, "buf"), buf.numel(), _stream(stream)),
          "nest_util_l2_flush")


def shutdown() -> None:
    check(N.nest_shutdown(), "nest_shutdown")


def region_program(regions, *, stream=None, **team_cfg):
    """NEXT-3: run up to NEST_MAX_REGIONS parallel regions, each with its own
    simdlen and mode, inside ONE kernel.

    ``regions``: dicts with ``kind`` in {"spmv", "batched", "stencil"},
    ``simdlen``, ``mode`` (default "spmd"), ``blocked`` (default False) and the
    kind's tensors -- spmv: rowptr, colind, val, x, y (ncols = x.numel());
    batched: A, x, y, batch, m, n; stencil: inp, coef, w, out, nouter, L, visits
    (optional).  ``team_cfg``: threads_per_team, num_teams, sharing_bytes."""
    torch = _torch()
    arr = (N.nest_region * len(regions))()
    for k, r in enumerate(regions):
        g = arr[k]
        g.simdlen = r["simdlen"]
        m = r.get("mode", "spmd")
        g.mode = MODES[m] if isinstance(m, str) else int(m)
        g.blocked = int(bool(r.get("blocked", False)))
        kind = r["kind"]
        if kind == "spmv":
            nrows, nnz = r["rowptr"].numel() - 1, r["val"].numel()
            ncols = r["x"].numel()
            g.kind = N.NEST_REGION_SPMV_CSR_F64
            g.n[:] = [nrows, ncols, nnz]
            g.in_[:] = [_dev(r["rowptr"], torch.int64, nrows + 1, "rowptr"), _dev(r["colind"], torch.int32, nnz, "colind"),
                        _dev(r["val"], torch.float64, nnz, "val"), _dev(r["x"], torch.float64, ncols, "x")]
            g.out[0] = _dev(r["y"], torch.float64, nrows, "y")
        elif kind == "batched":
            b, mm, n = r["batch"], r["m"], r["n"]
            g.kind = N.NEST_REGION_BATCHED_MATVEC_F32
            g.n[:] = [b, mm, n]
            g.in_[0] = _dev(r["A"], torch.float32, b * mm * n, "A")
            g.in_[1] = _dev(r["x"], torch.float32, b * n, "x")
            g.out[0] = _dev(r["y"], torch.float32, b * mm, "y")
        elif kind == "stencil":
            no, L = r["nouter"], r["L"]
            g.kind = N.NEST_REGION_NESTED_STENCIL_F64
            g.n[:] = [no, L, 0]
            g.in_[:] = [_dev(r["inp"], torch.float64, no * L + 2, "in"), _dev(r["coef"], torch.float64, L, "coef"),
                        _dev(r["w"], torch.float64, no, "w"), None]
            g.out[0] = _dev(r["out"], torch.float64, no, "out")
            v = r.get("visits")
            g.out[1] = _dev(v, torch.int64, 1, "visits") if v is not None else None
        else:
            raise ValueError(f"unknown region kind {kind!r}")
    d = make_desc(**team_cfg)
    check(N.nest_region_program(ctypes.byref(d), arr, len(regions), _stream(stream)), "nest_region_program")
