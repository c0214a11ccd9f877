"""CPU-side checks of the C ABI: the library loads, exports every symbol
include/nest.h declares, and the host planner (a1) validates descriptors and
computes the geometry the oracle's plain definition gives.  No compute calls
(there is no GPU here)."""
import ctypes
import os
import re

import pytest

import oracle

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
P = pytest.importorskip("paper_conf_icpp_wrightdtcc23_b200")
from paper_conf_icpp_wrightdtcc23_b200 import _nest as N  # noqa: E402


def header_symbols():
    with open(os.path.join(ROOT, "include", "nest.h")) as f:
        text = f.read()
    text = re.sub(r"/\*.*?\*/", "", text, flags=re.S)
    return sorted(set(re.findall(r"\b(nest_[a-z0-9_]+)\s*\(", text)))


def test_every_header_symbol_is_exported_and_bound():
    syms = header_symbols()
    assert len(syms) >= 15
    for s in syms:
        assert hasattr(N.lib, s), s
        assert s in N.SIGNATURES, f"binding lacks {s}"
    assert set(N.SIGNATURES) == set(syms)


def test_abi_version_and_status_strings():
    assert N.nest_abi_version() == N.NEST_ABI_VERSION == 1
    assert N.nest_status_str(0) == b"NEST_OK"
    assert N.nest_status_str(2) == b"NEST_ERR_UNSUPPORTED"


SIMDLENS = (1, 2, 4, 8, 16, 32)


@pytest.mark.parametrize("T", [32, 128, 256, 512, 1024])
@pytest.mark.parametrize("S", SIMDLENS)
@pytest.mark.parametrize("payload", [0, 24, 32, 200])
def test_plan_matches_oracle_geometry(T, S, payload):
    ref = oracle.plan_geometry(T, S, 2048, payload)
    info = P.plan(1 << 20, payload, simdlen=S, threads_per_team=T, mode="generic_smem", num_teams=7)
    assert (info["groups_per_team"], info["slot_bytes"]) == ref[:2]
    # S == 1 runs SPMD: no sharing space, never a fallback
    assert info["uses_global_fallback"] == (ref[2] if S > 1 else 0)
    assert info["grid"] == 7 and info["block"] == T
    assert info["smem_bytes"] == (2048 if S > 1 else 0)


def test_plan_auto_grid_one_pass():
    # one outer iteration per group per pass: grid = ceil(outer / (G*U))
    for S, U, outer in ((8, 1, 1000), (8, 2, 1000), (1, 4, 10_000_001), (32, 1, 5)):
        G = 256 // S
        info = P.plan(outer, 24, simdlen=S, outer_unroll=U)
        assert info["grid"] == -(-outer // (G * U))
        assert info["smem_bytes"] == 0 and info["uses_global_fallback"] == 0


@pytest.mark.parametrize("cfg", [dict(simdlen=3), dict(simdlen=64), dict(simdlen=0),
                                 dict(threads_per_team=48), dict(threads_per_team=2048),
                                 dict(mode=3), dict(reduce=7), dict(sharing_bytes=-1),
                                 dict(sharing_bytes=1 << 20), dict(outer_unroll=3),
                                 dict(num_teams=-1), dict(flags=1 << 9)])
def test_plan_rejects_invalid(cfg):
    with pytest.raises(P.NestError) as e:
        P.plan(100, 24, **cfg)
    assert e.value.status == N.NEST_ERR_INVALID_ARG


def test_plan_rejects_bad_abi_version_and_reserved():
    d = P.make_desc()
    d.abi_version = 99
    info = N.nest_plan_info()
    assert N.nest_plan(ctypes.byref(d), 10, 0, ctypes.byref(info)) == N.NEST_ERR_INVALID_ARG
    d = P.make_desc()
    d.reserved = 5
    assert N.nest_plan(ctypes.byref(d), 10, 0, ctypes.byref(info)) == N.NEST_ERR_INVALID_ARG
    assert b"reserved" in N.nest_last_error()


def test_invalid_args_rejected_before_any_launch():
    d = P.make_desc()
    # negative extents / NULL pointers: validated on the host, no device touched
    assert N.nest_spmv_csr_f64(ctypes.byref(d), -1, 4, 4, None, None, None, None, None, None) == 1
    assert N.nest_spmv_csr_f64(ctypes.byref(d), 4, 4, 4, None, None, None, None, None, None) == 1
    assert N.nest_spmv_csr_f64(ctypes.byref(d), 0, 4, 0, None, None, None, None, None, None) == 0
    assert N.nest_batched_matvec_f32(ctypes.byref(d), 0, 64, 64, None, None, None, None) == 0
    assert N.nest_nested_stencil_f64(ctypes.byref(d), 0, 8, None, None, None, None, None, None) == 0
    assert N.nest_nested_stencil_f64(ctypes.byref(d), -2, 8, None, None, None, None, None, None) == 1
    bad = P.make_desc(simdlen=5)
    assert N.nest_batched_matvec_f32(ctypes.byref(bad), 1, 64, 64, None, None, None, None) == 1


def test_shard_rows_matches_oracle():
    for n, Pn in ((0, 1), (7, 8), (1024, 3), (100_000_000, 8)):
        for r in range(Pn):
            assert P.shard_rows(n, Pn, r) == oracle.shard_rows(n, Pn, r)


def test_teams_generic_mode_rules():
    # the two-level teams-generic baseline: SpMV only, simdlen 1
    with pytest.raises(P.NestError):
        P.plan(100, 24, simdlen=2, mode="teams_generic")
    d = P.make_desc(simdlen=1, mode="teams_generic")
    assert N.nest_batched_matvec_f32(ctypes.byref(d), 1, 64, 64, None, None, None, None) == N.NEST_ERR_INVALID_ARG


def test_team_chunk_validation():
    # team_chunk needs the blocked schedule and is non-negative
    with pytest.raises(P.NestError) as e:
        P.plan(1000, 24, team_chunk=64)
    assert e.value.status == N.NEST_ERR_INVALID_ARG and "NEST_F_BLOCKED" in str(e.value)
    with pytest.raises(P.NestError) as e:
        P.plan(1000, 24, team_chunk=-1, blocked=True, num_teams=4)
    assert e.value.status == N.NEST_ERR_INVALID_ARG
    info = P.plan(1000, 24, team_chunk=100, blocked=True, num_teams=4)
    assert info["grid"] == 4


def test_region_program_validates_before_any_device_call():
    d = P.make_desc()
    regs = (N.nest_region * 5)()
    assert N.nest_region_program(ctypes.byref(d), regs, 0, None) == N.NEST_ERR_INVALID_ARG
    assert N.nest_region_program(ctypes.byref(d), regs, 5, None) == N.NEST_ERR_INVALID_ARG
    regs[0].kind, regs[0].simdlen = N.NEST_REGION_SPMV_CSR_F64, 3      # not a divisor of the warp
    assert N.nest_region_program(ctypes.byref(d), regs, 1, None) == N.NEST_ERR_INVALID_ARG
    regs[0].simdlen, regs[0].kind = 8, 7                                # unknown body
    assert N.nest_region_program(ctypes.byref(d), regs, 1, None) == N.NEST_ERR_INVALID_ARG
    regs[0].kind, regs[0].n[0] = N.NEST_REGION_SPMV_CSR_F64, 10         # rows but NULL arrays
    assert N.nest_region_program(ctypes.byref(d), regs, 1, None) == N.NEST_ERR_INVALID_ARG
    d.reduce = N.NEST_REDUCE_MAX
    assert N.nest_region_program(ctypes.byref(d), regs, 1, None) == N.NEST_ERR_UNSUPPORTED
