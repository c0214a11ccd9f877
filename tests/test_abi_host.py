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
    assert N.nest_abi_version() == N.NEST_ABI_VERSION == 2
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


def test_plan_rejects_bad_abi_version_and_teams_per_sm():
    d = P.make_desc()
    d.abi_version = 99
    info = N.nest_plan_info()
    assert N.nest_plan(ctypes.byref(d), 10, 0, ctypes.byref(info)) == N.NEST_ERR_INVALID_ARG
    d = P.make_desc()
    d.teams_per_sm = 1
    assert N.nest_plan(ctypes.byref(d), 10, 0, ctypes.byref(info)) == N.NEST_ERR_INVALID_ARG
    assert b"teams_per_sm" in N.nest_last_error()


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


# ---------------------------------------------------------------- nest_spmv_plan (a1 for a8)
# Generic payload = sizeof(Slot{int32 fn, int32 count, Loop}) of the body that RUNS
# (the plan used to report the 64-bit scalar body's 24 bytes for every
# variant).  Loop: scalar {I trip, I base}; 128-bit tuples {I base, int32 trip, int32 len}.
SLOT_HEADER = 8


def expected_payload(vec, bits):
    if vec:
        return SLOT_HEADER + (bits // 8) + 8 if bits == 32 else SLOT_HEADER + 16
    return SLOT_HEADER + 2 * (bits // 8)


@pytest.mark.parametrize("vec", [False, True])
@pytest.mark.parametrize("S", SIMDLENS)
@pytest.mark.parametrize("T", [64, 256, 1024])
@pytest.mark.parametrize("sharing", [0, 256, 2048, 8192])
def test_spmv_plan_payload_and_fallback_are_the_launched_bodys(vec, S, T, sharing):
    nrows, ncols = 10_000, 10_000
    for nnz, bits in ((80_000, 32), ((1 << 31) + 100, 64)):
        info = P.spmv_plan(nrows, ncols, nnz, simdlen=S, threads_per_team=T, mode="generic_smem",
                           sharing_bytes=sharing, num_teams=5, vec128=vec)
        assert info["kernel"] == N.NEST_KERNEL_NEST and info["index_bits"] == bits
        assert info["payload_bytes"] == expected_payload(vec, bits)
        G = T // S
        slot = ((sharing or 2048) // G) & ~7
        assert info["slot_bytes"] == slot
        # global fallback exactly when the payload exceeds the slot
        assert info["uses_global_fallback"] == (int(info["payload_bytes"] > slot) if S > 1 else 0)


def test_spmv_plan_fallback_flips_at_the_bodys_own_size():
    # S = 2, T = 256: G = 128; a 2048-byte space gives 16-byte slots.  The 32-bit
    # scalar body posts 16 bytes (fits); the 32-bit pair body 20 (global fallback).
    base = dict(simdlen=2, threads_per_team=256, mode="generic_smem", num_teams=3)
    assert P.spmv_plan(1000, 1000, 8000, **base)["uses_global_fallback"] == 0
    assert P.spmv_plan(1000, 1000, 8000, vec128=True, **base)["uses_global_fallback"] == 1
    # SPMD never uses the sharing space
    assert P.spmv_plan(1000, 1000, 8000, vec128=True, **dict(base, mode="spmd"))["uses_global_fallback"] == 0


@pytest.mark.parametrize("S", SIMDLENS)
@pytest.mark.parametrize("T,tps", [(64, 0), (256, 0), (768, 2), (1024, 1), (1024, 0)])
@pytest.mark.parametrize("U", [1, 2, 4])
def test_spmv_plan_x_ring_geometry(S, T, tps, U):
    H, nrows = 4096, 1_000_000
    G = (T - 32) // S                      # the last warp is the copy engine
    R = G * U
    span = -(-(R + 2 * H) // 256) + 1      # segments one round's window can touch
    cfg = dict(simdlen=S, threads_per_team=T, x_halo=H, outer_unroll=U, teams_per_sm=tps, num_teams=17,
               vec128=True)
    budget = (228 * 1024) // (tps or 1) - 1024
    stages = (T // 32 - 1) * 4 * ((U * (32 // S + 1) + 1) & ~1) * 8   # row-bound stages of the consumer warps
    if (span + 1) * 2064 + stages > budget:   # the forced team count cannot hold one round's window
        with pytest.raises(P.NestError) as e:
            P.spmv_plan(nrows, nrows, 8 * nrows, **cfg)
        assert e.value.status == N.NEST_ERR_UNSUPPORTED
        return
    info = P.spmv_plan(nrows, nrows, 8 * nrows, **cfg)
    assert info["kernel"] == N.NEST_KERNEL_XRING and info["groups_per_team"] == G
    assert info["ring_segments"] >= span + 1
    assert info["smem_bytes"] <= 227 * 1024
    assert info["ring_segments"] * 2048 <= info["smem_bytes"]
    assert info["grid"] == 17 and info["chunk"] == -(-nrows // 17)
    assert info["payload_bytes"] == expected_payload(True, 32)


def test_spmv_plan_x_ring_rejections():
    with pytest.raises(P.NestError) as e:    # one warp: no consumer beside the copy warp
        P.spmv_plan(1000, 1000, 8000, x_halo=100, threads_per_team=32, num_teams=1)
    assert e.value.status == N.NEST_ERR_INVALID_ARG
    with pytest.raises(P.NestError) as e:    # the window cannot fit shared memory
        P.spmv_plan(1000, 1000, 8000, x_halo=200_000, num_teams=1)
    assert e.value.status == N.NEST_ERR_UNSUPPORTED
    with pytest.raises(P.NestError) as e:    # teams_per_sm only with the ring
        P.spmv_plan(1000, 1000, 8000, teams_per_sm=2, num_teams=1)
    assert e.value.status == N.NEST_ERR_INVALID_ARG
    with pytest.raises(P.NestError) as e:    # two teams per SM need T <= 768 (registers)
        P.spmv_plan(1000, 1000, 8000, x_halo=100, teams_per_sm=2, threads_per_team=1024, num_teams=1)
    assert e.value.status == N.NEST_ERR_UNSUPPORTED
    with pytest.raises(P.NestError) as e:    # the removed staged-pipeline bit is an unknown flag
        P.spmv_plan(1000, 1000, 8000, flags=1 << 2, num_teams=1)
    assert e.value.status == N.NEST_ERR_INVALID_ARG


def test_spmv_plan_index_width_covers_the_cyclic_schedule():
    """32-bit cursors only when grid * G (the cyclic schedule's group
    ids and stride) also stays below 2^30 -- a caller-set league of 3M teams of
    1024 lanes at simdlen 1 would overflow them."""
    small = P.spmv_plan(1000, 1000, 8000, simdlen=1, threads_per_team=1024, num_teams=100)
    assert small["index_bits"] == 32
    big = P.spmv_plan(1000, 1000, 8000, simdlen=1, threads_per_team=1024, num_teams=3_000_000)
    assert big["index_bits"] == 64


def test_x_l2_persist_flag_rules():
    # NEST_F_X_L2_PERSIST: CSR SpMV only (nest_kernel variants); rejected before any device call
    with pytest.raises(P.NestError) as e:
        P.plan(1000, 24, x_l2_persist=True)
    assert e.value.status == N.NEST_ERR_INVALID_ARG and "SpMV" in str(e.value)
    d = P.make_desc(x_l2_persist=True)
    assert N.nest_batched_matvec_f32(ctypes.byref(d), 1, 64, 64, None, None, None, None) == N.NEST_ERR_INVALID_ARG
    assert N.nest_nested_stencil_f64(ctypes.byref(d), 1, 4, None, None, None, None, None, None) == \
        N.NEST_ERR_INVALID_ARG
    with pytest.raises(P.NestError) as e:   # the two-level teams-generic baseline: unsupported
        P.spmv_plan(1000, 1000, 8000, simdlen=1, mode="teams_generic", x_l2_persist=True)
    assert e.value.status == N.NEST_ERR_UNSUPPORTED
    assert N.NEST_F_X_L2_PERSIST == 1 << 6
    with open(os.path.join(ROOT, "include", "nest.h")) as f:
        assert "NEST_F_X_L2_PERSIST = 1u << 6" in f.read()


def test_c_example_builds_against_the_header_and_library():
    # the boundary is a C ABI: a plain C program (examples/spmv_c.c) compiles against
    # include/nest.h and links libnest.so with gcc alone (tests/test_gpu_parity.py runs it)
    import subprocess
    r = subprocess.run(["make", "-C", ROOT, "examples/spmv_c"], capture_output=True, text=True)
    assert r.returncode == 0, r.stdout + r.stderr
    exe = os.path.join(ROOT, "examples", "spmv_c")
    assert os.access(exe, os.X_OK)
    ldd = subprocess.run(["ldd", exe], capture_output=True, text=True).stdout
    assert "libnest.so" in ldd and "not found" not in ldd, ldd
