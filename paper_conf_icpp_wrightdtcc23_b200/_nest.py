"""ctypes binding of libnest.so (include/nest.h), argument marshalling only.

Every C entry point is exposed under its own name (``nest_spmv_csr_f64`` ...)
with its C signature; the friendlier wrappers in ``api.py`` accept torch
tensors and turn a non-OK status into ``NestError``.  There is no fallback:
if libnest.so is missing or fails to load, importing this module raises.
"""
from __future__ import annotations

import ctypes
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libnest.so")

if not os.path.exists(LIB_PATH):
    raise ImportError(f"{LIB_PATH} is missing: build it with `make -C {os.path.dirname(_HERE)}` "
                      "(there is no CPU fallback)")
lib = ctypes.CDLL(LIB_PATH)

NEST_ABI_VERSION = 2
NEST_OK, NEST_ERR_INVALID_ARG, NEST_ERR_UNSUPPORTED, NEST_ERR_CUDA, NEST_ERR_NCCL, NEST_ERR_NO_MEMORY = range(6)
NEST_MODE_SPMD, NEST_MODE_GENERIC_SMEM, NEST_MODE_GENERIC_SHFL, NEST_MODE_TEAMS_GENERIC = 0, 1, 2, 3
NEST_REDUCE_SUM, NEST_REDUCE_MAX, NEST_REDUCE_MIN = 0, 1, 2
NEST_F_PERSISTENT_GRID = 1 << 0
NEST_F_STREAM_HINTS = 1 << 1
NEST_F_BLOCKED = 1 << 3
NEST_F_VEC128 = 1 << 4
NEST_F_VEC_QUAD = 1 << 5
NEST_F_X_L2_PERSIST = 1 << 6
NEST_KERNEL_NEST, NEST_KERNEL_XRING, NEST_KERNEL_TEAMS_GENERIC = 0, 1, 2


class nest_desc(ctypes.Structure):
    _fields_ = [("abi_version", ctypes.c_uint32), ("num_teams", ctypes.c_int32),
                ("threads_per_team", ctypes.c_int32), ("simdlen", ctypes.c_int32),
                ("mode", ctypes.c_int32), ("reduce", ctypes.c_int32),
                ("sharing_bytes", ctypes.c_int32), ("flags", ctypes.c_uint32),
                ("outer_unroll", ctypes.c_int32), ("x_halo", ctypes.c_int32),
                ("team_chunk", ctypes.c_int32), ("teams_per_sm", ctypes.c_int32)]


NEST_MAX_REGIONS = 4
NEST_REGION_SPMV_CSR_F64, NEST_REGION_BATCHED_MATVEC_F32, NEST_REGION_NESTED_STENCIL_F64 = 0, 1, 2


class nest_region(ctypes.Structure):
    _fields_ = [("kind", ctypes.c_int32), ("simdlen", ctypes.c_int32), ("mode", ctypes.c_int32),
                ("blocked", ctypes.c_int32), ("n", ctypes.c_int64 * 3), ("in_", ctypes.c_void_p * 4),
                ("out", ctypes.c_void_p * 2)]


class nest_plan_info(ctypes.Structure):
    _fields_ = [("grid", ctypes.c_int32), ("block", ctypes.c_int32),
                ("groups_per_team", ctypes.c_int32), ("slot_bytes", ctypes.c_int32),
                ("payload_bytes", ctypes.c_int32), ("uses_global_fallback", ctypes.c_int32),
                ("outer_unroll", ctypes.c_int32), ("smem_bytes", ctypes.c_int32),
                ("kernel", ctypes.c_int32), ("index_bits", ctypes.c_int32),
                ("ring_segments", ctypes.c_int32), ("ring_row_slots", ctypes.c_int32),
                ("chunk", ctypes.c_int64), ("l2_window_bytes", ctypes.c_int64),
                ("l2_setaside_bytes", ctypes.c_int64)]


_i32, _i64, _u32, _vp, _sz = ctypes.c_int32, ctypes.c_int64, ctypes.c_uint32, ctypes.c_void_p, ctypes.c_size_t
_st = ctypes.c_int
_D = ctypes.POINTER(nest_desc)

# name -> (restype, argtypes); every symbol include/nest.h declares
SIGNATURES = {
    "nest_abi_version": (_u32, []),
    "nest_status_str": (ctypes.c_char_p, [_st]),
    "nest_last_error": (ctypes.c_char_p, []),
    "nest_plan": (_st, [_D, _i64, _i32, ctypes.POINTER(nest_plan_info)]),
    "nest_spmv_plan": (_st, [_D, _i64, _i64, _i64, ctypes.POINTER(nest_plan_info)]),
    "nest_spmv_csr_f64": (_st, [_D, _i64, _i64, _i64, _vp, _vp, _vp, _vp, _vp, _vp]),
    "nest_spmv_hostio_workspace_bytes": (_sz, [_i64, _i64, _i64]),
    "nest_spmv_csr_f64_hostio": (_st, [_D, _i64, _i64, _i64, _vp, _vp, _vp, _vp, _vp, _vp, _sz, _vp]),
    "nest_batched_matvec_f32": (_st, [_D, _i64, _i32, _i32, _vp, _vp, _vp, _vp]),
    "nest_nested_stencil_f64": (_st, [_D, _i64, _i32, _vp, _vp, _vp, _vp, _vp, _vp]),
    "nest_probe_mapping": (_st, [_D, _vp, _i64, _vp, _vp, _vp, _vp]),
    "nest_laplace3d_f64": (_st, [_D, _i64, _i64, _i64, ctypes.c_double, _vp, _vp, _vp]),
    "nest_csr_validate": (_st, [_i64, _i64, _i64, _vp, _vp, _vp, _vp]),
    "nest_util_l2_flush": (_st, [_vp, _sz, _vp]),
    "nest_comm_unique_id": (_st, [_vp]),
    "nest_comm_init": (_st, [_vp, _i32, _i32, ctypes.POINTER(_vp)]),
    "nest_comm_destroy": (_st, [_vp]),
    "nest_spmv_csr_f64_dist": (_st, [_D, _vp, _i64, _i64, _i64, _i64, _vp, _vp, _vp, _vp, _vp, _vp, _vp]),
    "nest_comm_allgather_x": (_st, [_vp, _vp, _vp, _i64, _vp]),
    "nest_spmv_dist_hostio_workspace_bytes": (_sz, [_i64, _i64, _i64, _i32]),
    "nest_spmv_csr_f64_dist_hostio": (_st, [_D, _vp, _i64, _i64, _i64, _i64, _vp, _vp, _vp, _vp, _vp, _vp, _sz,
                                            _vp]),
    "nest_region_program": (_st, [_D, ctypes.POINTER(nest_region), _i32, _vp]),
    "nest_xpeer_handle_bytes": (_sz, []),
    "nest_xpeer_create": (_st, [_i32, _i32, _i64, ctypes.POINTER(_vp), _vp]),
    "nest_xpeer_open": (_st, [_vp, _vp]),
    "nest_xpeer_create_local": (_st, [_i32, _i32, _i64, ctypes.POINTER(_vp), ctypes.POINTER(_vp)]),
    "nest_xpeer_local_x": (_vp, [_vp]),
    "nest_xpeer_xchunk": (_i64, [_vp]),
    "nest_xpeer_set_x": (_st, [_vp, _vp, _i64, _vp]),
    "nest_xpeer_barrier": (_st, [_vp, _vp]),
    "nest_spmv_csr_f64_xpeer": (_st, [_D, _vp, _i64, _i64, _i64, _vp, _vp, _vp, _vp, _vp]),
    "nest_xpeer_destroy": (_st, [_vp]),
    "nest_shutdown": (_st, []),
    "nest_xsym_create": (_st, [_i32, _i32, _i64, ctypes.POINTER(ctypes.c_void_p), ctypes.POINTER(_i32)]),
    "nest_xsym_open": (_st, [_vp, ctypes.POINTER(_i32)]),
    "nest_xsym_create_local": (_st, [_i32, _i64, ctypes.POINTER(ctypes.c_void_p)]),
    "nest_xsym_x": (_vp, [_vp]),
    "nest_xsym_local_x": (_vp, [_vp]),
    "nest_xsym_xchunk": (_i64, [_vp]),
    "nest_xsym_set_x": (_st, [_vp, _i32, _vp, _i64, _vp]),
    "nest_xsym_destroy": (_st, [_vp]),
}

for _name, (_res, _args) in SIGNATURES.items():
    _f = getattr(lib, _name)
    _f.restype = _res
    _f.argtypes = _args
    globals()[_name] = _f

if lib.nest_abi_version() != NEST_ABI_VERSION:
    raise ImportError(f"libnest.so ABI {lib.nest_abi_version()} != {NEST_ABI_VERSION}")
