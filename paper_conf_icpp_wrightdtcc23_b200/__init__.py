"""B200-native three-level (teams -> parallel -> simd) loop nests.

The data-parallel hot path of Wright et al., "Implementing OpenMP's SIMD
Directive in LLVM's GPU Runtime" (ICPP'23): SIMD groups of simdlen lanes,
generic (SIMD main + state machine) and SPMD execution of the parallel region,
in-group __shfl_xor_sync reductions, behind the C ABI of include/nest.h.
Importing this package loads libnest.so and fails loudly if it is missing.
"""
from . import _nest  # noqa: F401  (loads libnest.so or raises)
from .api import (MODES, REDUCES, SIMDLENS, NestError, batched_matvec_f32, check, csr_validate,
                  hostio_workspace_bytes, l2_flush, laplace3d_f64, make_desc, nested_stencil_f64, plan,
                  probe_mapping, region_program, shutdown, spmv_csr_f64, spmv_csr_f64_hostio, spmv_plan)
from .dist import Comm, XPeer, XSym, broadcast_unique_id, local_x_range, shard_rows, x_chunk

__all__ = ["MODES", "REDUCES", "SIMDLENS", "NestError", "batched_matvec_f32", "check", "XSym",
           "csr_validate", "hostio_workspace_bytes", "l2_flush", "laplace3d_f64", "make_desc",
           "nested_stencil_f64", "plan", "probe_mapping", "region_program", "shutdown", "spmv_csr_f64",
           "spmv_csr_f64_hostio", "spmv_plan", "Comm", "XPeer", "broadcast_unique_id", "local_x_range", "shard_rows",
           "x_chunk"]
