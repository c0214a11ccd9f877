"""compute-sanitizer driver workload: small cfg1-sized SpMV / stencil / batched /
probe launches in every mode (generic modes exercise the slot handshake and the
warp barriers).  Run under compute-sanitizer --tool {memcheck,racecheck,synccheck}."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_wrightdtcc23_b200 as P  # noqa: E402
from nestgen import recipes as R  # noqa: E402

rp, col, val, x = [torch.from_numpy(a).cuda() for a in R.spmv_inputs(R.CFG1)]
inp, coef, w = [torch.from_numpy(a).cuda() for a in R.stencil_inputs(4099, 8)]
A, xb = [torch.from_numpy(a).cuda() for a in R.batched_inputs(64)]
for S in (2, 8, 32):
    for mode in ("spmd", "generic_smem", "generic_shfl"):
        for extra in ({}, {"blocked": True}, {"vec128": True}, {"sharing_bytes": 64}):
            P.spmv_csr_f64(rp, col, val, x, simdlen=S, mode=mode, **extra)
        # x ring: copy warp + mbarrier segment ring, per-warp cp.async row-bound stages
        P.spmv_csr_f64(rp, col, val, x, simdlen=S, mode=mode, x_halo=100)
        P.spmv_csr_f64(rp, col, val, x, simdlen=S, mode=mode, x_halo=300, vec128=True, threads_per_team=768,
                       outer_unroll=2, num_teams=3)
        P.spmv_csr_f64(rp[1:], col, val, x, simdlen=S, mode=mode, x_halo=50, threads_per_team=64)
        P.nested_stencil_f64(inp, coef, w, 4099, 8, simdlen=S, mode=mode)
        # pair tuples with the speculative head; U simd loops in flight (transpose-reduce in SPMD)
        P.nested_stencil_f64(inp, coef, w, 4099, 8, simdlen=S, mode=mode, vec128=True)
        P.nested_stencil_f64(inp, coef, w, 4099, 8, simdlen=S, mode=mode, outer_unroll=4)
        P.spmv_csr_f64(rp, col, val, x, simdlen=S, mode=mode, outer_unroll=2, threads_per_team=512)
        P.spmv_csr_f64(rp, col, val, x, simdlen=S, mode=mode, quad=True, blocked=True, threads_per_team=1024)
        # x under a persisting-L2 access-policy window (cudaLaunchKernelEx), then the flush's reset
        P.spmv_csr_f64(rp, col, val, x, simdlen=S, mode=mode, quad=True, blocked=True, threads_per_team=1024,
                       x_l2_persist=True)
        P.l2_flush(torch.empty(4 << 20, dtype=torch.uint8, device="cuda"))
        P.batched_matvec_f32(A, xb, 64, simdlen=S, mode=mode, outer_unroll=2)
        P.batched_matvec_f32(A, xb, 64, simdlen=S, mode=mode)   # lean SPMD / generic drivers (U = 1)
        P.spmv_csr_f64(rp, col, val, x, simdlen=S, mode=mode, blocked=True, vec128=True, threads_per_team=1024,
                       team_chunk=64)
        u = torch.rand(12 * 10 * 9, dtype=torch.float64, device="cuda")
        P.laplace3d_f64(u, u.clone(), 12, 10, 9, 0.1, simdlen=S, mode=mode)
        P.probe_mapping(2, 37, simdlen=S, mode=mode)
torch.cuda.synchronize()
print("sanitize workload done")
