"""compute-sanitizer workload for the pair-tuple stencil (StencilVecBody):
small N, every simdlen and mode, L = 2 and 34 (ragged pair counts per lane)."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_wrightdtcc23_b200 as P  # noqa: E402
from nestgen import recipes as R  # noqa: E402

N = 517
for L in (2, 34):
    t = [torch.from_numpy(a).cuda() for a in R.stencil_inputs(N, L)]
    for S in (1, 2, 4, 8, 16, 32):
        for mode in ("spmd", "generic_smem", "generic_shfl"):
            for U in (1, 2):
                P.nested_stencil_f64(*t, N, L, simdlen=S, mode=mode, outer_unroll=U, vec128=True)
torch.cuda.synchronize()
print("stencil vec sanitize workload done")
