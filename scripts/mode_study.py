"""Launch one kernel per (body, simdlen, mode) for an ncu metrics pass -- the
SPMD-vs-generic cost study of SURVEY.md §8(d) (warp execution efficiency,
branch divergence, shared-memory slot traffic, instructions).  Run under
scripts/mode_study.sh; prints the launch order (one line per kernel)."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_wrightdtcc23_b200 as P  # noqa: E402
from nestgen import recipes as R  # noqa: E402

spec = R.CFG2
rp, col, val = R.spmv_matrix(spec)
x = R.spmv_x(spec)
t = [torch.from_numpy(v).cuda() for v in (rp, col, val, x)]
y = torch.empty(spec.nrows, dtype=torch.float64, device="cuda")
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
N, L = 1 << 20, 32
inp, coef, w = (torch.from_numpy(a).cuda() for a in R.stencil_inputs(N, L))
out = torch.empty(N, dtype=torch.float64, device="cuda")
visits = torch.zeros(1, dtype=torch.int64, device="cuda")
runs = []
for S in (1, 2, 8, 32):
    for mode in (("spmd",) if S == 1 else ("spmd", "generic_smem", "generic_shfl")):
        runs.append(("spmv_cfg2_blocked_scalar", S, mode,
                     lambda S=S, mode=mode: P.spmv_csr_f64(*t, y, simdlen=S, mode=mode, threads_per_team=1024,
                                                           blocked=True)))
# the 128-bit quad body (the bench headline's, without the persisting window: ncu neutralises it)
for S in (1, 2, 4, 8):
    for mode in (("spmd",) if S == 1 else ("spmd", "generic_smem", "generic_shfl")):
        runs.append(("spmv_cfg2_blocked_quads", S, mode,
                     lambda S=S, mode=mode: P.spmv_csr_f64(*t, y, simdlen=S, mode=mode, threads_per_team=1024,
                                                           blocked=True, quad=True)))
# transpose-reduce: SPMD with two rows per group in flight
for S in (8, 16):
    runs.append(("spmv_cfg2_blocked_pairs_U2", S, "spmd",
                 lambda S=S: P.spmv_csr_f64(*t, y, simdlen=S, mode="spmd", threads_per_team=1024, blocked=True,
                                            vec128=True, outer_unroll=2)))
for S in (1, 4, 8, 32):
    for mode in (("spmd",) if S == 1 else ("spmd", "generic_smem", "generic_shfl")):
        runs.append((f"stencil_pairs_N2^20_L{L}", S, mode,
                     lambda S=S, mode=mode: P.nested_stencil_f64(inp, coef, w, N, L, out, visits, simdlen=S,
                                                                 mode=mode, vec128=True, blocked=True)))
for S in (1, 4, 8, 32):
    for mode in (("spmd",) if S == 1 else ("spmd", "generic_smem", "generic_shfl")):
        runs.append((f"stencil_N2^20_L{L}", S, mode,
                     lambda S=S, mode=mode: P.nested_stencil_f64(inp, coef, w, N, L, out, visits, simdlen=S,
                                                                 mode=mode)))
for name, S, mode, fn in runs:
    fn()   # warm (module load, fallback allocation): not the profiled launch
    torch.cuda.synchronize()
    P.l2_flush(flush)
    fn()
    torch.cuda.synchronize()
    print(f"RUN {name} S={S} {mode}", flush=True)
