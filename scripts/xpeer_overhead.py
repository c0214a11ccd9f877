"""NEXT-4 peer-gather SpMV on one GPU with P virtual ranks (x split into P device
slices, the owner of column c = c / xchunk looked up per gather) against the plain
kernel on the same rows with one x: the in-kernel cost of the owner lookup, without
NVLink.  Rank 0's shard of configs[4] at P = 8 (12.5M rows, x = 800 MB).  Median of 10
launches, L2 flushed before each (developer tool).  Also the symmetric x (NEXT-4b):
the same 8 slices mapped into one virtual range, plain kernel."""
import os
import statistics
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
import paper_conf_icpp_wrightdtcc23_b200 as P  # noqa: E402
from nestgen import recipes as R  # noqa: E402

spec, nranks = R.CFG5, 8
_, rb, nloc = P.shard_rows(spec.nrows, nranks, 0)
drp, dcol, dval, nnz, _, _ = bench.gen_to_device(torch, spec, torch.device("cuda"), row_begin=rb, nrows=nloc)
x = R.spmv_x(spec)
dx = torch.from_numpy(x).cuda()
xc = P.x_chunk(spec.ncols, nranks)
sl = []
for r in range(nranks):
    s = torch.zeros(xc, dtype=torch.float64, device="cuda")
    b, k = P.local_x_range(spec.ncols, nranks, r)
    s[:k] = dx[b:b + k]
    sl.append(s)
xsym = P.XSym(spec.ncols, nranks=nranks)   # the same slices, mapped into one virtual range
for r in range(nranks):
    lo = r * xsym.xchunk
    if lo < spec.ncols:
        xsym.set_x(dx[lo:lo + xsym.xchunk], rank=r)
torch.cuda.synchronize()
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
B = nnz * 12 + (nloc + 1) * 8 + nloc * 8 + spec.ncols * 8
y = torch.empty(nloc, dtype=torch.float64, device="cuda")
for S, vec in ((8, True), (2, True), (8, False)):
    cfg = dict(simdlen=S, vec128=vec, blocked=True, threads_per_team=1024)
    xp = P.XPeer(spec.ncols, nranks=nranks, rank=0, local_slices=sl)
    plain = lambda: P.spmv_csr_f64(drp, dcol, dval, dx, y, ncols=spec.ncols, **cfg)
    peer = lambda: xp.spmv_csr_f64(spec.nrows, drp, dcol, dval, y, **cfg)
    res = {}
    sym = lambda: xsym.spmv_csr_f64(drp, dcol, dval, y, **cfg)
    for name, fn in (("plain x", plain), ("peer slices", peer), ("symmetric x", sym)):
        fn()
        ms = statistics.median(bench.time_steps(torch, fn, flush, P, 10))
        res[name] = ms
        print(f"S={S} {'pairs' if vec else 'scalar'} {name:12s} {ms:.4f} ms  {B / ms / 1e6:.0f} GB/s", flush=True)
    xp.close()
    print(f"   owner-lookup overhead {res['peer slices'] / res['plain x'] - 1:+.1%}, "
          f"symmetric x {res['symmetric x'] / res['plain x'] - 1:+.1%}", flush=True)
