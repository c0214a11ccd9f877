"""Dump the cfg2 CSR matrix and x (nestgen) as raw binaries for scripts/l2x_probe (file:<prefix>)."""
import sys
import os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from nestgen import recipes as R  # noqa: E402

pre = sys.argv[1] if len(sys.argv) > 1 else "/tmp/cfg2"
rp, col, val = R.spmv_matrix(R.CFG2)
x = R.spmv_x(R.CFG2)
for a, s in ((rp, "rp"), (col, "col"), (val, "val"), (x, "x")):
    a.tofile(f"{pre}_{s}.bin")
print(rp.dtype, col.dtype, val.dtype, x.dtype, rp.size - 1, val.size)
