"""GPU parity of the end-to-end a8 call (nest_spmv_csr_f64_hostio) in its
chunked-pipeline form: the matrix crosses PCIe in row chunks on an H2D stream
while earlier chunks' SpMV and y copies run.  The chunks run
the same kernel on the same rows, so the result must equal the device-resident
call bit for bit, and the oracle within the R3 tolerance."""
import os
import subprocess
import sys
import textwrap
from dataclasses import replace

import numpy as np
import pytest

import oracle
from nestgen import recipes as R

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

# the bench headline (quads), 128-bit pairs, the scalar body, a generic mode, and the
# x ring (chunks start at odd rows: 8-byte aligned row-bound copies)
CONFIGS = (dict(simdlen=2, threads_per_team=1024, blocked=True, quad=True),
           dict(simdlen=2, threads_per_team=1024, blocked=True, vec128=True),
           dict(simdlen=1, threads_per_team=1024, blocked=True, quad=True),
           dict(simdlen=8),
           dict(simdlen=4, mode="generic_smem", threads_per_team=1024, blocked=True),
           dict(simdlen=2, x_halo=300, threads_per_team=256, vec128=True))


@pytest.fixture(scope="module")
def P():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_icpp_wrightdtcc23_b200 as P
    return P


def assert_close(y, ref, absref, tol=1e-12):
    zero = absref == 0
    assert np.all(y[zero] == 0.0)
    assert not (np.abs(y - ref) > tol * absref).any()


def run_both(P, rp, col, val, x, cfg):
    pin = lambda a: torch.from_numpy(np.ascontiguousarray(a)).pin_memory()
    hy = torch.full((rp.size - 1,), np.nan, dtype=torch.float64).pin_memory()
    ws = torch.empty(P.hostio_workspace_bytes(rp.size - 1, x.size, val.size), dtype=torch.uint8, device="cuda")
    ws.fill_(0xFF)   # NaN bytes: a chunk that read an entry before its copy landed would show
    P.spmv_csr_f64_hostio(pin(rp), pin(col), pin(val), pin(x), hy, ws, **cfg)
    torch.cuda.synchronize()
    d = [torch.from_numpy(np.ascontiguousarray(a)).cuda() for a in (rp, col, val, x)]
    yd = P.spmv_csr_f64(*d, **cfg).cpu().numpy()
    return hy.numpy().copy(), yd


def test_hostio_pipelined_multi_chunk(P):
    """~21M nonzeros: three chunks of the default 8 Mi-nonzero size, rows with
    0..12 nonzeros (empty rows included)."""
    spec = replace(R.CFG2, name="hostio", seed=R.seed(8), nrows=3_500_000, ncols=3_500_000, nnz_min=0)
    rp, col, val = R.spmv_matrix(spec)
    x = R.spmv_x(spec)
    assert rp[-1] > 2 * (8 << 20)
    yref, aref = oracle.spmv_csr_f64(rp, col, val, x)
    for cfg in CONFIGS:
        yh, yd = run_both(P, rp, col, val, x, cfg)
        assert np.array_equal(yh.view(np.int64), yd.view(np.int64)), cfg
        assert_close(yh, yref, aref)


_CHILD = textwrap.dedent("""
    import sys, numpy as np, torch
    sys.path.insert(0, {root!r})
    import oracle, paper_conf_icpp_wrightdtcc23_b200 as P
    from dataclasses import replace
    from nestgen import recipes as R
    import importlib.util   # by path: a site-packages "tests" package may shadow ours
    spec_ = importlib.util.spec_from_file_location("_hostio_t", {path!r})
    T = importlib.util.module_from_spec(spec_)
    spec_.loader.exec_module(T)
    CONFIGS, run_both, assert_close = T.CONFIGS, T.run_both, T.assert_close
    for nrows, lo, hi in ((1, 0, 40), (7, 0, 3), (5000, 0, 9), (100_003, 2, 30)):
        spec = replace(R.CFG1, name="hio", seed=R.seed(9) + nrows, nrows=nrows, ncols=max(nrows, 64),
                       nnz_min=lo, nnz_max=hi)
        rp, col, val = R.spmv_matrix(spec)
        x = R.spmv_x(spec)
        yref, aref = oracle.spmv_csr_f64(rp, col, val, x)
        for cfg in CONFIGS:
            yh, yd = run_both(P, rp, col, val, x, cfg)
            assert np.array_equal(yh.view(np.int64), yd.view(np.int64)), (nrows, cfg)
            assert_close(yh, yref, aref)
    print("CHILD OK")
""")


@pytest.mark.parametrize("chunks", [2, 7, 32])
def test_hostio_forced_chunks_ragged(P, chunks):
    """Forced chunk counts (NEST_HOSTIO_CHUNKS, read once per process: a child
    process) on small ragged matrices: more chunks than rows, single rows,
    empty chunks, chunk boundaries inside 128-bit tuples."""
    env = dict(os.environ, NEST_HOSTIO_CHUNKS=str(chunks))
    r = subprocess.run([sys.executable, "-c", _CHILD.format(root=ROOT, path=os.path.abspath(__file__))], cwd=ROOT, env=env,
                       capture_output=True, text=True, timeout=600)
    assert r.returncode == 0 and "CHILD OK" in r.stdout, r.stdout[-2000:] + r.stderr[-4000:]


def test_hostio_rejects_rowptr_not_from_zero_to_nnz(P):
    rp = np.array([1, 3, 5], np.int64)
    col = np.zeros(5, np.int32)
    val = np.ones(5)
    x = np.ones(4)
    pin = lambda a: torch.from_numpy(a).pin_memory()
    ws = torch.empty(P.hostio_workspace_bytes(2, 4, 5), dtype=torch.uint8, device="cuda")
    hy = torch.empty(2, dtype=torch.float64).pin_memory()
    with pytest.raises(Exception, match="rowptr"):
        P.spmv_csr_f64_hostio(pin(rp), pin(col), pin(val), pin(x), hy, ws)
