"""NEXT-3: parallel regions with different simdlen in one kernel
(PAPER.md:511-513, 686-698).  EVERY region is checked against the CPU oracle
directly -- bit-exact on integer-valued inputs (R4), within R3 on real ones --
and is also bit-identical to the stand-alone entry point at the same simdlen
and mode; the stencil's visit counter equals nouter, and a tiny sharing space
forces some regions onto the global fallback without
changing any result."""
import numpy as np
import pytest

import oracle
from nestgen import recipes as R

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def P():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_icpp_wrightdtcc23_b200 as P
    return P


def bits(t):
    a = t.cpu().numpy()
    return a.view(np.int64 if a.dtype == np.float64 else np.int32)


def _data(values):
    spec = R.SpmvSpec("prog", 4343, 20_000, 20_000, 0, 40, band_w=900, far_den=8, values=values)
    rp, col, val, x = R.spmv_inputs(spec)
    ys, ya = oracle.spmv_csr_f64(rp, col, val, x)
    B = 777
    A, xb = R.batched_inputs(B, values=values)
    yb, ab = oracle.batched_matvec_f32(A, xb, B)
    N, L = 5003, 16
    inp, coef, w = R.stencil_inputs(N, L, values=values)
    yo, ao, vo = oracle.nested_stencil_f64(inp, coef, w, N, L)
    cu = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
    return dict(spmv=[cu(a) for a in (rp, col, val, x)], ys=ys, ya=ya, B=B, A=cu(A), xb=cu(xb), yb=yb, ab=ab,
                N=N, L=L, st=[cu(a) for a in (inp, coef, w)], yo=yo, ao=ao, vo=vo)


@pytest.fixture(scope="module")
def data():
    return {"real": _data("real"), "int": _data("int")}


def check_oracle(got, ref, absref, tol, integer):
    got = got.cpu().numpy()
    if integer:
        assert np.array_equal(got.view(np.int64 if got.dtype == np.float64 else np.int32),
                              np.ascontiguousarray(ref, got.dtype).view(np.int64 if got.dtype == np.float64
                                                                        else np.int32))
    else:
        zero = absref == 0
        assert np.all(got[zero] == 0.0)
        assert np.all(np.abs(got.astype(np.float64) - ref) <= tol * absref)


COMBOS = [  # (spmv S, mode), (batched S, mode), (stencil S, mode)
    ((8, "generic_smem"), (4, "spmd"), (32, "generic_shfl")),
    ((1, "spmd"), (32, "generic_smem"), (2, "generic_smem")),
    ((32, "spmd"), (2, "generic_shfl"), (16, "spmd")),
    ((4, "generic_shfl"), (16, "generic_smem"), (1, "spmd")),
]


@pytest.mark.parametrize("combo", COMBOS)
@pytest.mark.parametrize("T,sharing,teams", [(256, 0, 0), (128, 64, 0), (1024, 2048, 7)])
@pytest.mark.parametrize("values", ["int", "real"])
def test_region_program_matches_oracle(P, data, combo, T, sharing, teams, values):
    (s1, m1), (s2, m2), (s3, m3) = combo
    d = data[values]
    y = torch.empty(d["spmv"][0].numel() - 1, dtype=torch.float64, device="cuda")
    yb = torch.empty(d["B"] * 64, dtype=torch.float32, device="cuda")
    out = torch.empty(d["N"], dtype=torch.float64, device="cuda")
    visits = torch.zeros(1, dtype=torch.int64, device="cuda")
    rp, col, val, x = d["spmv"]
    inp, coef, w = d["st"]
    regions = [
        dict(kind="spmv", simdlen=s1, mode=m1, blocked=True, rowptr=rp, colind=col, val=val, x=x, y=y),
        dict(kind="batched", simdlen=s2, mode=m2, A=d["A"], x=d["xb"], y=yb, batch=d["B"], m=64, n=64),
        dict(kind="stencil", simdlen=s3, mode=m3, blocked=bool(teams), inp=inp, coef=coef, w=w, out=out,
             nouter=d["N"], L=d["L"], visits=visits),
    ]
    P.region_program(regions, threads_per_team=T, sharing_bytes=sharing, num_teams=teams)
    integer = values == "int"
    # every region against the oracle (the paper's definition), not just against the library
    check_oracle(y, d["ys"], d["ya"], 1e-12, integer)
    check_oracle(yb, d["yb"], d["ab"], 1e-5, integer)
    check_oracle(out, d["yo"], d["ao"], 1e-12, integer)
    assert int(visits.item()) == d["vo"] == d["N"]
    # and bit-identical to the stand-alone entry points (same lane order)
    ref_y = P.spmv_csr_f64(rp, col, val, x, simdlen=s1, mode=m1)
    ref_yb = P.batched_matvec_f32(d["A"], d["xb"], d["B"], simdlen=s2, mode=m2)
    ref_out = P.nested_stencil_f64(inp, coef, w, d["N"], d["L"], simdlen=s3, mode=m3)
    assert np.array_equal(bits(y), bits(ref_y))
    assert np.array_equal(bits(yb), bits(ref_yb))
    assert np.array_equal(bits(out), bits(ref_out))


def test_region_program_rejects(P, data):
    rp, col, val, x = data["real"]["spmv"]
    y = torch.empty(rp.numel() - 1, dtype=torch.float64, device="cuda")
    r = dict(kind="spmv", simdlen=8, rowptr=rp, colind=col, val=val, x=x, y=y)
    with pytest.raises(P.NestError):
        P.region_program([r] * 5)                         # more than NEST_MAX_REGIONS
    with pytest.raises(P.NestError):
        P.region_program([dict(r, simdlen=3)])            # not a divisor of the warp
    with pytest.raises(P.NestError):
        P.region_program([r], reduce="max")               # SUM only
