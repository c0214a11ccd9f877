"""Workload recipes: shapes, distributions and seeds of the synthetic inputs.

The paper gives no matrices or sizes (PAPER.md:877-884, 895-907 only describe
the kernels), so every workload is synthetic with the
structure the paper describes: CSR rows that are short and irregular ("the
inner-most loop ... is relatively small, and varies based on the sparsity",
PAPER.md:879-880), a small inner dot product (SU3_bench analogue,
PAPER.md:895-898) and a small non-collapsible inner loop behind a sequential
prologue.  Config k uses seed 20230807 + k.
No method arithmetic lives here.
"""
from __future__ import annotations

from dataclasses import dataclass, replace


from . import (STREAM_BATCH_A, STREAM_BATCH_X, STREAM_ST_COEF, STREAM_ST_IN, STREAM_ST_W,
               STREAM_X, csr_fill, csr_rowptr, vec_f32, vec_f64)

SEED_BASE = 20230807


def seed(cfg: int) -> int:
    return SEED_BASE + cfg


@dataclass(frozen=True)
class SpmvSpec:
    name: str
    seed: int
    nrows: int
    ncols: int
    nnz_min: int
    nnz_max: int
    structure: str = "banded_far"   # or "uniform"
    band_w: int = 4096
    far_den: int = 16               # far column with probability 1/far_den
    values: str = "real"            # "real": U[-1,1); "int": integers in [vlo, vhi]
    vlo: int = -4
    vhi: int = 4
    xlo: int = -8                   # integer-valued x range (values == "int")
    xhi: int = 8

    def integer(self) -> "SpmvSpec":
        return replace(self, name=self.name + "_int", values="int")


# BASELINE.json configs[0]: 1,024 x 1,024, 8-32 random nnz/row (parity case)
CFG1 = SpmvSpec("cfg1", seed(1), 1024, 1024, 8, 32, structure="uniform")
# BASELINE.json configs[1]: 10M rows, ~8 nnz/row (short-row regime) -- the bench workload
CFG2 = SpmvSpec("cfg2", seed(2), 10_000_000, 10_000_000, 4, 12)
CFG2_UNIFORM = replace(CFG2, name="cfg2_uniform", structure="uniform")
# north_star 70% gate: a 100M-nnz matrix, same row-length law as cfg2 (SURVEY.md §8(d) "G100"), own seed
G100 = SpmvSpec("g100", seed(6), 12_500_000, 12_500_000, 4, 12)
# BASELINE.json configs[4]: 100M rows, ~16 nnz/row, row-partitioned over P GPUs
CFG5 = SpmvSpec("cfg5", seed(5), 100_000_000, 100_000_000, 8, 24)


def spmv_matrix(spec: SpmvSpec, row_begin: int = 0, nrows: int | None = None,
                rowptr_out=None, col_out=None, val_out=None):
    """CSR block of global rows [row_begin, row_begin+nrows) (local rowptr)."""
    n = spec.nrows - row_begin if nrows is None else nrows
    rp = csr_rowptr(spec.seed, n, spec.ncols, spec.nnz_min, spec.nnz_max, row_begin, out=rowptr_out)
    col, val = csr_fill(spec.seed, rp, spec.ncols, spec.structure, spec.band_w, spec.far_den,
                        spec.values, spec.vlo, spec.vhi, row_begin, col_out=col_out, val_out=val_out)
    return rp, col, val


def spmv_x(spec: SpmvSpec, begin: int = 0, n: int | None = None, out=None):
    n = spec.ncols - begin if n is None else n
    if spec.values == "int":
        return vec_f64(spec.seed, STREAM_X, n, "int", spec.xlo, spec.xhi, begin=begin, out=out)
    return vec_f64(spec.seed, STREAM_X, n, "real", begin=begin, out=out)


def spmv_inputs(spec: SpmvSpec):
    rp, col, val = spmv_matrix(spec)
    return rp, col, val, spmv_x(spec)


# BASELINE.json configs[2]: nested loop, 1M outer iterations, inner length 4-64
STENCIL_LS = (4, 8, 16, 32, 64)


def stencil_inputs(nouter: int, L: int, values: str = "real", cfg_seed: int = seed(3)):
    """in f64[nouter*L+2] (one halo element each end), coef f64[L], w f64[nouter].
    Real: in, coef ~ U[-1,1), w ~ U[0.5,1.5) except w[i]=0 for i % 8 == 0 (the
    skip branch).  Integer: in, coef in {-4..4}, w in {0..7}."""
    s = cfg_seed + 1000 * L
    if values == "int":
        a = vec_f64(s, STREAM_ST_IN, nouter * L + 2, "int", -4, 4)
        c = vec_f64(s, STREAM_ST_COEF, L, "int", -4, 4)
        w = vec_f64(s, STREAM_ST_W, nouter, "int", 0, 7)
    else:
        a = vec_f64(s, STREAM_ST_IN, nouter * L + 2, "real")
        c = vec_f64(s, STREAM_ST_COEF, L, "real")
        w = vec_f64(s, STREAM_ST_W, nouter, "half3half")
        w[::8] = 0.0
    return a, c, w


# BASELINE.json configs[3]: 64x64 fp32 matvec, 500k batches
def batched_inputs(batch: int, m: int = 64, n: int = 64, values: str = "real",
                   cfg_seed: int = seed(4)):
    """A f32[batch][m][n] row-major, x f32[batch][n].  Real: U[-1,1); int: {-3..3}."""
    if values == "int":
        A = vec_f32(cfg_seed, STREAM_BATCH_A, batch * m * n, "int", -3, 3)
        x = vec_f32(cfg_seed, STREAM_BATCH_X, batch * n, "int", -3, 3)
    else:
        A = vec_f32(cfg_seed, STREAM_BATCH_A, batch * m * n, "real")
        x = vec_f32(cfg_seed, STREAM_BATCH_X, batch * n, "real")
    return A, x


# NEXT-2 laplace3d: a (nz, ny, nx) fp64 field, U[-1,1) or integers in {-8..8}
LAPLACE_SHAPE = (256, 256, 256)


def laplace_inputs(nz: int, ny: int, nx: int, values: str = "real", cfg_seed: int = seed(7)):
    from . import vec_f64
    if values == "int":
        return vec_f64(cfg_seed, 41, nz * ny * nx, "int", -8, 8)
    return vec_f64(cfg_seed, 41, nz * ny * nx, "real")


__all__ = ["SpmvSpec", "CFG1", "CFG2", "CFG2_UNIFORM", "G100", "CFG5", "spmv_matrix", "spmv_x",
           "spmv_inputs", "stencil_inputs", "batched_inputs", "STENCIL_LS", "seed", "LAPLACE_SHAPE",
           "laplace_inputs"]
