/*
 * oracle.c -- TEST INFRASTRUCTURE ONLY.  The plain, slow, sequential CPU
 * definition of what the three-level loop nests compute.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs may load this library.  The product path
 * (paper_conf_icpp_wrightdtcc23_b200/) never imports, links or calls it, and
 * it shares no code with the CUDA path: no headers, no helpers, no constants.
 *
 * Source of truth: /root/reference/PAPER.md (Wright et al., ICPP'23).  The
 * method is a parallel SCHEDULE of an ordinary loop nest (teams -> parallel ->
 * simd); the result it reaches is, up to
 * floating-point summation order, the plain sequential loop nest.  So each
 * body below is that loop nest written out in storage order, in fp64, compiled
 * with -O2 -ffp-contract=off (no FMA contraction, no -ffast-math), on one
 * thread -- except oracle_spmv_csr_f64_threads, the same per-row loop with the
 * rows split among host threads (the all-cores CPU baseline; bit-identical).
 * The simd reduction is the north_star's addition (the paper used an atomic
 * update, and lists reductions as future work,
 * PAPER.md:868-873); its identity/combine are the textbook ones (R2).
 *
 * The mapping functions (group partition, simd worksharing owner, plan
 * geometry) follow the paper's definitions: PAPER.md:484-496, 507-529
 * (groups of adjacent threads inside one warp; simdmask), Fig 8 /
 * PAPER.md:830-840 (cyclic lane assignment), PAPER.md:677-704 (sharing space
 * split evenly among groups; global fallback).
 *
 * Pinned by tests/test_oracle_*.py (closed forms, brute force, library special
 * cases, paper-printed values in tests/golden/).  Nothing here is "parity
 * unpinned".
 */
#include <math.h>
#include <omp.h>
#include <stdint.h>
#include <stddef.h>

enum { OR_SUM = 0, OR_MAX = 1, OR_MIN = 2 };

/* Reduction identity and combine (R2/R5): sum starts at +0.0. */
static double or_identity(int op) {
    if (op == OR_MAX) return -INFINITY;
    if (op == OR_MIN) return INFINITY;
    return +0.0;
}

static double or_combine(int op, double s, double t) {
    if (op == OR_MAX) return t > s ? t : s;
    if (op == OR_MIN) return t < s ? t : s;
    return s + t;
}

uint32_t oracle_version(void) { return 1u; }

/* a8 -- CSR SpMV (sparse_matvec): for each row i,
 *   y_i = (+)_{k in [rowptr_i, rowptr_{i+1})} val_k * x_{col_k}
 * in storage order.  absy_i = sum |val_k * x_{col_k}| (tolerance scale, R3).
 * rowptr is relative: rowptr[0] need not be 0 (entries index col/val). */
static void spmv_row(int64_t i, const int64_t *rowptr, const int32_t *col, const double *val,
                     const double *x, int op, double *y, double *absy) {
    double s = or_identity(op), a = 0.0;
    for (int64_t k = rowptr[i]; k < rowptr[i + 1]; ++k) {
        double t = val[k] * x[col[k]];
        s = or_combine(op, s, t);
        a += fabs(t);
    }
    y[i] = s;
    if (absy) absy[i] = a;
}

int oracle_spmv_csr_f64(int64_t nrows, const int64_t *rowptr, const int32_t *col,
                        const double *val, const double *x, int op, double *y, double *absy) {
    if (nrows < 0 || op < 0 || op > 2) return 1;
    for (int64_t i = 0; i < nrows; ++i) spmv_row(i, rowptr, col, val, x, op, y, absy);
    return 0;
}

/* The same per-row loop with the rows split among `nthreads` host threads
 * (OpenMP, static schedule) -- the all-cores CPU baseline of BASELINE.md §4.
 * Rows are independent and each row's sum runs in storage order on one thread,
 * so the result is bit-identical to oracle_spmv_csr_f64 for any thread count
 * (pinned by tests/test_oracle_spmv.py).  Returns the thread count used. */
int oracle_spmv_csr_f64_threads(int64_t nrows, const int64_t *rowptr, const int32_t *col,
                                const double *val, const double *x, int op, double *y, double *absy,
                                int nthreads) {
    if (nrows < 0 || op < 0 || op > 2 || nthreads < 1) return -1;
    int used = 1;
#pragma omp parallel num_threads(nthreads)
    {
#pragma omp single
        used = omp_get_num_threads();
#pragma omp for schedule(static)
        for (int64_t i = 0; i < nrows; ++i) spmv_row(i, rowptr, col, val, x, op, y, absy);
    }
    return used;
}

/* a9 -- batched small dense matvec (SU3_bench stand-in):
 *   y[b][r] = (float)( (+)_{k<n} (double)A[b][r][k] * (double)x[b][k] )
 * fp32 x fp32 products are exact in fp64, so this is the correctly-ordered
 * fp64 result rounded once (the more accurate side, R3). */
int oracle_batched_matvec_f32(int64_t batch, int32_t m, int32_t n, const float *A,
                              const float *x, int op, float *y, double *absy) {
    if (batch < 0 || m < 0 || n < 0 || op < 0 || op > 2) return 1;
    for (int64_t b = 0; b < batch; ++b)
        for (int32_t r = 0; r < m; ++r) {
            double s = or_identity(op), a = 0.0;
            for (int32_t k = 0; k < n; ++k) {
                double t = (double)A[(b * m + r) * (int64_t)n + k] * (double)x[b * (int64_t)n + k];
                s = or_combine(op, s, t);
                a += fabs(t);
            }
            y[b * m + r] = (float)s;
            if (absy) absy[b * m + r] = a;
        }
    return 0;
}

/* a10 -- nested loop with a sequential prologue ("benchmark kernel" stand-in,
 * PAPER.md:900-907, and the generic-vs-SPMD study):
 *   for i in [0,N):  scale = w[i]; base = 1 + i*L; visits += 1;
 *                    trip = (scale == 0) ? 0 : L
 *                    s = (+)_{j<trip} coef[j] * ((in[base+j-1] + 2*in[base+j]) + in[base+j+1])
 *                    out[i] = (trip == 0) ? +0.0 : scale * s
 * visits counts outer iterations (the non-idempotent side effect that SPMD
 * mode must guard). */
int oracle_nested_stencil_f64(int64_t nouter, int32_t L, const double *in, const double *coef,
                              const double *w, int op, double *out, double *absout,
                              uint64_t *visits) {
    if (nouter < 0 || L < 0 || op < 0 || op > 2) return 1;
    uint64_t v = 0;
    for (int64_t i = 0; i < nouter; ++i) {
        double scale = w[i];
        int64_t base = 1 + i * (int64_t)L;
        v += 1;
        int32_t trip = (scale == 0.0) ? 0 : L;
        double s = or_identity(op), a = 0.0;
        for (int32_t j = 0; j < trip; ++j) {
            double t = coef[j] * ((in[base + j - 1] + 2.0 * in[base + j]) + in[base + j + 1]);
            s = or_combine(op, s, t);
            a += fabs(t);
        }
        out[i] = (trip == 0) ? +0.0 : scale * s;
        if (absout) absout[i] = fabs(scale) * a;
    }
    if (visits) *visits = v;
    return 0;
}

/* NEXT-2 -- laplace3d heat-diffusion step ("a simple
 * three-dimensional heat diffusion kernel called laplace3d"; the paper gives no
 * formula; R21 fixes the 7-point Jacobi step, its summation order,
 * alpha as an argument and the untouched boundary):
 *   for i in [1,nz-1), j in [1,ny-1), k in [1,nx-1):
 *     lap = (((((u[i-1][j][k] + u[i+1][j][k]) + u[i][j-1][k]) + u[i][j+1][k])
 *              + u[i][j][k-1]) + u[i][j][k+1]) - 6*u[i][j][k]
 *     out[i][j][k] = u[i][j][k] + alpha*lap
 * Boundary points of out are left untouched. */
int oracle_laplace3d_f64(int64_t nz, int64_t ny, int64_t nx, double alpha, const double *u, double *out) {
    if (nz < 0 || ny < 0 || nx < 0) return 1;
    for (int64_t i = 1; i < nz - 1; ++i)
        for (int64_t j = 1; j < ny - 1; ++j)
            for (int64_t k = 1; k < nx - 1; ++k) {
                const int64_t c = (i * ny + j) * nx + k;
                double lap = u[c - ny * nx] + u[c + ny * nx];
                lap = lap + u[c - nx];
                lap = lap + u[c + nx];
                lap = lap + u[c - 1];
                lap = lap + u[c + 1];
                lap = lap - 6.0 * u[c];
                out[c] = u[c] + alpha * lap;
            }
    return 0;
}

/* a2 -- SIMD-group partition of a team of T threads into groups of S adjacent
 * threads, queried per thread as in
 * PAPER.md:507-529.  out[t*5 + {0..4}] = {getSimdGroup, getSimdGroupId,
 * getSimdGroupSize, isSimdGroupLeader, simdmask}.  The mask is built by
 * testing every lane of the thread's warp for group membership. */
int oracle_group_map(int32_t T, int32_t S, int32_t *out) {
    if (T <= 0 || S <= 0 || T % S || 32 % S) return 1;
    for (int32_t t = 0; t < T; ++t) {
        int32_t g = t / S, id = t - g * S;
        uint32_t mask = 0;
        int32_t warp0 = (t / 32) * 32;
        for (int32_t l = 0; l < 32; ++l)
            if (warp0 + l < T && (warp0 + l) / S == g) mask |= 1u << l;
        out[t * 5 + 0] = g;
        out[t * 5 + 1] = id;
        out[t * 5 + 2] = S;
        out[t * 5 + 3] = (id == 0);
        out[t * 5 + 4] = (int32_t)mask;
    }
    return 0;
}

/* a5 -- Fig 8 (__simd_loop) replayed per lane: lane `id`
 * starts at omp_iv = id and steps by the group size.  owner[j] = the lane that
 * executes iteration j.  Every j in [0,trip) is written exactly once. */
int oracle_simd_owner(int64_t trip, int32_t S, int32_t *owner) {
    if (trip < 0 || S <= 0) return 1;
    for (int64_t j = 0; j < trip; ++j) owner[j] = -1;
    for (int32_t id = 0; id < S; ++id)
        for (uint64_t iv = (uint64_t)id; iv < (uint64_t)trip; iv += (uint64_t)S) owner[iv] = id;
    return 0;
}

/* a1 -- launch geometry from the paper's constraints.  Valid iff S is a
 * power of two dividing the warp (groups equal-size, never spanning a warp:
 * PAPER.md:484-491, 511-513, 689-691) and T is whole warps in [32,1024].
 * groups/team G = T/S; the sharing space (default 2048 B)
 * is divided evenly among the groups: slot = sharing/G
 * rounded down to the 8-byte alignment of the payload entries (the paper's
 * entries are pointers; R8);
 * a payload larger than its slot falls back to global memory
 * (PAPER.md:680-684).  out = {G, slot_bytes, uses_global_fallback}. */
int oracle_plan_geometry(int32_t T, int32_t S, int32_t sharing_bytes, int32_t payload_bytes,
                         int32_t *out) {
    int s_ok = 0;
    for (int32_t p = 1; p <= 32; p *= 2) s_ok |= (S == p);
    if (!s_ok || T < 32 || T > 1024 || T % 32 || sharing_bytes < 0 || payload_bytes < 0) return 1;
    int32_t G = T / S;
    out[0] = G;
    out[1] = (sharing_bytes / G) / 8 * 8;   /* each slot holds 8-byte aligned payloads (R8) */
    out[2] = payload_bytes > out[1];
    return 0;
}

/* a12 -- equal-row partition of n rows over P ranks:
 * chunk = ceil(n/P); rank r owns [r*chunk, min((r+1)*chunk, n)). */
int oracle_shard_rows(int64_t n, int32_t P, int32_t r, int64_t *out /* chunk, begin, count */) {
    if (n < 0 || P <= 0 || r < 0 || r >= P) return 1;
    int64_t chunk = (n + P - 1) / P;
    int64_t b = (int64_t)r * chunk;
    if (b > n) b = n;
    int64_t e = b + chunk;
    if (e > n) e = n;
    out[0] = chunk;
    out[1] = b;
    out[2] = e - b;
    return 0;
}
