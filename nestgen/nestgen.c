/*
 * nestgen.c -- seeded, counter-based synthetic input generators.
 *
 * This module is shared by BOTH sides of the parity check (the CPU oracle in
 * oracle/ and the CUDA path in paper_conf_icpp_wrightdtcc23_b200/).  It holds
 * none of the method's arithmetic: it only draws matrices and vectors.  Every
 * element is a pure function of (seed, stream, index, k), so any row range
 * (a multi-GPU shard, a bounded CPU sample) regenerates independently and
 * bit-identically.  Recipe: DESIGN.md "Input recipe"; SURVEY.md §8(d).
 *
 * Build: gcc -O2 -fopenmp -fPIC -shared (see Makefile).
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

enum { NG_STREAM_ROWLEN = 1, NG_STREAM_COL = 2, NG_STREAM_VAL = 3 };
enum { NG_UNIFORM = 0, NG_BANDED_FAR = 1 };
enum { NG_REAL_PM1 = 0, NG_INT = 1, NG_REAL_HALF_3HALF = 2 };

static inline uint64_t ng_mix(uint64_t z) {            /* splitmix64 finaliser */
    z += 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

static inline uint64_t ng_draw(uint64_t seed, uint64_t stream, uint64_t idx, uint64_t k) {
    return ng_mix(ng_mix(ng_mix(seed ^ (stream * 0xD1B54A32D192ED03ull)) ^ idx) ^ k);
}

/* uniform integer in [lo, hi] (inclusive), multiply-shift, no division */
static inline int64_t ng_int(uint64_t u, int64_t lo, int64_t hi) {
    uint64_t span = (uint64_t)(hi - lo) + 1u;
    return lo + (int64_t)(((unsigned __int128)u * span) >> 64);
}

static inline double ng_f64(uint64_t u, int kind, int64_t lo, int64_t hi) {
    switch (kind) {
    case NG_INT: return (double)ng_int(u, lo, hi);
    case NG_REAL_HALF_3HALF: return 0.5 + (double)(u >> 11) * 0x1.0p-53;
    default: return -1.0 + (double)(u >> 11) * 0x1.0p-52;           /* U[-1,1) */
    }
}

static inline float ng_f32(uint64_t u, int kind, int64_t lo, int64_t hi) {
    switch (kind) {
    case NG_INT: return (float)ng_int(u, lo, hi);
    case NG_REAL_HALF_3HALF: return 0.5f + (float)(u >> 40) * 0x1.0p-24f;
    default: return -1.0f + (float)(u >> 40) * 0x1.0p-23f;            /* U[-1,1) */
    }
}

uint32_t nestgen_version(void) { return 1u; }

/* Row lengths U{nnz_min..nnz_max} (clamped to ncols) -> rowptr[0..nrows], rowptr[0]=0.
 * Returns the total nnz.  Row r of the block is global row row_begin + r. */
int64_t nestgen_csr_rowptr(uint64_t seed, int64_t row_begin, int64_t nrows, int64_t ncols,
                           int32_t nnz_min, int32_t nnz_max, int64_t *rowptr) {
    if (nrows < 0 || nnz_min < 0 || nnz_max < nnz_min || !rowptr) return -1;
    rowptr[0] = 0;
#pragma omp parallel for schedule(static)
    for (int64_t r = 0; r < nrows; ++r) {
        int64_t len = ng_int(ng_draw(seed, NG_STREAM_ROWLEN, (uint64_t)(row_begin + r), 0),
                             nnz_min, nnz_max);
        if (len > ncols) len = ncols;
        rowptr[r + 1] = len;
    }
    for (int64_t r = 0; r < nrows; ++r) rowptr[r + 1] += rowptr[r];
    return rowptr[nrows];
}

static int ng_cmp_i32(const void *a, const void *b) {
    int32_t x = *(const int32_t *)a, y = *(const int32_t *)b;
    return (x > y) - (x < y);
}

/* Column indices (distinct within a row, ascending) and values for the rows
 * described by rowptr.  structure: NG_UNIFORM = uniform over [0,ncols);
 * NG_BANDED_FAR = with probability 1 - 1/far_den a column in
 * [gi-band_w, gi+band_w] ∩ [0,ncols), else uniform.  vkind/vlo/vhi select the
 * value distribution (NG_REAL_PM1 or NG_INT in [vlo,vhi]).  val may be NULL. */
int nestgen_csr_fill(uint64_t seed, int64_t row_begin, int64_t nrows, int64_t ncols,
                     int32_t structure, int64_t band_w, int32_t far_den,
                     int32_t vkind, int64_t vlo, int64_t vhi,
                     const int64_t *rowptr, int32_t *col, double *val) {
    if (nrows < 0 || ncols < 0 || !rowptr || (nrows > 0 && rowptr[nrows] > 0 && !col)) return -1;
#pragma omp parallel for schedule(dynamic, 4096)
    for (int64_t r = 0; r < nrows; ++r) {
        const int64_t gi = row_begin + r;
        const int64_t b = rowptr[r], len = rowptr[r + 1] - rowptr[r];
        int32_t *c = col + b;
        int64_t lo = gi - band_w, hi = gi + band_w;
        if (lo < 0) lo = 0;
        if (hi > ncols - 1) hi = ncols - 1;
        const int band_ok = (structure == NG_BANDED_FAR) && lo <= hi && (hi - lo + 1) >= 2 * len;
        uint64_t attempt = 0;
        for (int64_t k = 0; k < len;) {
            uint64_t u1 = ng_draw(seed, NG_STREAM_COL, (uint64_t)gi, 2 * attempt);
            uint64_t u2 = ng_draw(seed, NG_STREAM_COL, (uint64_t)gi, 2 * attempt + 1);
            ++attempt;
            int far = !band_ok || far_den <= 1 || ng_int(u1, 0, far_den - 1) == 0;
            int64_t cand = far ? ng_int(u2, 0, ncols - 1) : ng_int(u2, lo, hi);
            int dup = 0;
            for (int64_t q = 0; q < k; ++q)
                if (c[q] == (int32_t)cand) { dup = 1; break; }
            if (!dup) c[k++] = (int32_t)cand;
        }
        if (len < 48) {                       /* insertion sort: rows are short */
            for (int64_t p = 1; p < len; ++p) {
                int32_t v = c[p];
                int64_t q = p - 1;
                while (q >= 0 && c[q] > v) { c[q + 1] = c[q]; --q; }
                c[q + 1] = v;
            }
        } else {
            qsort(c, (size_t)len, sizeof(int32_t), ng_cmp_i32);
        }
        if (val)
            for (int64_t k = 0; k < len; ++k)
                val[b + k] = ng_f64(ng_draw(seed, NG_STREAM_VAL, (uint64_t)gi, (uint64_t)k), vkind, vlo, vhi);
    }
    return 0;
}

/* out[t] = draw(seed, stream, begin + t) mapped to the value distribution. */
int nestgen_vec_f64(uint64_t seed, uint64_t stream, int64_t begin, int64_t n,
                    int32_t vkind, int64_t vlo, int64_t vhi, double *out) {
    if (n < 0 || (n > 0 && !out)) return -1;
#pragma omp parallel for schedule(static)
    for (int64_t t = 0; t < n; ++t)
        out[t] = ng_f64(ng_draw(seed, stream, (uint64_t)(begin + t), 0), vkind, vlo, vhi);
    return 0;
}

int nestgen_vec_f32(uint64_t seed, uint64_t stream, int64_t begin, int64_t n,
                    int32_t vkind, int64_t vlo, int64_t vhi, float *out) {
    if (n < 0 || (n > 0 && !out)) return -1;
#pragma omp parallel for schedule(static)
    for (int64_t t = 0; t < n; ++t)
        out[t] = ng_f32(ng_draw(seed, stream, (uint64_t)(begin + t), 0), vkind, vlo, vhi);
    return 0;
}
