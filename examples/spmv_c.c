/* examples/spmv_c.c -- the C ABI used from plain C (no Python, no torch): a small
 * banded CSR matrix, y = A x through nest_spmv_csr_f64 in the bench headline's
 * configuration (simdlen 2, SPMD, blocked teams of 1024, quad tuples, x persisting
 * in L2) and in generic-SMEM mode at simdlen 8, each checked against a plain C loop
 * on integer-valued data (exact in fp64, so the comparison is bit for bit).
 *
 *   make examples/spmv_c        (links libnest.so and the CUDA runtime)
 *   ./examples/spmv_c           (needs a GPU; exit status 0 = all checks passed)
 */
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include "nest.h"

#define CHECK_CUDA(x)                                                          \
    do {                                                                       \
        cudaError_t e_ = (x);                                                  \
        if (e_ != cudaSuccess) {                                               \
            fprintf(stderr, "%s: %s\n", #x, cudaGetErrorString(e_));           \
            return 2;                                                          \
        }                                                                      \
    } while (0)
#define CHECK_NEST(x)                                                          \
    do {                                                                       \
        nest_status s_ = (x);                                                  \
        if (s_ != NEST_OK) {                                                   \
            fprintf(stderr, "%s: %s: %s\n", #x, nest_status_str(s_), nest_last_error()); \
            return 3;                                                          \
        }                                                                      \
    } while (0)

static uint64_t mix(uint64_t z) {
    z += 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

int main(void) {
    const int64_t n = 100003;   /* rows = columns; several teams, a ragged tail */
    int64_t* rowptr = malloc((size_t)(n + 1) * sizeof *rowptr);
    rowptr[0] = 0;
    for (int64_t i = 0; i < n; ++i) rowptr[i + 1] = rowptr[i] + 4 + (int64_t)(mix((uint64_t)i) % 9);
    const int64_t nnz = rowptr[n];
    int32_t* col = malloc((size_t)nnz * sizeof *col);
    double* val = malloc((size_t)nnz * sizeof *val);
    double* x = malloc((size_t)n * sizeof *x);
    double* y = malloc((size_t)n * sizeof *y);
    double* yref = malloc((size_t)n * sizeof *yref);
    for (int64_t i = 0; i < n; ++i) {   /* sorted distinct columns in a band around i */
        const int64_t len = rowptr[i + 1] - rowptr[i];
        int64_t c = i - 40 < 0 ? 0 : i - 40;
        for (int64_t k = 0; k < len; ++k) {
            c += 1 + (int64_t)(mix((uint64_t)(i * 31 + k)) % 8);
            col[rowptr[i] + k] = (int32_t)(c % n);
            val[rowptr[i] + k] = (double)((int64_t)(mix((uint64_t)(i * 17 + k)) % 9) - 4);
        }
    }
    for (int64_t j = 0; j < n; ++j) x[j] = (double)((int64_t)(mix((uint64_t)j + 7) % 17) - 8);
    for (int64_t i = 0; i < n; ++i) {   /* the reference: the loop nest in storage order */
        double s = 0.0;
        for (int64_t k = rowptr[i]; k < rowptr[i + 1]; ++k) s += val[k] * x[col[k]];
        yref[i] = s;
    }

    int64_t* d_rowptr;
    int32_t* d_col;
    double *d_val, *d_x, *d_y;
    CHECK_CUDA(cudaMalloc((void**)&d_rowptr, (size_t)(n + 1) * sizeof *d_rowptr));
    CHECK_CUDA(cudaMalloc((void**)&d_col, (size_t)nnz * sizeof *d_col));
    CHECK_CUDA(cudaMalloc((void**)&d_val, (size_t)nnz * sizeof *d_val));
    CHECK_CUDA(cudaMalloc((void**)&d_x, (size_t)n * sizeof *d_x));
    CHECK_CUDA(cudaMalloc((void**)&d_y, (size_t)n * sizeof *d_y));
    CHECK_CUDA(cudaMemcpy(d_rowptr, rowptr, (size_t)(n + 1) * sizeof *rowptr, cudaMemcpyHostToDevice));
    CHECK_CUDA(cudaMemcpy(d_col, col, (size_t)nnz * sizeof *col, cudaMemcpyHostToDevice));
    CHECK_CUDA(cudaMemcpy(d_val, val, (size_t)nnz * sizeof *val, cudaMemcpyHostToDevice));
    CHECK_CUDA(cudaMemcpy(d_x, x, (size_t)n * sizeof *x, cudaMemcpyHostToDevice));

    nest_desc runs[2];
    memset(runs, 0, sizeof runs);
    runs[0].abi_version = NEST_ABI_VERSION;   /* the bench headline */
    runs[0].simdlen = 2;
    runs[0].threads_per_team = 1024;
    runs[0].mode = NEST_MODE_SPMD;
    runs[0].flags = NEST_F_BLOCKED | NEST_F_VEC128 | NEST_F_VEC_QUAD | NEST_F_X_L2_PERSIST;
    runs[1].abi_version = NEST_ABI_VERSION;   /* the paper's generic mode, sharing space in smem */
    runs[1].simdlen = 8;
    runs[1].mode = NEST_MODE_GENERIC_SMEM;
    int bad = 0;
    for (int r = 0; r < 2; ++r) {
        nest_plan_info info;
        CHECK_NEST(nest_spmv_plan(&runs[r], n, n, nnz, &info));
        CHECK_CUDA(cudaMemset(d_y, 0xff, (size_t)n * sizeof *d_y));
        CHECK_NEST(nest_spmv_csr_f64(&runs[r], n, n, nnz, d_rowptr, d_col, d_val, d_x, d_y, NULL));
        CHECK_CUDA(cudaMemcpy(y, d_y, (size_t)n * sizeof *y, cudaMemcpyDeviceToHost));
        int64_t mism = 0;
        for (int64_t i = 0; i < n; ++i) mism += memcmp(&y[i], &yref[i], sizeof(double)) != 0;
        printf("run %d: simdlen %d mode %d grid %d x %d, %d-bit indices: %lld mismatching rows of %lld\n", r,
               runs[r].simdlen, runs[r].mode, info.grid, info.block, info.index_bits, (long long)mism,
               (long long)n);
        bad += mism != 0;
    }
    CHECK_NEST(nest_shutdown());
    cudaFree(d_rowptr), cudaFree(d_col), cudaFree(d_val), cudaFree(d_x), cudaFree(d_y);
    free(rowptr), free(col), free(val), free(x), free(y), free(yref);
    return bad ? 1 : 0;
}
