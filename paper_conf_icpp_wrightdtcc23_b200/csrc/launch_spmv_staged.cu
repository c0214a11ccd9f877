// launch_spmv_staged.cu -- a8 CSR SpMV, warp-specialised bulk-copy pipeline
// (NEST_F_STAGED): planning of the stage sizes and the template dispatch.
#include "device/spmv_staged.cuh"
#include "internal.h"

namespace nest {

static constexpr int32_t kStagedMaxSmem = 227 * 1024;

// Stage sizes: with G consumer groups and R = G*U rows per chunk, pick the
// deepest pipeline (NS <= 4) whose stages hold >= 1.5x the chunk's expected
// nonzeros, else the largest stages at NS = 2; the x ring needs NS*R + 2H
// doubles (spmv_staged.cuh).  One team per SM (the stages fill shared memory).
nest_status plan_spmv_staged(Plan* p, int64_t nrows, int64_t nnz, int32_t sharing_bytes) {
    const int32_t T = p->block;
    const int32_t S = p->simdlen;
    const int32_t G = (T - 32) / S;
    if (G <= 0) return fail(NEST_ERR_INVALID_ARG, "NEST_F_STAGED: no consumer groups");
    const int32_t R = G * p->unroll;
    const bool smem_mode = p->mode == NEST_MODE_GENERIC_SMEM;
    p->groups = G;
    p->slot_bytes = (sharing_bytes / G) & ~7;   // even split, 8-byte aligned slots (R8)
    p->fallback = smem_mode && p->payload_bytes > p->slot_bytes;
    const int32_t sh = smem_mode ? p->slot_bytes * G : 0;
    const double avg = nrows > 0 ? (double)nnz / (double)nrows : 0.0;
    const int64_t want = (int64_t)(1.5 * avg * R) + 16;
    int32_t best_ns = 0, best_nb = 0, best_xw = 0;
    for (int32_t ns = 4; ns >= 2; --ns) {
        int64_t xw = p->x_halo > 0 ? (int64_t)ns * R + 2 * (int64_t)p->x_halo : 0;
        xw = (xw + 1) & ~(int64_t)1;
        // bytes without the nonzero buffers, then the largest NB (multiple of 4) that fits
        const StagedLayout l0 = staged_layout((int32_t)xw, 0, ns, R, sh);
        const int64_t room = (int64_t)kStagedMaxSmem - (int64_t)l0.total;
        if (room <= 0) continue;
        int64_t nb = (room / ns) / 12;
        nb &= ~(int64_t)3;
        while (nb > 0 && staged_layout((int32_t)xw, (int32_t)nb, ns, R, sh).total > (uint32_t)kStagedMaxSmem) nb -= 4;
        if (nb < 4) continue;
        if (nb > (1 << 20)) nb = 1 << 20;
        if (nb >= want || ns == 2) {
            if (nb > best_nb || nb >= want) {
                best_ns = ns;
                best_nb = (int32_t)nb;
                best_xw = (int32_t)xw;
            }
            if (nb >= want) break;
        }
    }
    if (best_ns == 0)
        return fail(NEST_ERR_UNSUPPORTED,
                    "NEST_F_STAGED: x_halo %d with %d rows per chunk does not fit shared memory", p->x_halo, R);
    p->ns = best_ns;
    p->nb = best_nb;
    p->xw = best_xw;
    p->smem_bytes = (int32_t)staged_layout(best_xw, best_nb, best_ns, R, sh).total;
    if (p->grid <= 0) {
        int64_t resident = 0;
        nest_status s = resident_blocks(T, p->smem_bytes, &resident);
        if (s != NEST_OK) return s;
        const int64_t needed = (nrows + R - 1) / R;
        p->grid = (int32_t)(needed < resident ? (needed > 0 ? needed : 1) : resident);
    }
    return NEST_OK;
}

template <int S, int MODE, int OP, int U>
static nest_status staged_one(const Plan& p, const StagedArgs& a, cudaStream_t st) {
    auto* k = spmv_staged_kernel<S, MODE, OP, U>;
    cudaError_t e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, p.smem_bytes);
    if (e != cudaSuccess) return cuda_fail(e, "cudaFuncSetAttribute(max dynamic smem)");
    k<<<p.grid, p.block, p.smem_bytes, st>>>(a);
    e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_fail(e, "spmv_staged launch");
    return NEST_OK;
}

template <int S, int MODE, int U>
static nest_status staged_op(const Plan& p, const StagedArgs& a, cudaStream_t st) {
    switch (p.reduce) {
        case RED_SUM: return staged_one<S, MODE, RED_SUM, U>(p, a, st);
        case RED_MAX: return staged_one<S, MODE, RED_MAX, U>(p, a, st);
        case RED_MIN: return staged_one<S, MODE, RED_MIN, U>(p, a, st);
    }
    return fail(NEST_ERR_INVALID_ARG, "reduce %d", p.reduce);
}

template <int S, int U>
static nest_status staged_mode(const Plan& p, const StagedArgs& a, cudaStream_t st) {
    if constexpr (S == 1) {
        return staged_op<1, MODE_SPMD, U>(p, a, st);
    } else {
        switch (p.mode) {
            case MODE_SPMD: return staged_op<S, MODE_SPMD, U>(p, a, st);
            case MODE_GENERIC_SMEM: return staged_op<S, MODE_GENERIC_SMEM, U>(p, a, st);
            case MODE_GENERIC_SHFL: return staged_op<S, MODE_GENERIC_SHFL, U>(p, a, st);
        }
    }
    return fail(NEST_ERR_INVALID_ARG, "mode %d", p.mode);
}

template <int U>
static nest_status staged_simdlen(const Plan& p, const StagedArgs& a, cudaStream_t st) {
    switch (p.simdlen) {
        case 1: return staged_mode<1, U>(p, a, st);
        case 2: return staged_mode<2, U>(p, a, st);
        case 4: return staged_mode<4, U>(p, a, st);
        case 8: return staged_mode<8, U>(p, a, st);
        case 16: return staged_mode<16, U>(p, a, st);
        case 32: return staged_mode<32, U>(p, a, st);
    }
    return fail(NEST_ERR_INVALID_ARG, "simdlen %d", p.simdlen);
}

nest_status launch_spmv_staged(const Plan& p, int64_t nrows, int64_t ncols, int64_t nnz,
                               const int64_t* rowptr, const int32_t* col, const double* val,
                               const double* x, double* y, unsigned char* fb, cudaStream_t st) {
    const StagedArgs a{rowptr, col, val, x, y, nrows, ncols, nnz, p.x_halo, p.xw, p.nb, p.ns,
                       p.slot_bytes, fb};
    switch (p.unroll) {
        case 1: return staged_simdlen<1>(p, a, st);
        case 2: return staged_simdlen<2>(p, a, st);
        case 4: return staged_simdlen<4>(p, a, st);
    }
    return fail(NEST_ERR_INVALID_ARG, "outer_unroll %d", p.unroll);
}

}  // namespace nest
