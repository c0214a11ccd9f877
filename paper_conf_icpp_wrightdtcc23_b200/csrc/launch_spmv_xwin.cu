// launch_spmv_xwin.cu -- a8 CSR SpMV with the shared-memory x window.
#include "device/spmv_xwin.cuh"
#include "internal.h"

namespace nest {

template <int S, int MODE, int OP, int U>
static nest_status xwin_one(const Plan& p, const XwinArgs& a, cudaStream_t st) {
    auto* k = spmv_xwin_kernel<S, MODE, OP, U, false>;
    // opt in to > 48 KB of dynamic shared memory (idempotent, cheap)
    cudaError_t e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, p.smem_bytes);
    if (e != cudaSuccess) return cuda_fail(e, "cudaFuncSetAttribute(max dynamic smem)");
    k<<<p.grid, p.block, p.smem_bytes, st>>>(a);
    e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_fail(e, "spmv_xwin launch");
    return NEST_OK;
}

template <int S, int MODE, int U>
static nest_status xwin_op(const Plan& p, const XwinArgs& a, cudaStream_t st) {
    switch (p.reduce) {
        case RED_SUM: return xwin_one<S, MODE, RED_SUM, U>(p, a, st);
        case RED_MAX: return xwin_one<S, MODE, RED_MAX, U>(p, a, st);
        case RED_MIN: return xwin_one<S, MODE, RED_MIN, U>(p, a, st);
    }
    return fail(NEST_ERR_INVALID_ARG, "reduce %d", p.reduce);
}

template <int S, int U>
static nest_status xwin_mode(const Plan& p, const XwinArgs& a, cudaStream_t st) {
    if constexpr (S == 1) {
        return xwin_op<1, MODE_SPMD, U>(p, a, st);
    } else {
        switch (p.mode) {
            case MODE_SPMD: return xwin_op<S, MODE_SPMD, U>(p, a, st);
            case MODE_GENERIC_SMEM: return xwin_op<S, MODE_GENERIC_SMEM, U>(p, a, st);
            case MODE_GENERIC_SHFL: return xwin_op<S, MODE_GENERIC_SHFL, U>(p, a, st);
        }
    }
    return fail(NEST_ERR_INVALID_ARG, "mode %d", p.mode);
}

template <int U>
static nest_status xwin_simdlen(const Plan& p, const XwinArgs& a, cudaStream_t st) {
    switch (p.simdlen) {
        case 1: return xwin_mode<1, U>(p, a, st);
        case 2: return xwin_mode<2, U>(p, a, st);
        case 4: return xwin_mode<4, U>(p, a, st);
        case 8: return xwin_mode<8, U>(p, a, st);
        case 16: return xwin_mode<16, U>(p, a, st);
        case 32: return xwin_mode<32, U>(p, a, st);
    }
    return fail(NEST_ERR_INVALID_ARG, "simdlen %d", p.simdlen);
}

nest_status launch_spmv_xwin(const Plan& p, int64_t nrows, int64_t ncols, const int64_t* rowptr,
                             const int32_t* col, const double* val, const double* x, double* y,
                             unsigned char* fb, cudaStream_t st) {
    const XwinArgs a{rowptr, col, val, x, y, nrows, ncols, p.x_halo, p.xw, p.slot_bytes, fb};
    switch (p.unroll) {
        case 1: return xwin_simdlen<1>(p, a, st);
        case 2: return xwin_simdlen<2>(p, a, st);
        case 4: return xwin_simdlen<4>(p, a, st);
    }
    return fail(NEST_ERR_INVALID_ARG, "outer_unroll %d", p.unroll);
}

}  // namespace nest
