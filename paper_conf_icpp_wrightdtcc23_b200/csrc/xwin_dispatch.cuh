// xwin_dispatch.cuh -- Plan -> spmv_xwin_kernel<S, MODE, OP, U, Body>.
#pragma once

#include "device/spmv_xwin.cuh"
#include "internal.h"

namespace nest {

template <class Body, int S, int MODE, int OP, int U>
nest_status xwin_one(const Plan& p, const XwinArgs& a, cudaStream_t st) {
    auto* k = spmv_xwin_kernel<S, MODE, OP, U, Body>;
    // opt in to > 48 KB of dynamic shared memory (idempotent, cheap)
    cudaError_t e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, p.smem_bytes);
    if (e != cudaSuccess) return cuda_fail(e, "cudaFuncSetAttribute(max dynamic smem)");
    k<<<p.grid, p.block, p.smem_bytes, st>>>(a);
    e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_fail(e, "spmv_xwin launch");
    return NEST_OK;
}

template <class Body, int S, int MODE, int U>
nest_status xwin_op(const Plan& p, const XwinArgs& a, cudaStream_t st) {
    switch (p.reduce) {
        case RED_SUM: return xwin_one<Body, S, MODE, RED_SUM, U>(p, a, st);
        case RED_MAX: return xwin_one<Body, S, MODE, RED_MAX, U>(p, a, st);
        case RED_MIN: return xwin_one<Body, S, MODE, RED_MIN, U>(p, a, st);
    }
    return fail(NEST_ERR_INVALID_ARG, "reduce %d", p.reduce);
}

template <class Body, int S, int U>
nest_status xwin_mode(const Plan& p, const XwinArgs& a, cudaStream_t st) {
    if constexpr (S == 1) {
        return xwin_op<Body, 1, MODE_SPMD, U>(p, a, st);
    } else {
        switch (p.mode) {
            case MODE_SPMD: return xwin_op<Body, S, MODE_SPMD, U>(p, a, st);
            case MODE_GENERIC_SMEM: return xwin_op<Body, S, MODE_GENERIC_SMEM, U>(p, a, st);
            case MODE_GENERIC_SHFL: return xwin_op<Body, S, MODE_GENERIC_SHFL, U>(p, a, st);
        }
    }
    return fail(NEST_ERR_INVALID_ARG, "mode %d", p.mode);
}

template <class Body, int U>
nest_status xwin_simdlen(const Plan& p, const XwinArgs& a, cudaStream_t st) {
    switch (p.simdlen) {
        case 1: return xwin_mode<Body, 1, U>(p, a, st);
        case 2: return xwin_mode<Body, 2, U>(p, a, st);
        case 4: return xwin_mode<Body, 4, U>(p, a, st);
        case 8: return xwin_mode<Body, 8, U>(p, a, st);
        case 16: return xwin_mode<Body, 16, U>(p, a, st);
        case 32: return xwin_mode<Body, 32, U>(p, a, st);
    }
    return fail(NEST_ERR_INVALID_ARG, "simdlen %d", p.simdlen);
}

template <class Body>
nest_status xwin_dispatch(const Plan& p, const XwinArgs& a, cudaStream_t st) {
    switch (p.unroll) {
        case 1: return xwin_simdlen<Body, 1>(p, a, st);
        case 2: return xwin_simdlen<Body, 2>(p, a, st);
        case 4: return xwin_simdlen<Body, 4>(p, a, st);
    }
    return fail(NEST_ERR_INVALID_ARG, "outer_unroll %d", p.unroll);
}

}  // namespace nest
