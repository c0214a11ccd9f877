// dispatch.cuh -- host-side template dispatch from a runtime Plan to one
// kernel instantiation nest_kernel<S, MODE, OP, U, Body>.  This is the B200
// analogue of the paper's if-cascade over known outlined regions
// (PAPER.md:794-800): every (simdlen, mode, reduction, unroll, body) is a
// compile-time variant, so the hot loop has no indirect call.
#pragma once

#include "bodies/bodies.cuh"
#include "internal.h"

namespace nest {

template <class Body, int U, int S, int MODE, int OP>
constexpr auto kernel_of() {
    if constexpr (U == 1 && two_teams_per_sm<Body, S>::value) return nest_kernel_2pm<S, MODE, OP, U, Body>;
    else return nest_kernel<S, MODE, OP, U, Body>;
}

template <class Body, int U, int S, int MODE, int OP>
nest_status launch_one(const Plan& p, const Body& body, unsigned char* fb, cudaStream_t st) {
    constexpr auto kern = kernel_of<Body, U, S, MODE, OP>();
    // a team size the instantiation cannot run (registers) is reported before launching
    static int max_threads = 0;
    if (max_threads == 0) {
        cudaFuncAttributes fa;
        if (cudaFuncGetAttributes(&fa, kern) == cudaSuccess)
            max_threads = fa.maxThreadsPerBlock;
        else
            cudaGetLastError();
    }
    if (max_threads > 0 && p.block > max_threads)
        return fail(NEST_ERR_UNSUPPORTED,
                    "threads_per_team %d exceeds this variant's limit of %d (registers); use a smaller team or "
                    "outer_unroll", p.block, max_threads);
    if (p.smem_bytes > 48 * 1024) {
        const cudaError_t e = cudaFuncSetAttribute(kern,
                                                   cudaFuncAttributeMaxDynamicSharedMemorySize, p.smem_bytes);
        if (e != cudaSuccess) return cuda_fail(e, "cudaFuncSetAttribute(max dynamic smem)");
    }
    const int64_t chunk = (p.flags & NEST_F_BLOCKED) ? p.chunk : 0;
    const cudaError_t e = launch_with_plan(p, kern, dim3((unsigned)p.grid), dim3((unsigned)p.block),
                                           (size_t)p.smem_bytes, st, body, p.outer, p.slot_bytes, fb, chunk);
    if (e != cudaSuccess) return cuda_fail(e, "kernel launch");
    return NEST_OK;
}

template <class Body, int U, int S, int MODE>
nest_status dispatch_op(const Plan& p, const Body& b, unsigned char* fb, cudaStream_t st) {
    switch (p.reduce) {
        case RED_SUM: return launch_one<Body, U, S, MODE, RED_SUM>(p, b, fb, st);
        case RED_MAX: return launch_one<Body, U, S, MODE, RED_MAX>(p, b, fb, st);
        case RED_MIN: return launch_one<Body, U, S, MODE, RED_MIN>(p, b, fb, st);
    }
    return fail(NEST_ERR_INVALID_ARG, "reduce %d", p.reduce);
}

template <class Body, int U, int S>
nest_status dispatch_mode(const Plan& p, const Body& b, unsigned char* fb, cudaStream_t st) {
    if constexpr (S == 1) {
        return dispatch_op<Body, U, 1, MODE_SPMD>(p, b, fb, st);
    } else {
        switch (p.mode) {
            case MODE_SPMD: return dispatch_op<Body, U, S, MODE_SPMD>(p, b, fb, st);
            case MODE_GENERIC_SMEM: return dispatch_op<Body, U, S, MODE_GENERIC_SMEM>(p, b, fb, st);
            case MODE_GENERIC_SHFL: return dispatch_op<Body, U, S, MODE_GENERIC_SHFL>(p, b, fb, st);
        }
    }
    return fail(NEST_ERR_INVALID_ARG, "mode %d", p.mode);
}

template <class Body, int U>
nest_status dispatch_simdlen(const Plan& p, const Body& b, unsigned char* fb, cudaStream_t st) {
    switch (p.simdlen) {
        case 1: return dispatch_mode<Body, U, 1>(p, b, fb, st);
        case 2: return dispatch_mode<Body, U, 2>(p, b, fb, st);
        case 4: return dispatch_mode<Body, U, 4>(p, b, fb, st);
        case 8: return dispatch_mode<Body, U, 8>(p, b, fb, st);
        case 16: return dispatch_mode<Body, U, 16>(p, b, fb, st);
        case 32: return dispatch_mode<Body, U, 32>(p, b, fb, st);
    }
    return fail(NEST_ERR_INVALID_ARG, "simdlen %d", p.simdlen);
}

template <class Body>
nest_status dispatch(const Plan& p, const Body& b, unsigned char* fb, cudaStream_t st) {
    switch (p.unroll) {
        case 1: return dispatch_simdlen<Body, 1>(p, b, fb, st);
        case 2: return dispatch_simdlen<Body, 2>(p, b, fb, st);
        case 4: return dispatch_simdlen<Body, 4>(p, b, fb, st);
    }
    return fail(NEST_ERR_INVALID_ARG, "outer_unroll %d", p.unroll);
}

}  // namespace nest
