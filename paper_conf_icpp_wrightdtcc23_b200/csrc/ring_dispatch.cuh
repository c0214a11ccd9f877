// ring_dispatch.cuh -- Plan -> spmv_ring_kernel<S, MODE, OP, Body> (the x-ring
// SpMV, device/spmv_ring.cuh); instantiated per body in ring_*.cu.
#pragma once

#include "device/spmv_ring.cuh"
#include "internal.h"

namespace nest {

template <class Body, int S, int MODE, int OP>
nest_status ring_one(const Plan& p, const RingArgs& a, cudaStream_t st) {
    Body body{a.rowptr, a.col, a.val, XRing{a.x, nullptr, 0, 0u, 0u, (uint32_t)(a.nseg * kRingSeg)}, a.y,
              a.nnz};
    auto* k = p.ring_tps == 2 ? spmv_ring_kernel<S, MODE, OP, 2, Body> : spmv_ring_kernel<S, MODE, OP, 1, Body>;
    cudaError_t e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, p.smem_bytes);
    if (e != cudaSuccess) return cuda_fail(e, "cudaFuncSetAttribute(max dynamic smem)");
    e = launch_with_plan(p, k, dim3((unsigned)p.grid), dim3((unsigned)p.block), (size_t)p.smem_bytes, st, body, a);
    if (e != cudaSuccess) return cuda_fail(e, "spmv_ring launch");
    return NEST_OK;
}

template <class Body, int S, int MODE>
nest_status ring_op(const Plan& p, const RingArgs& a, cudaStream_t st) {
    switch (p.reduce) {
        case RED_SUM: return ring_one<Body, S, MODE, RED_SUM>(p, a, st);
        case RED_MAX: return ring_one<Body, S, MODE, RED_MAX>(p, a, st);
        case RED_MIN: return ring_one<Body, S, MODE, RED_MIN>(p, a, st);
    }
    return fail(NEST_ERR_INVALID_ARG, "reduce %d", p.reduce);
}

template <class Body, int S>
nest_status ring_mode(const Plan& p, const RingArgs& a, cudaStream_t st) {
    if constexpr (S == 1) {
        return ring_op<Body, 1, MODE_SPMD>(p, a, st);
    } else {
        switch (p.mode) {
            case MODE_SPMD: return ring_op<Body, S, MODE_SPMD>(p, a, st);
            case MODE_GENERIC_SMEM: return ring_op<Body, S, MODE_GENERIC_SMEM>(p, a, st);
            case MODE_GENERIC_SHFL: return ring_op<Body, S, MODE_GENERIC_SHFL>(p, a, st);
        }
    }
    return fail(NEST_ERR_INVALID_ARG, "mode %d", p.mode);
}

template <class Body>
nest_status ring_dispatch(const Plan& p, const RingArgs& a, cudaStream_t st) {
    switch (p.simdlen) {
        case 1: return ring_mode<Body, 1>(p, a, st);
        case 2: return ring_mode<Body, 2>(p, a, st);
        case 4: return ring_mode<Body, 4>(p, a, st);
        case 8: return ring_mode<Body, 8>(p, a, st);
        case 16: return ring_mode<Body, 16>(p, a, st);
        case 32: return ring_mode<Body, 32>(p, a, st);
    }
    return fail(NEST_ERR_INVALID_ARG, "simdlen %d", p.simdlen);
}

using RingScalar32 = SpmvBody<false, int32_t, XRing>;
using RingScalar64 = SpmvBody<false, int64_t, XRing>;
using RingPair32 = SpmvVecBody<false, 2, int32_t, XRing>;
using RingQuad32 = SpmvVecBody<false, 4, int32_t, XRing>;

nest_status ring_scalar32(const Plan& p, const RingArgs& a, cudaStream_t st);
nest_status ring_scalar64(const Plan& p, const RingArgs& a, cudaStream_t st);
nest_status ring_pair32(const Plan& p, const RingArgs& a, cudaStream_t st);
nest_status ring_quad32(const Plan& p, const RingArgs& a, cudaStream_t st);

}  // namespace nest
