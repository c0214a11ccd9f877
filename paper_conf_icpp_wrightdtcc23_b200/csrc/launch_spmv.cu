// launch_spmv.cu -- a8 CSR SpMV: body selection (scalar / 128-bit pairs / quads,
// 32- or 64-bit indices) for nest_kernel; the instantiations live in spmv_*.cu.
#include "spmv_variants.h"

namespace nest {

int32_t spmv_payload(int32_t U) {
    switch (U) {
        case 1: return payload_bytes<SpmvBody<false, int64_t>, 1>();
        case 2: return payload_bytes<SpmvBody<false, int64_t>, 2>();
        case 4: return payload_bytes<SpmvBody<false, int64_t>, 4>();
    }
    return -1;
}

template <class Body>
static int32_t payload_u(int32_t U) {
    switch (U) {
        case 1: return payload_bytes<Body, 1>();
        case 2: return payload_bytes<Body, 2>();
        case 4: return payload_bytes<Body, 4>();
    }
    return -1;
}

// The generic payload of the body launch_spmv runs (the same selection as below).
int32_t spmv_body_payload(const Plan& p, int64_t nnz) {
    const bool i32 = spmv_index32(p, nnz);
    static_assert(sizeof(SpmvVecBody<false, 2, int32_t>::Loop) == sizeof(SpmvVecBody<false, 4, int32_t>::Loop), "");
    if (p.flags & NEST_F_VEC128)
        return i32 ? payload_u<SpmvVecBody<false, 2, int32_t>>(p.unroll) : payload_u<SpmvVecBody<false, 2, int64_t>>(p.unroll);
    return i32 ? payload_u<SpmvBody<false, int32_t>>(p.unroll) : payload_u<SpmvBody<false, int64_t>>(p.unroll);
}

nest_status launch_spmv(const Plan& p, bool hints, int64_t nrows, const int64_t* rowptr,
                        const int32_t* col, const double* val, const double* x, double* y,
                        unsigned char* fb, cudaStream_t st, int64_t nnz) {
    (void)nrows;
    // 32-bit row / nonzero indices when they fit (fewer registers)
    const bool i32 = spmv_index32(p, nnz);
    if (p.flags & NEST_F_VEC128) {
        if (p.flags & NEST_F_VEC_QUAD) {
            if (i32) return spmv_dispatch(p, SpmvVecBody<false, 4, int32_t>{rowptr, col, val, x, y, nnz}, fb, st);
            return spmv_dispatch(p, SpmvVecBody<false, 4, int64_t>{rowptr, col, val, x, y, nnz}, fb, st);
        }
        if (hints && i32) return spmv_dispatch(p, SpmvVecBody<true, 2, int32_t>{rowptr, col, val, x, y, nnz}, fb, st);
        if (i32) return spmv_dispatch(p, SpmvVecBody<false, 2, int32_t>{rowptr, col, val, x, y, nnz}, fb, st);
        return spmv_dispatch(p, SpmvVecBody<false, 2, int64_t>{rowptr, col, val, x, y, nnz}, fb, st);
    }
    if (i32) {
        if (hints) return spmv_dispatch(p, SpmvBody<true, int32_t>{rowptr, col, val, x, y, nnz}, fb, st);
        return spmv_dispatch(p, SpmvBody<false, int32_t>{rowptr, col, val, x, y, nnz}, fb, st);
    }
    if (hints) return spmv_dispatch(p, SpmvBody<true, int64_t>{rowptr, col, val, x, y, nnz}, fb, st);
    return spmv_dispatch(p, SpmvBody<false, int64_t>{rowptr, col, val, x, y, nnz}, fb, st);
}

}  // namespace nest
