// launch_spmv.cu -- a8 CSR SpMV instantiations.
#include <cstdlib>

#include "spmv_variants.h"

namespace nest {

int32_t spmv_payload(int32_t U) {
    switch (U) {
        case 1: return payload_bytes<SpmvBody<false, false, int64_t>, 1>();
        case 2: return payload_bytes<SpmvBody<false, false, int64_t>, 2>();
        case 4: return payload_bytes<SpmvBody<false, false, int64_t>, 4>();
    }
    return -1;
}

nest_status launch_spmv_body(const Plan& p, bool hints, const int64_t* rowptr, const int32_t* col,
                             const double* val, const double* x, double* y, unsigned char* fb,
                             cudaStream_t st, int64_t nnz, int64_t ahead, int64_t len);

nest_status launch_spmv(const Plan& p, bool hints, int64_t nrows, const int64_t* rowptr,
                        const int32_t* col, const double* val, const double* x, double* y,
                        unsigned char* fb, cudaStream_t st, int64_t nnz) {
    // blocked schedule: the team leader L2-prefetches `rounds` rounds of G*U rows ahead
    static const int rounds = [] {
        const char* e = std::getenv("NEST_L2PF_ROUNDS");
        return e ? std::atoi(e) : 0;   // measured: L2 prefetch hurts on B200
    }();
    int64_t ahead = 0, len = 0;
    if ((p.flags & NEST_F_BLOCKED) && rounds > 0 && nrows > 0) {
        const double avg = (double)nnz / (double)nrows;
        len = (int64_t)(avg * p.groups * p.unroll) + 4;
        ahead = len * rounds;
    }
    // loop-bound pipeline: 3 rounds x U x 16 B per thread after the sharing space
    static const int pipe = [] {
        const char* e = std::getenv("NEST_RP_PIPE");
        return e ? std::atoi(e) : 0;
    }();
    Plan q = p;
    if (pipe) {
        q.pipe_off = (p.smem_bytes + 15) & ~15;
        q.smem_bytes = q.pipe_off + 3 * p.unroll * p.block * 16;
    }
    return launch_spmv_body(q, hints, rowptr, col, val, x, y, fb, st, nnz, ahead, len);
}

template <bool HINTS, bool PIPE>
static nest_status launch_spmv_t(const Plan& p, const int64_t* rowptr, const int32_t* col, const double* val,
                                 const double* x, double* y, unsigned char* fb, cudaStream_t st, int64_t nnz,
                                 int64_t ahead, int64_t len) {
    // 32-bit row / nonzero indices when they fit (fewer registers)
    if (spmv_index32(p, nnz)) {
        SpmvBody<HINTS, PIPE, int32_t> b{rowptr, col, val, x, y};
        b.nnz = nnz, b.pf_ahead = ahead, b.pf_len = len;
        return spmv_dispatch(p, b, fb, st);
    }
    SpmvBody<HINTS, PIPE, int64_t> b{rowptr, col, val, x, y};
    b.nnz = nnz, b.pf_ahead = ahead, b.pf_len = len;
    return spmv_dispatch(p, b, fb, st);
}

nest_status launch_spmv_body(const Plan& p, bool hints, const int64_t* rowptr, const int32_t* col,
                             const double* val, const double* x, double* y, unsigned char* fb,
                             cudaStream_t st, int64_t nnz, int64_t ahead, int64_t len) {
    const bool pipe = p.pipe_off >= 0;
    if (p.flags & NEST_F_VEC128) {
        // 32-bit row / nonzero indices when they fit (fewer registers)
        const bool i32 = spmv_index32(p, nnz);
        if (p.flags & NEST_F_VEC_QUAD) {
            if (i32) return spmv_dispatch(p, SpmvVecBody<false, 4, int32_t>{rowptr, col, val, x, y, nnz}, fb, st);
            return spmv_dispatch(p, SpmvVecBody<false, 4, int64_t>{rowptr, col, val, x, y, nnz}, fb, st);
        }
        if (hints && i32) return spmv_dispatch(p, SpmvVecBody<true, 2, int32_t>{rowptr, col, val, x, y, nnz}, fb, st);
        if (i32) return spmv_dispatch(p, SpmvVecBody<false, 2, int32_t>{rowptr, col, val, x, y, nnz}, fb, st);
        return spmv_dispatch(p, SpmvVecBody<false, 2, int64_t>{rowptr, col, val, x, y, nnz}, fb, st);
    }
    if (hints) {
        if (pipe) return launch_spmv_t<true, true>(p, rowptr, col, val, x, y, fb, st, nnz, ahead, len);
        return launch_spmv_t<true, false>(p, rowptr, col, val, x, y, fb, st, nnz, ahead, len);
    }
    if (pipe) return launch_spmv_t<false, true>(p, rowptr, col, val, x, y, fb, st, nnz, ahead, len);
    return launch_spmv_t<false, false>(p, rowptr, col, val, x, y, fb, st, nnz, ahead, len);
}

}  // namespace nest
