// launch_spmv.cu -- a8 CSR SpMV instantiations.
#include <cstdlib>

#include "dispatch.cuh"

namespace nest {

int32_t spmv_payload(int32_t U) {
    switch (U) {
        case 1: return payload_bytes<SpmvBody<false>, 1>();
        case 2: return payload_bytes<SpmvBody<false>, 2>();
        case 4: return payload_bytes<SpmvBody<false>, 4>();
    }
    return -1;
}

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
    if (hints) {
        SpmvBody<true> b{rowptr, col, val, x, y};
        b.nnz = nnz, b.pf_ahead = ahead, b.pf_len = len;
        return dispatch(p, b, fb, st);
    }
    SpmvBody<false> b{rowptr, col, val, x, y};
    b.nnz = nnz, b.pf_ahead = ahead, b.pf_len = len;
    return dispatch(p, b, fb, st);
}

}  // namespace nest
