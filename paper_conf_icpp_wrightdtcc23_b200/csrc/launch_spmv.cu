// launch_spmv.cu -- a8 CSR SpMV instantiations.
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

nest_status launch_spmv(const Plan& p, bool hints, int64_t, const int64_t* rowptr,
                        const int32_t* col, const double* val, const double* x, double* y,
                        unsigned char* fb, cudaStream_t st) {
    if (hints) return dispatch(p, SpmvBody<true>{rowptr, col, val, x, y}, fb, st);
    return dispatch(p, SpmvBody<false>{rowptr, col, val, x, y}, fb, st);
}

}  // namespace nest
