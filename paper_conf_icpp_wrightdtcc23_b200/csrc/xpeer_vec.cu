// xpeer_vec.cu -- NEXT-4 peer-gather SpMV instantiations, 128-bit pair loads
// (separate translation unit: compiles in parallel with xpeer.cu).
#include "dispatch.cuh"

namespace nest {

nest_status launch_spmv_xpeer_vec(const Plan& p, const int64_t* rowptr, const int32_t* col, const double* val,
                                  XPeer xa, double* y, unsigned char* fb, cudaStream_t st, int64_t nnz) {
    return dispatch(p, SpmvVecBody<false, 2, int32_t, XPeer>{rowptr, col, val, xa, y, nnz}, fb, st);
}

}  // namespace nest
