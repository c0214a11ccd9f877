// launch_spmv_xwin.cu -- a8 CSR SpMV with the shared-memory x window
// (spmv_xwin.cuh), scalar loads; the 128-bit pair body is in
// launch_spmv_xwin_vec.cu (separate translation units compile in parallel).
#include "xwin_dispatch.cuh"

namespace nest {

nest_status launch_spmv_xwin_vec(const Plan& p, const XwinArgs& a, cudaStream_t st);

nest_status launch_spmv_xwin(const Plan& p, int64_t nrows, int64_t ncols, int64_t nnz, const int64_t* rowptr,
                             const int32_t* col, const double* val, const double* x, double* y,
                             unsigned char* fb, cudaStream_t st) {
    const XwinArgs a{rowptr, col, val, x, y, nrows, ncols, nnz, p.x_halo, p.xw, p.kb, p.slot_bytes, fb};
    if (p.flags & NEST_F_VEC128) return launch_spmv_xwin_vec(p, a, st);
    return xwin_dispatch<SpmvBody<false, false, int64_t, XWindow>>(p, a, st);
}

}  // namespace nest
