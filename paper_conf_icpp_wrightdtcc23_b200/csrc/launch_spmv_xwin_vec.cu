// launch_spmv_xwin_vec.cu -- the x-window SpMV with 128-bit pair loads.
#include "xwin_dispatch.cuh"

namespace nest {

nest_status launch_spmv_xwin_vec(const Plan& p, const XwinArgs& a, cudaStream_t st) {
    return xwin_dispatch<SpmvVecBody<false, 2, int32_t, XWindow>>(p, a, st);
}

}  // namespace nest
