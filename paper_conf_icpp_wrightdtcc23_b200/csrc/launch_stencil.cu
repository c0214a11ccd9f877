// launch_stencil.cu -- a10 nested stencil loop instantiations.
#include "dispatch.cuh"

namespace nest {

int32_t stencil_payload(int32_t U) {
    switch (U) {
        case 1: return payload_bytes<StencilBody, 1>();
        case 2: return payload_bytes<StencilBody, 2>();
        case 4: return payload_bytes<StencilBody, 4>();
    }
    return -1;
}

nest_status launch_stencil(const Plan& p, int64_t, int32_t L, const double* in, const double* coef,
                           const double* w, double* out, unsigned long long* visits,
                           unsigned char* fb, cudaStream_t st) {
    const StencilBody b{in, coef, w, out, visits, L};
    if (p.flags & NEST_F_VEC128) return dispatch(p, StencilVecBody{b}, fb, st);
    return dispatch(p, b, fb, st);
}

}  // namespace nest
