// launch_laplace.cu -- NEXT-2 laplace3d (non-reducing simd loops) instantiations.
#include "dispatch.cuh"

namespace nest {

int32_t laplace_payload(int32_t U) {
    switch (U) {
        case 1: return payload_bytes<LaplaceBody, 1>();
        case 2: return payload_bytes<LaplaceBody, 2>();
        case 4: return payload_bytes<LaplaceBody, 4>();
    }
    return -1;
}

nest_status launch_laplace(const Plan& p, int64_t nz, int64_t ny, int64_t nx, double alpha, const double* u,
                           double* out, unsigned char* fb, cudaStream_t st) {
    (void)nz;
    const LaplaceBody b{u, out, ny, nx, alpha};
    if (p.flags & NEST_F_VEC128) return dispatch(p, LaplaceVecBody{b}, fb, st);
    return dispatch(p, b, fb, st);
}

}  // namespace nest
