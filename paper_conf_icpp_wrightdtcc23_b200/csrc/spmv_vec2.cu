// spmv_vec2.cu -- SpMV instantiations: 128-bit pair loads.
#include "dispatch.cuh"
#include "spmv_variants.h"

namespace nest {

template <class Body>
nest_status spmv_dispatch(const Plan& p, const Body& body, unsigned char* fb, cudaStream_t st) {
    return dispatch(p, body, fb, st);
}

template nest_status spmv_dispatch<SpmvVecBody<true, 2, int32_t>>(const Plan&, const SpmvVecBody<true, 2, int32_t>&, unsigned char*, cudaStream_t);
template nest_status spmv_dispatch<SpmvVecBody<false, 2, int32_t>>(const Plan&, const SpmvVecBody<false, 2, int32_t>&, unsigned char*, cudaStream_t);
template nest_status spmv_dispatch<SpmvVecBody<false, 2, int64_t>>(const Plan&, const SpmvVecBody<false, 2, int64_t>&, unsigned char*, cudaStream_t);

}  // namespace nest
