// spmv_scalar_i64.cu -- SpMV instantiations: scalar loads, 64-bit indices.
#include "dispatch.cuh"
#include "spmv_variants.h"

namespace nest {

template <class Body>
nest_status spmv_dispatch(const Plan& p, const Body& body, unsigned char* fb, cudaStream_t st) {
    return dispatch(p, body, fb, st);
}

template nest_status spmv_dispatch<SpmvBody<false, int64_t>>(const Plan&, const SpmvBody<false, int64_t>&, unsigned char*, cudaStream_t);
template nest_status spmv_dispatch<SpmvBody<true, int64_t>>(const Plan&, const SpmvBody<true, int64_t>&, unsigned char*, cudaStream_t);

}  // namespace nest
