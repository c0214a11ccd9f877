// spmv_pipe.cu -- SpMV instantiations: loop-bound pipeline.
#include "dispatch.cuh"
#include "spmv_variants.h"

namespace nest {

template <class Body>
nest_status spmv_dispatch(const Plan& p, const Body& body, unsigned char* fb, cudaStream_t st) {
    return dispatch(p, body, fb, st);
}

template nest_status spmv_dispatch<SpmvBody<false, true, int32_t>>(const Plan&, const SpmvBody<false, true, int32_t>&, unsigned char*, cudaStream_t);
template nest_status spmv_dispatch<SpmvBody<true, true, int32_t>>(const Plan&, const SpmvBody<true, true, int32_t>&, unsigned char*, cudaStream_t);
template nest_status spmv_dispatch<SpmvBody<false, true, int64_t>>(const Plan&, const SpmvBody<false, true, int64_t>&, unsigned char*, cudaStream_t);
template nest_status spmv_dispatch<SpmvBody<true, true, int64_t>>(const Plan&, const SpmvBody<true, true, int64_t>&, unsigned char*, cudaStream_t);

}  // namespace nest
