// launch_batched.cu -- a9 batched small dense matvec instantiations.
#include "dispatch.cuh"

namespace nest {

int32_t batched_payload(int32_t U) {
    switch (U) {
        case 1: return payload_bytes<BatchedBody, 1>();
        case 2: return payload_bytes<BatchedBody, 2>();
        case 4: return payload_bytes<BatchedBody, 4>();
    }
    return -1;
}
static_assert(sizeof(BatchedVecBody::Loop) == sizeof(BatchedBody::Loop), "same generic payload");

nest_status launch_batched(const Plan& p, int64_t, int32_t m, int32_t n, const float* A,
                           const float* x, float* y, unsigned char* fb, cudaStream_t st) {
    if (p.flags & NEST_F_VEC128)
        return dispatch(p, BatchedVecBody{reinterpret_cast<const float4*>(A), reinterpret_cast<const float4*>(x), y, m, n},
                        fb, st);
    return dispatch(p, BatchedBody{A, x, y, m, n}, fb, st);
}

}  // namespace nest
