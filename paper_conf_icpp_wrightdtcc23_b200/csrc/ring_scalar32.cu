// ring_scalar32.cu -- x-ring SpMV instantiations (RingScalar32; separate translation units compile in parallel).
#include "ring_dispatch.cuh"

namespace nest {

nest_status ring_scalar32(const Plan& p, const RingArgs& a, cudaStream_t st) { return ring_dispatch<RingScalar32>(p, a, st); }

}  // namespace nest
