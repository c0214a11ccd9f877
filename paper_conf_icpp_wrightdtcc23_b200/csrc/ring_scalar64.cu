// ring_scalar64.cu -- x-ring SpMV instantiations (RingScalar64; separate translation units compile in parallel).
#include "ring_dispatch.cuh"

namespace nest {

nest_status ring_scalar64(const Plan& p, const RingArgs& a, cudaStream_t st) { return ring_dispatch<RingScalar64>(p, a, st); }

}  // namespace nest
