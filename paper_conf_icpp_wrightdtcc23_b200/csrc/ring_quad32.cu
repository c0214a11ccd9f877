// ring_quad32.cu -- x-ring SpMV instantiations (RingQuad32; separate translation units compile in parallel).
#include "ring_dispatch.cuh"

namespace nest {

nest_status ring_quad32(const Plan& p, const RingArgs& a, cudaStream_t st) { return ring_dispatch<RingQuad32>(p, a, st); }

}  // namespace nest
