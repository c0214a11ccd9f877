// ring_pair32.cu -- x-ring SpMV instantiations (RingPair32; separate translation units compile in parallel).
#include "ring_dispatch.cuh"

namespace nest {

nest_status ring_pair32(const Plan& p, const RingArgs& a, cudaStream_t st) { return ring_dispatch<RingPair32>(p, a, st); }

}  // namespace nest
