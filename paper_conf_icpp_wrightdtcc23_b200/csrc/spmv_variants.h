// spmv_variants.h -- the SpMV body instantiations live in separate translation
// units (spmv_*.cu) so they compile in parallel; launch_spmv.cu only calls them.
#pragma once

#include "bodies/bodies.cuh"
#include "internal.h"

namespace nest {

// dispatch(p, body) for one SpMV body type (explicitly instantiated in spmv_*.cu)
template <class Body>
nest_status spmv_dispatch(const Plan& p, const Body& body, unsigned char* fb, cudaStream_t st);

}  // namespace nest
