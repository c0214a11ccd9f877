// launch_probe.cu -- a2 mapping probe and the a5/a6 coverage probe.
#include "dispatch.cuh"

namespace nest {

// out_map[t] = {getSimdGroup, getSimdGroupId, getSimdGroupSize, isSimdGroupLeader, simdmask}
template <int S>
__global__ void probe_map_kernel(int32_t* __restrict__ out) {
    const SimdGroup<S> g;
    int32_t* o = out + ((size_t)blockIdx.x * blockDim.x + threadIdx.x) * 5;
    o[0] = g.group();
    o[1] = g.id();
    o[2] = g.size();
    o[3] = g.leader() ? 1 : 0;
    o[4] = (int32_t)g.mask();
}

int32_t probe_payload(int32_t U) {
    switch (U) {
        case 1: return payload_bytes<ProbeBody, 1>();
        case 2: return payload_bytes<ProbeBody, 2>();
        case 4: return payload_bytes<ProbeBody, 4>();
    }
    return -1;
}

nest_status launch_probe(const Plan& p, int32_t* out_map, int64_t trip, int32_t* hits,
                         int32_t* owner, double* totals, unsigned char* fb, cudaStream_t st) {
    if (out_map) {
        switch (p.simdlen) {
            case 1: probe_map_kernel<1><<<p.grid, p.block, 0, st>>>(out_map); break;
            case 2: probe_map_kernel<2><<<p.grid, p.block, 0, st>>>(out_map); break;
            case 4: probe_map_kernel<4><<<p.grid, p.block, 0, st>>>(out_map); break;
            case 8: probe_map_kernel<8><<<p.grid, p.block, 0, st>>>(out_map); break;
            case 16: probe_map_kernel<16><<<p.grid, p.block, 0, st>>>(out_map); break;
            case 32: probe_map_kernel<32><<<p.grid, p.block, 0, st>>>(out_map); break;
            default: return fail(NEST_ERR_INVALID_ARG, "simdlen %d", p.simdlen);
        }
        const cudaError_t e = cudaGetLastError();
        if (e != cudaSuccess) return cuda_fail(e, "probe_map launch");
    }
    return dispatch(p, ProbeBody{hits, owner, totals, trip}, fb, st);
}

}  // namespace nest
