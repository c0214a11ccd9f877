// program.cu -- NEXT-3: several parallel regions with
// different SIMD group sizes inside ONE target region (one kernel).
//
// "All SIMD groups are the same size and the size could
// differ between parallel regions"; with 128 threads the
// number of groups ranges over 4..64 and "different parallel regions can use a
// different number of threads per group which results in a varying number of
// groups", so the sharing space -- divided evenly among the groups
// -- is re-divided per region and falls back to global
// memory when a region's slot is too small.  Every team runs the regions in
// order; each region re-partitions the team into groups of its own simdlen
// (a static tile per S, chosen by a uniform switch) and ends with the team
// barrier of the end of a parallel region.
#include "dispatch.cuh"

namespace nest {

struct RegionArgs {
    int32_t kind, simdlen, mode, slot_bytes;
    int64_t n_outer, chunk;     // outer iterations; team chunk (0 = cyclic)
    int64_t fb_offset;          // byte offset of this region's global fallback
    int32_t use_fb;             // the region's payload exceeds its slot
    int64_t n[3];
    const void* in[4];
    void* out[2];
};

struct Program {
    RegionArgs r[NEST_MAX_REGIONS];
    int32_t count;
};

// Each (simdlen, mode, body) region is its own non-inlined function, so the
// kernel's register allocation is the largest region's, not their sum.
template <int S, int MODE, class Body>
__device__ __noinline__ void region_call(const Body b, const RegionArgs& R, unsigned char* fb, unsigned char* smem) {
    parallel_region<S, MODE, RED_SUM, 1>(b, R.n_outer, R.slot_bytes, fb, R.chunk, smem);
}

template <int S, class Body>
__device__ __forceinline__ void region_s(const Body& b, const RegionArgs& R, unsigned char* fb, unsigned char* smem) {
    if constexpr (S == 1) {
        region_call<1, MODE_SPMD>(b, R, fb, smem);
    } else {
        switch (R.mode) {
            case MODE_SPMD:
                region_call<S, MODE_SPMD>(b, R, fb, smem);
                break;
            case MODE_GENERIC_SMEM:
                region_call<S, MODE_GENERIC_SMEM>(b, R, fb, smem);
                break;
            default:
                region_call<S, MODE_GENERIC_SHFL>(b, R, fb, smem);
                break;
        }
    }
}

template <class Body>
__device__ __forceinline__ void region(const Body& b, const RegionArgs& R, unsigned char* fb, unsigned char* smem) {
    switch (R.simdlen) {   // the region's group size (uniform over the grid)
        case 1: region_s<1>(b, R, fb, smem); break;
        case 2: region_s<2>(b, R, fb, smem); break;
        case 4: region_s<4>(b, R, fb, smem); break;
        case 8: region_s<8>(b, R, fb, smem); break;
        case 16: region_s<16>(b, R, fb, smem); break;
        default: region_s<32>(b, R, fb, smem); break;
    }
}

__global__ void __launch_bounds__(1024, 1) region_program_kernel(const Program prog, unsigned char* __restrict__ gfallback) {
    extern __shared__ __align__(16) unsigned char sharing_space[];
#pragma unroll   // static region index: the arguments stay in the kernel's parameter bank
    for (int k = 0; k < NEST_MAX_REGIONS; ++k) {
        if (k >= prog.count) break;
        const RegionArgs& R = prog.r[k];
        unsigned char* fb = R.use_fb ? gfallback + R.fb_offset : nullptr;
        switch (R.kind) {
            case NEST_REGION_SPMV_CSR_F64: {
                SpmvBody<false, int64_t> b{static_cast<const int64_t*>(R.in[0]),
                                                  static_cast<const int32_t*>(R.in[1]),
                                                  static_cast<const double*>(R.in[2]),
                                                  static_cast<const double*>(R.in[3]), static_cast<double*>(R.out[0])};
                b.nnz = R.n[2];
                region(b, R, fb, sharing_space);
                break;
            }
            case NEST_REGION_BATCHED_MATVEC_F32:
                region(BatchedBody{static_cast<const float*>(R.in[0]), static_cast<const float*>(R.in[1]),
                                   static_cast<float*>(R.out[0]), (int32_t)R.n[1], (int32_t)R.n[2]},
                       R, fb, sharing_space);
                break;
            default:
                region(StencilBody{static_cast<const double*>(R.in[0]), static_cast<const double*>(R.in[1]),
                                   static_cast<const double*>(R.in[2]), static_cast<double*>(R.out[0]),
                                   static_cast<unsigned long long*>(R.out[1]), (int32_t)R.n[1]},
                       R, fb, sharing_space);
                break;
        }
        __syncthreads();   // end of the parallel region: team barrier; the sharing space is re-divided next
    }
}

}  // namespace nest

using namespace nest;

NEST_API nest_status nest_region_program(const nest_desc* desc, const nest_region* regions, int32_t nregions,
                                         void* stream) {
    if (!regions || nregions < 1 || nregions > NEST_MAX_REGIONS)
        return fail(NEST_ERR_INVALID_ARG, "nregions %d: need 1..%d regions", nregions, NEST_MAX_REGIONS);
    Plan base;
    nest_status s = make_plan_fixed(desc, 1, 1, 0, &base);   // validates the team descriptor
    if (s != NEST_OK) return s;
    if (desc->reduce != NEST_REDUCE_SUM || (desc->outer_unroll > 1) || desc->flags || desc->team_chunk)
        return fail(NEST_ERR_UNSUPPORTED, "region programs: SUM reduction, outer_unroll 1, no flags "
                                          "(the schedule is per region)");
    const int32_t T = base.block;
    const int32_t sharing = desc->sharing_bytes ? desc->sharing_bytes : 2048;
    bool any_smem = false;
    for (int k = 0; k < nregions; ++k) any_smem |= regions[k].mode == NEST_MODE_GENERIC_SMEM && regions[k].simdlen > 1;
    const int32_t smem = any_smem ? sharing : 0;
    Program prog{};
    prog.count = nregions;
    int64_t fb_bytes = 0;
    for (int k = 0; k < nregions; ++k) {
        const nest_region& g = regions[k];
        RegionArgs& R = prog.r[k];
        const int32_t S = g.simdlen;
        if (!(S == 1 || S == 2 || S == 4 || S == 8 || S == 16 || S == 32))
            return fail(NEST_ERR_INVALID_ARG, "region %d: simdlen %d", k, S);
        if (g.mode < NEST_MODE_SPMD || g.mode > NEST_MODE_GENERIC_SHFL)
            return fail(NEST_ERR_INVALID_ARG, "region %d: mode %d", k, g.mode);
        if (g.blocked != 0 && g.blocked != 1) return fail(NEST_ERR_INVALID_ARG, "region %d: blocked %d", k, g.blocked);
        for (int q = 0; q < 3; ++q)
            if (g.n[q] < 0) return fail(NEST_ERR_INVALID_ARG, "region %d: negative extent", k);
        int32_t payload;
        switch (g.kind) {
            case NEST_REGION_SPMV_CSR_F64:
                if (g.n[1] > INT32_MAX) return fail(NEST_ERR_INVALID_ARG, "region %d: ncols > int32", k);
                if (g.n[0] > 0 && (!g.in[0] || !g.out[0])) return fail(NEST_ERR_INVALID_ARG, "region %d: NULL", k);
                if (g.n[2] > 0 && (!g.in[1] || !g.in[2] || !g.in[3]))
                    return fail(NEST_ERR_INVALID_ARG, "region %d: NULL", k);
                payload = spmv_payload(1);
                break;
            case NEST_REGION_BATCHED_MATVEC_F32:
                if (g.n[1] > INT32_MAX || g.n[2] > INT32_MAX) return fail(NEST_ERR_INVALID_ARG, "region %d: m/n", k);
                if (g.n[0] > 0 && g.n[1] > 0 && (!g.out[0] || (g.n[2] > 0 && (!g.in[0] || !g.in[1]))))
                    return fail(NEST_ERR_INVALID_ARG, "region %d: NULL", k);
                payload = batched_payload(1);
                break;
            case NEST_REGION_NESTED_STENCIL_F64:
                if (g.n[1] > INT32_MAX) return fail(NEST_ERR_INVALID_ARG, "region %d: L", k);
                if (g.n[0] > 0 && (!g.in[2] || !g.out[0] || (g.n[1] > 0 && (!g.in[0] || !g.in[1]))))
                    return fail(NEST_ERR_INVALID_ARG, "region %d: NULL", k);
                payload = stencil_payload(1);
                break;
            default:
                return fail(NEST_ERR_INVALID_ARG, "region %d: kind %d", k, g.kind);
        }
        const int32_t G = T / S;
        R.kind = g.kind;
        R.simdlen = S;
        R.mode = S == 1 ? NEST_MODE_SPMD : g.mode;
        R.slot_bytes = (sharing / G) & ~7;   // the space re-divided among this region's groups
        R.n_outer = g.kind == NEST_REGION_BATCHED_MATVEC_F32 && g.n[1] == 0 ? 0 : g.n[0];
        R.chunk = g.blocked;   // resolved below, once the grid is known
        R.fb_offset = payload;
        for (int q = 0; q < 3; ++q) R.n[q] = g.n[q];
        for (int q = 0; q < 4; ++q) R.in[q] = g.in[q];
        for (int q = 0; q < 2; ++q) R.out[q] = g.out[q];
    }
    // all arguments validated: now the league (device queries may fail)
    int64_t grid = desc->num_teams;
    if (grid <= 0 && (s = resident_blocks(T, smem, &grid)) != NEST_OK) return s;
    for (int k = 0; k < nregions; ++k) {
        RegionArgs& R = prog.r[k];
        const int32_t G = T / R.simdlen;
        const int64_t payload = R.fb_offset;
        if (R.chunk) {
            R.chunk = ((R.n_outer + grid - 1) / grid + G - 1) / G * G;
            if (R.chunk == 0) R.chunk = G;
        }
        R.fb_offset = fb_bytes;
        R.use_fb = R.mode == NEST_MODE_GENERIC_SMEM && payload > R.slot_bytes;
        if (R.use_fb) fb_bytes += grid * G * payload;
    }
    unsigned char* fb = nullptr;
    if (fb_bytes > 0 && (s = fallback_scratch((size_t)fb_bytes, &fb, stream)) != NEST_OK) return s;
    region_program_kernel<<<(unsigned)grid, T, smem, static_cast<cudaStream_t>(stream)>>>(prog, fb);
    const cudaError_t e = cudaGetLastError();
    return e == cudaSuccess ? NEST_OK : cuda_fail(e, "region program launch");
}
