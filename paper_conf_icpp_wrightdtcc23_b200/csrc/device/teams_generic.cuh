// teams_generic.cuh -- NEXT-1: the paper's two-level SpMV baseline.
//
// "To utilize the original two levels of parallelism we
// parallelize the outer loop with teams distribute and the inner loop with
// parallel for.  With this structure the teams region will run in generic
// mode."  Generic teams: an extra warp
// holds the team main thread, which alone runs the teams region's sequential
// code; the workers wait in the team state machine at a block-level barrier
// until the main reaches a parallel region, read which region to run and its
// arguments from the team state, run it, and meet the main at a barrier
// again.  A null region pointer ends the teams region.
//
// Here: block = 32 (the main warp; lane 0 is the team main) + T worker
// threads.  Team b takes rows b, b + grid, ... (teams distribute, chunk 1).
// For each row the main loads the loop bounds and posts {fn, trip, base} to
// the team state, then named barrier 1 releases the workers; they run the
// `parallel for` over the row's nonzeros (thread t takes t, t + T, ...), the
// sum is reduced across the workers (warp butterflies, then the warp partials
// in order -- the paper used an atomic update instead), the
// first worker stores y[i], and named barrier 2 returns control to the main.
// No simd level: this is the comparison point of the paper's 3.5x claim.
#pragma once

#include "bodies/bodies.cuh"

namespace nest {

struct TeamState {
    int32_t fn;       // 0 = end of the teams region
    int32_t pad;
    int64_t trip;
    int64_t base;
    int64_t row;
};

template <int OP>
__global__ void spmv_teams_generic_kernel(const int64_t* __restrict__ rowptr, const int32_t* __restrict__ col,
                                          const double* __restrict__ val, const double* __restrict__ x,
                                          double* __restrict__ y, int64_t nrows) {
    __shared__ TeamState ts;
    __shared__ double warp_part[32];
    const int nworkers = (int)blockDim.x - 32;
    const int nthreads = (int)blockDim.x;
    if (threadIdx.x < 32) {
        // the team main warp: lane 0 is the team main and runs the teams region's
        // sequential code; the warp's other lanes only take part in the barriers
        for (int64_t i = blockIdx.x; i < nrows; i += gridDim.x) {
            if (threadIdx.x == 0) {
                const int64_t b = __ldg(rowptr + i), e = __ldg(rowptr + i + 1);
                ts.fn = 1;
                ts.trip = e - b;
                ts.base = b;
                ts.row = i;
            }
            __syncwarp();
            asm volatile("bar.sync 1, %0;" ::"r"(nthreads) : "memory");   // release the workers
            asm volatile("bar.sync 2, %0;" ::"r"(nthreads) : "memory");   // parallel region done
        }
        if (threadIdx.x == 0) ts.fn = 0;                                    // null region: terminate
        __syncwarp();
        asm volatile("bar.sync 1, %0;" ::"r"(nthreads) : "memory");
        return;
    }
    // workers: the team state machine
    const int t = (int)threadIdx.x - 32;
    const int lane = t & 31, wid = t >> 5;
    for (;;) {
        asm volatile("bar.sync 1, %0;" ::"r"(nthreads) : "memory");             // wait for work
        if (ts.fn == 0) return;
        const int64_t trip = ts.trip, base = ts.base, row = ts.row;
        double acc = Red<OP, double>::identity();
        for (int64_t j = t; j < trip; j += nworkers)                            // parallel for
            acc = Red<OP, double>::accum(acc, __ldg(val + base + j), __ldg(x + __ldg(col + base + j)));
#pragma unroll
        for (int off = 16; off >= 1; off >>= 1) acc = Red<OP, double>::combine(acc, __shfl_xor_sync(0xffffffffu, acc, off));
        if (nworkers > 32) {
            if (lane == 0) warp_part[wid] = acc;
            asm volatile("bar.sync 3, %0;" ::"r"(nworkers) : "memory");
            if (t == 0) {
                double s = warp_part[0];
                for (int w = 1; w < nworkers / 32; ++w) s = Red<OP, double>::combine(s, warp_part[w]);
                acc = s;
            }
        }
        if (t == 0) y[row] = acc;
        asm volatile("bar.sync 2, %0;" ::"r"(nthreads) : "memory");             // end of the parallel region
    }
}

}  // namespace nest
