// spmv_xwin.cuh -- a8 CSR SpMV with a team-level shared-memory window of x
// (NEST desc.x_halo > 0): the north_star's "shared staging of x tiles".
//
// Same three levels as nest_kernel -- teams (blocks) -> parallel (SIMD groups
// over rows) -> simd (lanes over a row's nonzeros, Fig 8 cyclic) -- and the
// same SPMD / generic mode engine (simd_batch), with a different teams-level
// schedule: each team owns a contiguous block of rows ("teams distribute"
// with a static block schedule, R6) and walks it in chunks of
// R = G*U rows (group g takes rows r0 + u*G + g).  Before a chunk is computed
// the team has staged, with cp.async into shared memory,
//   * rowptr[r0 .. r0+R]                      (double-buffered), and
//   * x[lo, hi), lo = r0 - H, hi = r0 + R + H (a ring of XW doubles),
// and it stages the NEXT chunk's rowptr and the newly needed tail of x while
// the current chunk computes.  A nonzero whose column lies in [lo, hi) reads x
// from the ring (LDS), any other column reads global memory (__ldg), so the
// result is identical for any H; H only decides how many gathers hit shared
// memory.  The ring never overwrites an entry the current chunk may read
// because XW >= 2R + 2H (checked by the planner).
#pragma once

#include "bodies/bodies.cuh"

namespace nest {

__device__ __forceinline__ void cp_async8(void* smem_dst, const void* gsrc) {
    const unsigned s = (unsigned)__cvta_generic_to_shared(smem_dst);
    asm volatile("cp.async.ca.shared.global [%0], [%1], 8;\n" ::"r"(s), "l"(gsrc) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;\n" ::: "memory"); }
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_all;\n" ::: "memory"); }

template <bool HINTS>
struct SpmvXwinBody {
    using Acc = double;
    struct Loop {
        int64_t trip;
        int64_t base;
    };
    struct Step {
        int64_t i;
    };
    const int32_t* col;
    const double* val;
    const double* x;
    double* y;
    const double* ring;
    int32_t lo;         // window [lo, lo + span)
    uint32_t span;
    uint32_t lo_slot;   // ring slot of column lo
    uint32_t xw;        // ring capacity (doubles)

    template <int OP>
    __device__ __forceinline__ double accum(const Loop& L, int64_t j, double acc) const {
        const int64_t k = L.base + j;
        const int32_t c = HINTS ? __ldcs(col + k) : __ldg(col + k);
        const double v = HINTS ? __ldcs(val + k) : __ldg(val + k);
        const uint32_t d = (uint32_t)(c - lo);
        double xv;
        if (d < span) {
            uint32_t sl = d + lo_slot;
            sl = sl >= xw ? sl - xw : sl;
            xv = ring[sl];
        } else {
            xv = __ldg(x + c);
        }
        return Red<OP, double>::accum(acc, v, xv);
    }
    __device__ __forceinline__ void epilogue(const Step& st, double total) const { y[st.i] = total; }
};

struct XwinArgs {
    const int64_t* rowptr;
    const int32_t* col;
    const double* val;
    const double* x;
    double* y;
    int64_t nrows;
    int64_t ncols;
    int32_t halo;
    int32_t xw;          // ring capacity in doubles (>= 2R + 2H)
    int32_t slot_bytes;
    unsigned char* gfallback;
};

template <int S, int MODE, int OP, int U, bool HINTS>
__global__ void __launch_bounds__(1024, 2) spmv_xwin_kernel(const XwinArgs a) {
    using Body = SpmvXwinBody<HINTS>;
    using Loop = typename Body::Loop;
    using Step = typename Body::Step;
    extern __shared__ __align__(16) unsigned char smem[];
    const uint32_t XW = (uint32_t)a.xw;
    double* ring = reinterpret_cast<double*>(smem);
    const SimdGroup<S> g;
    const int G = (int)(blockDim.x / S);
    const int R = G * U;
    int64_t* rps = reinterpret_cast<int64_t*>(smem + (size_t)XW * 8);   // [2][R+1]
    unsigned char* sharing = reinterpret_cast<unsigned char*>(rps + 2 * (R + 1));

    // this team's block of rows
    const int64_t per_team = (a.nrows + gridDim.x - 1) / gridDim.x;
    const int64_t rb = (int64_t)blockIdx.x * per_team;
    const int64_t re = rb + per_team < a.nrows ? rb + per_team : a.nrows;
    const int64_t gid = (int64_t)blockIdx.x * G + g.group();
    Slot<Loop, U>* slot = group_slot<MODE, Loop, U>(sharing, a.slot_bytes, a.gfallback, g.group(), gid);

    Body body{a.col, a.val, a.x, a.y, ring, 0, 0, 0, XW};
    auto win_lo = [&](int64_t r0) { return r0 - a.halo > 0 ? r0 - a.halo : (int64_t)0; };
    auto win_hi = [&](int64_t r0) {
        const int64_t h = r0 + R + a.halo;
        return h < a.ncols ? h : a.ncols;
    };
    // cp.async the rowptr of chunk r0 into buffer `buf` and x[xf, xt) into the ring
    auto stage = [&](int64_t r0, int buf, int64_t xf, int64_t xt) {
        const int64_t rows = re - r0 < R ? re - r0 : R;
        int64_t* dst = rps + buf * (R + 1);
        for (int t = threadIdx.x; t <= rows; t += blockDim.x) cp_async8(dst + t, a.rowptr + r0 + t);
        if (xt > xf) {
            const uint32_t s0 = (uint32_t)(xf % XW);
            for (uint32_t t = threadIdx.x; t < (uint32_t)(xt - xf); t += blockDim.x) {
                uint32_t sl = s0 + t;
                sl = sl >= XW ? sl - XW : sl;
                cp_async8(ring + sl, a.x + xf + t);
            }
        }
        cp_async_commit();
    };

    if (rb < re) {
        stage(rb, 0, win_lo(rb), win_hi(rb));
        cp_async_wait_all();
        __syncthreads();
        int buf = 0;
        for (int64_t r0 = rb; r0 < re; r0 += R, buf ^= 1) {
            const int64_t rend = r0 + R < re ? r0 + R : re;
            const int64_t hi = win_hi(r0);
            if (rend < re) stage(rend, buf ^ 1, hi, win_hi(rend));       // prefetch the next chunk
            const int64_t lo = win_lo(r0);
            body.lo = (int32_t)lo;
            body.span = hi > lo ? (uint32_t)(hi - lo) : 0u;
            body.lo_slot = (uint32_t)(lo % XW);
            const int64_t* rp = rps + buf * (R + 1);
            auto gather = [&](Loop (&L)[U], Step (&st)[U], bool) {
                int cnt = 0;
#pragma unroll
                for (int u = 0; u < U; ++u) {
                    const int64_t r = r0 + (int64_t)u * G + g.group();
                    if (r < rend) {
                        const int off = (int)(r - r0);
                        const int64_t b = rp[off];
                        L[u] = Loop{rp[off + 1] - b, b};
                        st[u].i = r;
                        ++cnt;
                    } else {
                        L[u].trip = 0;
                    }
                }
                return cnt;   // an empty batch keeps the workers in step; never ends the region
            };
            simd_batch<S, MODE, OP, U>(body, g, slot, gather);
            cp_async_wait_all();
            __syncthreads();
        }
    }
    // end of the parallel region: the main posts the null fn
    auto done = [&](Loop (&L)[U], Step (&)[U], bool) {
#pragma unroll
        for (int u = 0; u < U; ++u) L[u].trip = 0;
        return -1;
    };
    simd_batch<S, MODE, OP, U>(body, g, slot, done);
}

}  // namespace nest
