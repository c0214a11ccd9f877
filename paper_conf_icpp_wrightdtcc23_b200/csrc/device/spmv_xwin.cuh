// spmv_xwin.cuh -- a8 CSR SpMV with a team-level shared-memory window of x
// (nest_desc.x_halo > 0): the north_star's "shared staging of x tiles".
//
// Why: with x gathered through L1 every nonzero costs one L1 data-pipe
// wavefront (the 32 lanes of a gather hit ~32 different lines); that pipe is
// the limiter of the unstaged kernel (profiles/r01_l2_traffic_experiments.md).
// Gathers served from shared memory cost a few wavefronts per warp instead.
//
// Same three levels as nest_kernel -- teams (blocks) -> parallel (SIMD groups
// over rows) -> simd (lanes over a row's nonzeros, Fig 8 cyclic, or over pairs
// of nonzeros with NEST_F_VEC128) -- and the same SPMD / generic mode engine
// (simd_batch), with a blocked teams-level schedule: team b owns the rows
// [b*C, (b+1)*C) and walks them in chunks of R = G*U*KB rows; inside a chunk
// group g runs KB batches of U rows (row r0 + (m*U + u)*G + g) with no team
// barrier.  While chunk r0 computes, the team's x window
//   [lo, hi) = [r0 - H, r0 + R + H) ∩ [0, ncols)
// is resident in a shared-memory ring of XW = 2R + 2H doubles (slot of column
// c: c mod XW), and the NEXT chunk's new tail [hi, hi + R) is already in
// flight: one thread issues 1D bulk copies (cp.async.bulk, the TMA engine)
// completing on an mbarrier.  Those slots held columns [r0 - R - H, r0 - H),
// which only the previous chunk read, so one team barrier per chunk suffices.
// A nonzero whose column lies in [lo, hi) reads the ring, any other column
// reads global memory: the result is identical for every H, H only decides how
// many gathers hit shared memory.
#pragma once

#include "bodies/bodies.cuh"
#include "device/ptx.cuh"

namespace nest {

// x access policy of the window (bodies.cuh XA): ring hit or global gather.
struct XWindow {
    const double* x;
    const double* ring;
    int32_t lo;         // window [lo, lo + span)
    uint32_t span;
    uint32_t lo_slot;   // ring slot of column lo
    uint32_t xw;        // ring capacity (doubles)
    __device__ __forceinline__ double operator()(int32_t c) const {
        const uint32_t d = (uint32_t)(c - lo);
        if (d < span) {
            uint32_t sl = d + lo_slot;
            sl = sl >= xw ? sl - xw : sl;
            return ring[sl];
        }
        return __ldg(x + c);
    }
};

struct XwinArgs {
    const int64_t* rowptr;
    const int32_t* col;
    const double* val;
    const double* x;
    double* y;
    int64_t nrows;
    int64_t ncols;
    int64_t nnz;
    int32_t halo;        // H (even)
    int32_t xw;          // ring capacity in doubles (= 2R + 2H)
    int32_t kb;          // batches per chunk
    int32_t slot_bytes;
    unsigned char* gfallback;
};

// The fill of x[from, to) into the ring (slot c mod XW): 1D bulk copies of the
// even-length part (16-byte multiples; `from` is even) completing on `bar`, and
// a plain store of a trailing odd double (to == ncols).  Returns the bulk bytes.
__device__ __forceinline__ uint32_t xwin_fill_bytes(int64_t from, int64_t to) {
    const int64_t te = to & ~(int64_t)1;
    return te > from ? (uint32_t)(te - from) * 8u : 0u;
}
__device__ __forceinline__ void xwin_fill_tail(const double* x, double* ring, uint32_t xw, int64_t from, int64_t to) {
    const int64_t te = to & ~(int64_t)1;
    if (to > te && te >= from) ring[(uint32_t)(te % xw)] = x[te];
}
__device__ __forceinline__ void xwin_fill(const double* x, double* ring, uint32_t xw, int64_t from, int64_t to,
                                          uint64_t* bar) {
    const int64_t te = to & ~(int64_t)1;
    while (from < te) {
        const uint32_t s0 = (uint32_t)(from % xw);
        int64_t n = te - from;
        if ((int64_t)s0 + n > (int64_t)xw) n = (int64_t)xw - s0;   // up to the ring's end
        bulk_g2s(ring + s0, x + from, (uint32_t)n * 8u, bar);
        from += n;
    }
}

template <int S, int MODE, int OP, int U, class Body>
__global__ void __launch_bounds__(1024, 2) spmv_xwin_kernel(const XwinArgs a) {
    using Loop = typename Body::Loop;
    using Step = typename Body::Step;
    extern __shared__ __align__(16) unsigned char smem[];
    const uint32_t XW = (uint32_t)a.xw;
    double* ring = reinterpret_cast<double*>(smem);
    uint64_t* bars = reinterpret_cast<uint64_t*>(smem + (size_t)XW * 8);   // [2]: chunk c uses bars[c & 1]
    unsigned char* sharing = smem + (size_t)XW * 8 + 16;
    const SimdGroup<S> g;
    const int G = (int)(blockDim.x / S);
    const int64_t R = (int64_t)G * U * a.kb;
    typename Body::TeamShared tsh;

    // this team's block of rows: a multiple of R (every window start is even)
    const int64_t per_team = ((a.nrows + gridDim.x - 1) / gridDim.x + R - 1) / R * R;
    const int64_t rb = (int64_t)blockIdx.x * per_team;
    const int64_t re = rb + per_team < a.nrows ? rb + per_team : a.nrows;
    const int64_t gid = (int64_t)blockIdx.x * G + g.group();
    Slot<Loop, U>* slot = group_slot<MODE, Loop, U>(sharing, a.slot_bytes, a.gfallback, g.group(), gid);

    Body body{a.rowptr, a.col, a.val, XWindow{a.x, ring, 0, 0u, 0u, XW}, a.y};
    body.nnz = a.nnz;
    auto win_lo = [&](int64_t r0) { return r0 - a.halo > 0 ? r0 - a.halo : (int64_t)0; };
    auto win_hi = [&](int64_t r0) {
        const int64_t h = r0 + R + a.halo;
        return h < a.ncols ? h : a.ncols;
    };
    auto fill = [&](int64_t from, int64_t to, uint64_t* bar) {   // thread 0
        xwin_fill_tail(a.x, ring, XW, from, to);                    // plain store, released by the arrive
        mbar_arrive_expect_tx(bar, xwin_fill_bytes(from, to));
        xwin_fill(a.x, ring, XW, from, to, bar);
    };
    if (threadIdx.x == 0) {
        mbar_init(&bars[0], 1);
        mbar_init(&bars[1], 1);
        mbar_fence_init();
    }
    __syncthreads();
    if (rb < re && threadIdx.x == 0) fill(win_lo(rb), win_hi(rb), &bars[0]);   // the first window
    int64_t c = 0;
    for (int64_t r0 = rb; r0 < re; r0 += R, ++c) {
        mbar_wait(&bars[c & 1], (uint32_t)((c >> 1) & 1));   // this chunk's window has landed
        const int64_t hi = win_hi(r0);
        const int64_t lo = win_lo(r0) < hi ? win_lo(r0) : hi;   // rows past the last column: empty window
        // the next chunk's new tail overwrites the slots of [r0 - R - H, r0 - H):
        // only the previous chunk read them, and it ended at a team barrier
        if (threadIdx.x == 0 && r0 + R < re) fill(hi, win_hi(r0 + R), &bars[(c + 1) & 1]);
        body.x.lo = (int32_t)lo;
        body.x.span = (uint32_t)(hi - lo);
        body.x.lo_slot = (uint32_t)(lo % XW);
        const int64_t rend = r0 + R < re ? r0 + R : re;
        for (int m = 0; m < a.kb; ++m) {
            auto gather = [&](Loop (&L)[U], Step (&st)[U], bool fx) {
                int cnt = 0;
#pragma unroll
                for (int u = 0; u < U; ++u) {
                    const int64_t r = r0 + ((int64_t)m * U + u) * G + g.group();
                    if (r < rend) {
                        L[u] = body.prologue(r, 0, st[u], fx, tsh);
                        ++cnt;
                    } else {
                        L[u].trip = 0;
                    }
                }
                return cnt;   // an empty batch keeps the workers in step; never ends the region
            };
            simd_batch<S, MODE, OP, U>(body, g, slot, gather);
        }
        __syncthreads();
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
