// spmv_staged.cuh -- a8 CSR SpMV, B200 pipeline variant (NEST_F_STAGED).
//
// The same three levels and mode engine as nest_kernel -- teams (CTAs) ->
// parallel (SIMD groups over rows) -> simd (lanes over a row's nonzeros,
// Fig 8 cyclic) with SPMD or generic execution of the parallel region
// (simd_batch) -- but the memory traffic is decoupled from the loop nest:
//
//   * warp 0 of every team is a PRODUCER.  For each chunk of R = G*U rows of
//     the team's contiguous block of rows it loads rowptr[r0 .. r0+R] into a
//     shared-memory stage and issues 1D bulk async copies (cp.async.bulk,
//     the TMA engine: SASS UBLKCP) of the chunk's colind and val ranges, plus
//     the newly needed tail of the x window into a ring.  Completion is
//     tracked by a "full" mbarrier (expect_tx); a stage is reused only after
//     every consumer warp arrived on its "empty" mbarrier.  NS stages are in
//     flight, so HBM streams while the consumers compute.
//   * warps 1.. are CONSUMERS: the SIMD groups.  They run the loop nest over
//     the staged chunk out of shared memory; x comes from the ring when the
//     column lies in the window [r0 - H, r0 + R + H), else from global memory.
//     Anything that did not fit a stage (rows longer than the stage capacity,
//     the unaligned last elements of the arrays) is read from global memory,
//     so the result is the same for any matrix, H, NB or NS.
//
// Alignment: the bulk copies need 16-byte aligned global and shared addresses
// and sizes; the copied ranges are the 16-byte aligned subranges, everything
// else takes the global path.  The host launcher requires colind, val and x
// to be 16-byte aligned base pointers (else it uses nest_kernel).
#pragma once

#include "bodies/bodies.cuh"

namespace nest {

// ------------------------------------------------------------ PTX helpers
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
    return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;\n" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_fence_init() {
    asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
    asm volatile("{\n .reg .b64 st;\n mbarrier.arrive.shared::cta.b64 st, [%0];\n}\n" ::"r"(smem_u32(bar))
                 : "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* bar, uint32_t tx) {
    asm volatile("{\n .reg .b64 st;\n mbarrier.arrive.expect_tx.shared::cta.b64 st, [%0], %1;\n}\n" ::"r"(
                     smem_u32(bar)),
                 "r"(tx)
                 : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
    const uint32_t a = smem_u32(bar);
    uint32_t done = 0;
    do {
        asm volatile(
            "{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n selp.u32 %0, 1, 0, p;\n}\n"
            : "=r"(done)
            : "r"(a), "r"(parity)
            : "memory");
    } while (!done);
}
// 1D bulk global -> shared copy completing on an mbarrier (TMA engine).
__device__ __forceinline__ void bulk_g2s(void* sdst, const void* gsrc, uint32_t bytes, uint64_t* bar) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];\n" ::"r"(
            smem_u32(sdst)),
        "l"(gsrc), "r"(bytes), "r"(smem_u32(bar))
        : "memory");
}

// The staged ranges of a chunk whose nonzeros are [b, e): colind [cb, cb+cn),
// val [vb, vb+vn) -- 16-byte aligned, at most NB elements, never past the
// 16-byte aligned prefix of the arrays.  Producer and consumers evaluate the
// same function of (b, e, nnz, NB).
struct StagedRange {
    int64_t cb, vb;
    int32_t cn, vn;
};
__device__ __forceinline__ StagedRange staged_range(int64_t b, int64_t e, int64_t nnz, int32_t NB) {
    StagedRange r;
    r.cb = b & ~(int64_t)3;
    int64_t ce = (e + 3) & ~(int64_t)3;
    const int64_t cmax = nnz & ~(int64_t)3;
    if (ce > cmax) ce = cmax;
    if (ce > r.cb + NB) ce = r.cb + NB;
    r.cn = ce > r.cb ? (int32_t)(ce - r.cb) : 0;
    r.vb = b & ~(int64_t)1;
    int64_t ve = (e + 1) & ~(int64_t)1;
    const int64_t vmax = nnz & ~(int64_t)1;
    if (ve > vmax) ve = vmax;
    if (ve > r.vb + NB) ve = r.vb + NB;
    r.vn = ve > r.vb ? (int32_t)(ve - r.vb) : 0;
    return r;
}

// Body: nonzeros from the stage (or global), x from the ring (or global).
struct SpmvStagedBody {
    using Acc = double;
    struct Loop {
        int64_t trip;
        int64_t base;   // global nonzero index of the row's first entry
    };
    struct Step {
        int64_t i;
    };
    const int32_t* col;
    const double* val;
    const double* x;
    double* y;
    const double* ring;
    // per chunk
    const int32_t* s_col;
    const double* s_val;
    int64_t cb, vb;
    uint32_t cn, vn;
    int64_t lo;      // window [lo, lo + span)
    int64_t org;     // ring slot of column c = c - org (mod XW)
    uint32_t span;
    uint32_t xw;

    template <int OP>
    __device__ __forceinline__ double accum(const Loop& L, int64_t j, double acc) const {
        const int64_t k = L.base + j;
        const uint32_t kc = (uint32_t)(k - cb), kv = (uint32_t)(k - vb);
        const int32_t c = kc < cn ? s_col[kc] : __ldg(col + k);
        const double v = kv < vn ? s_val[kv] : __ldg(val + k);
        double xv;
        if ((uint64_t)((int64_t)c - lo) < (uint64_t)span) {
            uint32_t s = (uint32_t)((int64_t)c - org);
            if (s >= xw) s -= xw;
            xv = ring[s];
        } else {
            xv = __ldg(x + c);
        }
        return Red<OP, double>::accum(acc, v, xv);
    }
    __device__ __forceinline__ void epilogue(const Step& st, double total) const { y[st.i] = total; }
};

struct StagedArgs {
    const int64_t* rowptr;
    const int32_t* col;
    const double* val;
    const double* x;
    double* y;
    int64_t nrows, ncols, nnz;
    int32_t halo;        // 0 = no x window
    int32_t xw;          // ring capacity in doubles (even), 0 if no window
    int32_t nb;          // stage capacity in nonzeros (multiple of 4)
    int32_t ns;          // number of stages
    int32_t slot_bytes;  // generic sharing-space slot
    unsigned char* gfallback;
};

// Shared-memory layout (all offsets 16-byte aligned), see stage_bytes().
struct StagedLayout {
    uint32_t ring, stage0, stage_stride, val_off, col_off, rp_off, bars, sharing, total;
};
__host__ __device__ __forceinline__ StagedLayout staged_layout(int32_t xw, int32_t nb, int32_t ns, int32_t R,
                                                            int32_t sharing_bytes) {
    auto al = [](uint32_t v) { return (v + 15u) & ~15u; };
    StagedLayout l;
    l.ring = 0;
    l.stage0 = al((uint32_t)xw * 8u);
    l.val_off = 0;
    l.col_off = al((uint32_t)nb * 8u);
    l.rp_off = l.col_off + al((uint32_t)nb * 4u);
    l.stage_stride = l.rp_off + al((uint32_t)(R + 1) * 8u);
    l.bars = l.stage0 + (uint32_t)ns * l.stage_stride;
    l.sharing = al(l.bars + (uint32_t)ns * 16u);
    l.total = l.sharing + (uint32_t)sharing_bytes;
    return l;
}

template <int S, int MODE, int OP, int U>
__global__ void __launch_bounds__(1024, 1) spmv_staged_kernel(const StagedArgs a) {
    using Body = SpmvStagedBody;
    using Loop = Body::Loop;
    using Step = Body::Step;
    extern __shared__ __align__(16) unsigned char smem[];
    const int nconsumer = (int)blockDim.x - 32;
    const int G = nconsumer / S;                 // consumer SIMD groups per team
    const int R = G * U;                         // rows per chunk
    const int32_t sharing_bytes = a.slot_bytes * G;
    const StagedLayout lay = staged_layout(a.xw, a.nb, a.ns, R, MODE == MODE_GENERIC_SMEM ? sharing_bytes : 0);
    double* ring = reinterpret_cast<double*>(smem + lay.ring);
    uint64_t* full = reinterpret_cast<uint64_t*>(smem + lay.bars);
    uint64_t* empty = full + a.ns;
    auto st_val = [&](int s) { return reinterpret_cast<double*>(smem + lay.stage0 + s * lay.stage_stride + lay.val_off); };
    auto st_col = [&](int s) { return reinterpret_cast<int32_t*>(smem + lay.stage0 + s * lay.stage_stride + lay.col_off); };
    auto st_rp = [&](int s) { return reinterpret_cast<int64_t*>(smem + lay.stage0 + s * lay.stage_stride + lay.rp_off); };

    const int64_t per_team = (a.nrows + gridDim.x - 1) / gridDim.x;
    const int64_t rb = (int64_t)blockIdx.x * per_team;
    const int64_t re = rb + per_team < a.nrows ? rb + per_team : a.nrows;
    const int warp = (int)(threadIdx.x >> 5), lane = (int)(threadIdx.x & 31);
    const int H = a.halo;

    if (threadIdx.x == 0) {
        for (int s = 0; s < a.ns; ++s) {
            mbar_init(full + s, 1);
            mbar_init(empty + s, (uint32_t)(nconsumer / 32));
        }
        mbar_fence_init();
    }
    __syncthreads();

    auto win_lo = [&](int64_t r0) { return r0 - H > 0 ? r0 - H : (int64_t)0; };
    auto win_hi = [&](int64_t r0) {
        const int64_t h = r0 + R + H;
        return h < a.ncols ? h : a.ncols;
    };

    if (warp == 0) {
        // ------------------------------------------------------------ producer
        int64_t xdone = 0;   // x staged up to (exclusive)
        int k = 0;
        for (int64_t r0 = rb; r0 < re; r0 += R, ++k) {
            const int s = k % a.ns;
            if (k >= a.ns) mbar_wait(empty + s, (uint32_t)((k / a.ns) - 1) & 1u);
            const int rows = (int)(re - r0 < R ? re - r0 : R);
            int64_t* rp = st_rp(s);
            for (int t = lane; t <= rows; t += 32) rp[t] = __ldg(a.rowptr + r0 + t);
            const int64_t b = __ldg(a.rowptr + r0), e = __ldg(a.rowptr + r0 + rows);
            const StagedRange sr = staged_range(b, e, a.nnz, a.nb);
            // x window tail [xa, xb): 16-byte aligned interior by bulk copy, odd ends by hand
            int64_t xa = 0, xb = 0, xa2 = 0, xb2 = 0;
            if (a.xw > 0) {
                xa = k == 0 ? win_lo(r0) : xdone;
                xb = win_hi(r0);
                if (xb < xa) xb = xa;
                xdone = xb;
                xa2 = (xa + 1) & ~(int64_t)1;
                xb2 = xb & ~(int64_t)1;
                if (xb2 < xa2) xb2 = xa2;
                if (lane == 1 && (xa & 1) && xa < xb) ring[(uint32_t)(xa % a.xw)] = __ldg(a.x + xa);
                if (lane == 2 && (xb & 1) && xb - 1 >= xa2 && xb - 1 >= xa) ring[(uint32_t)((xb - 1) % a.xw)] = __ldg(a.x + xb - 1);
            }
            __syncwarp();
            if (lane == 0) {
                const uint32_t xbytes = (uint32_t)(xb2 - xa2) * 8u;
                mbar_arrive_expect_tx(full + s, (uint32_t)sr.cn * 4u + (uint32_t)sr.vn * 8u + xbytes);
                if (sr.vn) bulk_g2s(st_val(s), a.val + sr.vb, (uint32_t)sr.vn * 8u, full + s);
                if (sr.cn) bulk_g2s(st_col(s), a.col + sr.cb, (uint32_t)sr.cn * 4u, full + s);
                if (xbytes) {
                    const uint32_t slot = (uint32_t)(xa2 % a.xw);
                    const uint32_t n = (uint32_t)(xb2 - xa2);
                    const uint32_t n1 = slot + n <= (uint32_t)a.xw ? n : (uint32_t)a.xw - slot;
                    bulk_g2s(ring + slot, a.x + xa2, n1 * 8u, full + s);
                    if (n1 < n) bulk_g2s(ring, a.x + xa2 + n1, (n - n1) * 8u, full + s);
                }
            }
        }
        return;
    }

    // -------------------------------------------------------------- consumers
    const SimdGroup<S> g;
    const int cg = g.group() - 32 / S;           // consumer group index
    const int64_t gid = (int64_t)blockIdx.x * G + cg;
    Slot<Loop, U>* slot = group_slot<MODE, Loop, U>(smem + lay.sharing, a.slot_bytes, a.gfallback, cg, gid);
    Body body{a.col, a.val, a.x, a.y, ring, nullptr, nullptr, 0, 0, 0, 0, 0, 0, 0, (uint32_t)a.xw};
    int k = 0;
    for (int64_t r0 = rb; r0 < re; r0 += R, ++k) {
        const int s = k % a.ns;
        mbar_wait(full + s, (uint32_t)(k / a.ns) & 1u);
        const int rows = (int)(re - r0 < R ? re - r0 : R);
        const int64_t* rp = st_rp(s);
        const StagedRange sr = staged_range(rp[0], rp[rows], a.nnz, a.nb);
        body.s_col = st_col(s);
        body.s_val = st_val(s);
        body.cb = sr.cb;
        body.vb = sr.vb;
        body.cn = (uint32_t)sr.cn;
        body.vn = (uint32_t)sr.vn;
        if (a.xw > 0) {
            body.lo = win_lo(r0);
            const int64_t hi = win_hi(r0);
            body.span = hi > body.lo ? (uint32_t)(hi - body.lo) : 0u;
            body.org = body.lo - (body.lo % a.xw);
        }
        auto gather = [&](Loop (&L)[U], Step (&st)[U], bool) {
            int cnt = 0;
#pragma unroll
            for (int u = 0; u < U; ++u) {
                const int off = u * G + cg;
                if (off < rows) {
                    const int64_t bb = rp[off];
                    L[u] = Loop{rp[off + 1] - bb, bb};
                    st[u].i = r0 + off;
                    ++cnt;
                } else {
                    L[u].trip = 0;
                }
            }
            return cnt;
        };
        simd_batch<S, MODE, OP, U>(body, g, slot, gather);
        __syncwarp();
        if (lane == 0) mbar_arrive(empty + s);
    }
    auto done = [&](Loop (&L)[U], Step (&)[U], bool) {
#pragma unroll
        for (int u = 0; u < U; ++u) L[u].trip = 0;
        return -1;
    };
    simd_batch<S, MODE, OP, U>(body, g, slot, done);
}

}  // namespace nest
