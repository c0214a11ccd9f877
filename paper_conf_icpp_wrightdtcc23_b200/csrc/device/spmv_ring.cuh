// spmv_ring.cuh -- a8 CSR SpMV with the team's x window and row bounds staged
// in shared memory by a copy warp (nest_desc.x_halo > 0): the north_star's
// "shared staging of x tiles", without team barriers.
//
// Why: with x gathered through L1 every nonzero costs one L1 data-pipe
// wavefront (the 32 lanes of a gather touch ~32 different 128-byte lines), and
// that pipe bounds the unstaged kernel on the banded matrices of SURVEY.md
// §8(d) (profiles/r01_l2_traffic_experiments.md).  A gather served from shared
// memory costs a few bank-conflict wavefronts per warp instead.  Each row's
// bounds rowptr[i], rowptr[i+1] arrive in shared memory ahead of use, so the
// per-row dependent chain is one DRAM trip (colind/val) instead of two.
//
// Levels, as in nest_kernel: teams (blocks) -> parallel (SIMD groups of S
// lanes over rows) -> simd (lanes over a row's nonzeros, Fig 8, PAPER.md:
// 830-840; or over 128-bit pairs of nonzeros with NEST_F_VEC128, R1/R20).
// Team b owns the contiguous rows [rb, re) (blocked "teams distribute", R6) and
// walks them in rounds of R = G*KB rows: in round k group g runs the KB rows
// rb + k*R + m*G + g (m < KB).  Every group of a warp runs every round (rows
// past re are empty loops that store nothing), so warps stay converged and the
// group's shuffles use the full-warp mask (SimdGroup<S, true>).
//
// The last warp of the team is its x copy engine (one elected lane): it walks
// the rounds and bulk-copies (cp.async.bulk, the TMA engine) every x segment
// (SEG doubles, global column c in segment c / SEG) the round's window
//   [lo_k, hi_k) = [rb + k*R - H, rb + (k+1)*R + H) ∩ [0, ncols)
// reaches into a ring of NS segment slots (segment s -> slot (s - s_first) mod
// NS).  Each slot has a "full" mbarrier (transaction bytes of its copy) and an
// "empty" mbarrier (one arrival per consumer warp).  A consumer warp waits for
// the full barriers of its round, runs the round, and releases every segment
// the next round's window no longer reaches; the copy engine refills a slot
// once every consumer warp has released it, so the warps drift apart by up to
// the ring's slack and nobody waits at a team barrier.  A column inside the
// round's resident segments reads the ring, any other column reads x from
// global memory: the result does not depend on H.  Each consumer warp
// prefetches its own rows' bounds rowptr[i], rowptr[i+1] D rounds ahead into a
// private shared-memory stage with per-lane asynchronous copies (cp.async), so
// the per-row dependent chain is one DRAM trip (colind/val) instead of two.
#pragma once

#include "bodies/bodies.cuh"
#include "device/ptx.cuh"

namespace nest {

constexpr int kRingSeg = 256;   // x segment: 256 doubles (2 KiB), a multiple of 16 bytes
constexpr int kRingDepth = 4;   // row-bound stages per consumer warp (prefetch distance in rounds)

__device__ __forceinline__ double lds_f64(uint32_t addr) {
    double v;
    asm volatile("ld.shared.f64 %0, [%1];" : "=d"(v) : "r"(addr));
    return v;
}
__device__ __forceinline__ int64_t lds_s64(uint32_t addr) {
    int64_t v;
    asm volatile("ld.shared.s64 %0, [%1];" : "=l"(v) : "r"(addr));
    return v;
}
// A ring position: slot index and the parity of the slot's current use.
struct RingPos {
    int32_t slot;
    uint32_t phase;
    __device__ __forceinline__ void next(int32_t n) {
        if (++slot == n) slot = 0, phase ^= 1u;
    }
};

// x access policy of the ring (bodies.cuh XA): resident window or global gather.
struct XRing {
    const double* x;
    const double* ring;  // slot 0 of the shared-memory window
    int32_t base_c;      // first column of the round's resident window
    uint32_t span;       // columns in the window
    uint32_t base_pos;   // ring position (doubles) of base_c
    uint32_t xw;         // ring capacity (doubles)
    __device__ __forceinline__ double operator()(int32_t c) const {
        const uint32_t d = (uint32_t)(c - base_c);
        if (d < span) {
            uint32_t p = d + base_pos;
            p = p >= xw ? p - xw : p;
            return ring[p];
        }
        return __ldg(x + c);
    }
};

struct RingArgs {
    const int64_t* rowptr;
    const int32_t* col;
    const double* val;
    const double* x;
    double* y;
    int64_t nrows;
    int64_t ncols;
    int64_t nnz;
    int64_t per_team;    // rows per team
    int32_t halo;        // H
    int32_t nseg;        // NS: x ring slots of kRingSeg doubles
    int32_t depth;       // D: row-bound stages per warp (rounds prefetched ahead)
    int32_t stage;       // int64 entries per stage: KB * (32/S + 1), even
    int32_t kb;          // rows per group per round
    int32_t slot_bytes;  // generic sharing-space slot per group
    unsigned char* gfallback;
    FastDivU32 nseg_div; // division by NS (ring slot / phase of a segment)
};

// Shared-memory layout of one team (bytes):
//   x ring | row-bound stages [warp][D][stage] | x barriers | sharing space.
struct RingLayout {
    int32_t x_off, rp_off, bar_off, sharing_off, total;
    __host__ __device__ static RingLayout of(int32_t nseg, int32_t nwarps, int32_t depth, int32_t stage,
                                             int32_t sharing) {
        RingLayout l;
        l.x_off = 0;
        l.rp_off = nseg * kRingSeg * 8;
        l.bar_off = l.rp_off + nwarps * depth * stage * 8;
        l.sharing_off = l.bar_off + 2 * nseg * 8;
        l.sharing_off = (l.sharing_off + 15) & ~15;
        l.total = l.sharing_off + sharing;
        return l;
    }
};

// The window's segments of round k: [seg_lo(k), seg_hi(k)).
struct RingGeom {
    int64_t rb, R, H, ncols;
    __device__ __forceinline__ int64_t seg_lo(int64_t k) const {
        int64_t lo = rb + k * R - H;
        lo = lo < 0 ? 0 : (lo > ncols ? ncols : lo);
        return lo / kRingSeg;
    }
    __device__ __forceinline__ int64_t seg_hi(int64_t k) const {
        int64_t hi = rb + (k + 1) * R + H;
        hi = hi > ncols ? ncols : hi;
        return (hi + kRingSeg - 1) / kRingSeg;
    }
};

__device__ __forceinline__ void cp_async8(uint32_t dst, const void* src) {
    asm volatile("cp.async.ca.shared.global [%0], [%1], 8;\n" ::"r"(dst), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;\n" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() { asm volatile("cp.async.wait_group %0;\n" ::"n"(N) : "memory"); }

// TPS: teams per SM the launch is sized for: two teams of at most 768 threads
// (40 registers), or one team of up to 1024 (64 registers).
// D: row-bound stages per warp (prefetch distance in rounds).
template <int S, int MODE, int OP, int TPS, class Body>
__global__ void __launch_bounds__(TPS == 2 ? 768 : 1024, TPS) spmv_ring_kernel(const Body body, const RingArgs a) {
    using Loop = typename Body::Loop;
    using Step = typename Body::Step;
    constexpr int D = kRingDepth;
    extern __shared__ __align__(16) unsigned char smem[];
    const int nw = (int)(blockDim.x >> 5);
    const int nc = nw - 1;   // consumer warps; the last warp is the copy engine
    const int warp = (int)(threadIdx.x >> 5);
    const int lane = (int)(threadIdx.x & 31);
    const int G = nc * 32 / S;
    const int64_t R = (int64_t)G * a.kb;
    const int64_t rb = (int64_t)blockIdx.x * a.per_team;
    if (rb >= a.nrows) return;   // whole team: no barrier follows
    const int64_t re = rb + a.per_team < a.nrows ? rb + a.per_team : a.nrows;
    const int32_t nrounds = (int32_t)((re - rb + R - 1) / R);
    const RingGeom geo{rb, R, (int64_t)a.halo, a.ncols};
    const int64_t s_first = geo.seg_lo(0);
    const RingLayout lay = RingLayout::of(a.nseg, nc, D, a.stage, 0);
    double* xring = reinterpret_cast<double*>(smem + lay.x_off);
    uint64_t* full_x = reinterpret_cast<uint64_t*>(smem + lay.bar_off);
    uint64_t* empty_x = full_x + a.nseg;
    unsigned char* sharing = smem + lay.sharing_off;

    if (threadIdx.x == 0) {
        for (int i = 0; i < a.nseg; ++i) mbar_init(&full_x[i], 1), mbar_init(&empty_x[i], (uint32_t)nc);
        mbar_fence_init();
    }
    __syncthreads();

    if (warp == nc) {
        // ------------------------------------------------ the x copy engine
        if (lane != 0) return;
        RingPos px{0, 0u};
        int32_t uses_x = 0;   // fills so far (a slot's first fill waits for nothing)
        const int64_t s_end = geo.seg_hi(nrounds - 1);
        for (int64_t s_next = s_first; s_next < s_end; ++s_next) {
            if (uses_x >= a.nseg) mbar_wait(&empty_x[px.slot], px.phase ^ 1u);
            const int64_t c0 = s_next * kRingSeg;
            const int64_t c1 = c0 + kRingSeg < a.ncols ? c0 + kRingSeg : a.ncols;
            const int64_t cb = c1 & ~(int64_t)1;   // c0 is even: [c0, cb) in 16-byte units
            double* dst = xring + (int64_t)px.slot * kRingSeg;
            if (c1 > cb) dst[cb - c0] = __ldg(a.x + cb);   // odd tail: released by the arrive
            mbar_arrive_expect_tx(&full_x[px.slot], (uint32_t)((cb - c0) * 8));
            if (cb > c0) bulk_g2s(dst, a.x + c0, (uint32_t)((cb - c0) * 8), &full_x[px.slot]);
            px.next(a.nseg);
            ++uses_x;
        }
        return;
    }

    // ---------------------------------------------------- consumer warps
    // Nothing but the round index is carried from round to round: every window
    // quantity is recomputed from k (so the body's pointers stay kernel
    // parameters and the loop fits 32 registers); 32-bit columns (int32 colind).
    const SimdGroup<S, true> g;   // every group of the warp runs every round
    const int64_t gid = (int64_t)blockIdx.x * G + g.group();
    Slot<Loop, 1>* slot = group_slot<MODE, Loop, 1>(sharing, a.slot_bytes, a.gfallback, g.group(), gid);
    constexpr int GW = 32 / S;   // groups (rows) per warp per sub-batch
    constexpr int per_m = GW + 1;
    const int32_t rows = (int32_t)(re - rb);
    // this warp's row-bound stages: stage q holds, per sub-batch m, the GW + 1 bounds
    // rowptr[rb + k*R + m*G + warp*GW + j], j = 0..GW, of round k = q (mod D)
    const uint32_t my_stages = smem_u32(smem + lay.rp_off) + (uint32_t)(warp * D * a.stage * 8);
    auto prefetch = [&](int32_t k) {   // every lane commits one group per call (possibly empty)
        if (k < nrounds) {
            const uint32_t st = my_stages + (uint32_t)((k % D) * a.stage * 8);
            for (int32_t idx = lane; idx < a.kb * per_m; idx += 32) {
                const int32_t m = idx / per_m, j = idx - m * per_m;
                const int32_t rel = k * (int32_t)R + m * G + warp * GW + j;   // <= rows: rowptr has nrows + 1 entries
                if (rel <= rows) cp_async8(st + (uint32_t)idx * 8u, a.rowptr + rb + rel);
            }
        }
        cp_async_commit();
    };
#pragma unroll
    for (int q = 0; q < D; ++q) prefetch(q);
    // segment s of the team lives in slot (s - s_first) mod NS, its fills alternate parity
    auto seg_slot = [&](int32_t s, uint32_t& phase) {
        const uint32_t j = (uint32_t)(s - (int32_t)s_first);
        const uint32_t q = a.nseg_div.div(j);
        phase = q & 1u;
        return (int32_t)(j - q * (uint32_t)a.nseg);
    };
    for (int32_t k = 0; k < nrounds; ++k) {
        const int32_t sA = (int32_t)geo.seg_lo(k);
        const int32_t sB = (int32_t)geo.seg_hi(k);
        for (int32_t s = k > 0 ? (int32_t)geo.seg_hi(k - 1) : (int32_t)s_first; s < sB; ++s) {
            uint32_t ph;
            const int32_t sl = seg_slot(s, ph);
            mbar_wait(&full_x[sl], ph);
        }
        uint32_t ph_unused;
        Body b = body;   // the round's window; the rest are kernel parameters
        b.x.ring = xring;
        b.x.base_c = sA * kRingSeg;
        const int32_t cB = sB * kRingSeg < (int32_t)a.ncols ? sB * kRingSeg : (int32_t)a.ncols;
        b.x.span = (uint32_t)(cB > b.x.base_c ? cB - b.x.base_c : 0);
        b.x.base_pos = (uint32_t)(seg_slot(sA, ph_unused) * kRingSeg);
        cp_async_wait<D - 1>();   // this lane's copies of round k have landed ...
        __syncwarp();             // ... and every lane's are visible to the warp
        const int32_t k0 = k * (int32_t)R;   // first row of the round, relative to rb
        const uint32_t st = my_stages + (uint32_t)((k % D) * a.stage * 8);
        for (int m = 0; m < a.kb; ++m) {
            const int32_t rel = m * G + g.group();
            const bool valid = k0 + rel < rows;
            const uint32_t bnd = st + (uint32_t)((m * per_m + (g.group() - warp * GW)) * 8);
            if constexpr (MODE == MODE_SPMD || S == 1) {
                // every lane reads the bounds (a shared-memory broadcast) -- PAPER.md:713-723
                int64_t lb = 0, le = 0;
                if (valid) lb = lds_s64(bnd), le = lds_s64(bnd + 8u);
                const Loop L[1] = {Body::loop_of(lb, le)};
                typename Body::Acc acc[1];
                workshare_simd<S, OP, 1>(b, g, L, acc);   // Fig 8
                group_reduce<S, OP, 1>(g, acc);           // a6
                if (valid && g.leader()) {                // a7
                    Step sp;
                    sp.i = (decltype(sp.i))(rb + (k0 + rel));
                    b.epilogue(sp, acc[0]);
                }
            } else {
                // generic: the SIMD main reads the bounds and posts them (Figs 4/6)
                auto gather = [&](Loop (&L)[1], Step (&sp)[1], bool) {
                    int64_t lb = 0, le = 0;
                    if (valid) lb = lds_s64(bnd), le = lds_s64(bnd + 8u);
                    L[0] = Body::loop_of(lb, le);
                    sp[0].i = (decltype(sp[0].i))(rb + (k0 + rel));
                    return valid ? 1 : 0;   // an empty loop keeps the workers in step
                };
                simd_batch<S, MODE, OP, 1>(b, g, slot, gather);
            }
        }
        // the stage is free again: prefetch round k + D into it
        __syncwarp();
        prefetch(k + D);
        // release every segment the next window no longer reaches
        if (lane == 0) {
            const int32_t sA_next = k + 1 < nrounds ? (int32_t)geo.seg_lo(k + 1) : sB;
            for (int32_t s = sA; s < sA_next; ++s) {
                uint32_t ph;
                mbar_arrive(&empty_x[seg_slot(s, ph)]);
            }
        }
    }
    cp_async_wait<0>();
    if constexpr (MODE != MODE_SPMD && S > 1) {
        // end of the parallel region: the main posts the null fn
        auto done = [&](Loop (&L)[1], Step (&)[1], bool) {
            L[0].trip = 0;
            return -1;
        };
        simd_batch<S, MODE, OP, 1>(body, g, slot, done);
    }
}

}  // namespace nest
