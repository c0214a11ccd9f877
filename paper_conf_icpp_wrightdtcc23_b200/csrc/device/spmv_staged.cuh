// spmv_staged.cuh -- a8 CSR SpMV, B200 pipeline variant (NEST_F_STAGED).
//
// The same three levels and mode engine as nest_kernel -- teams (CTAs) ->
// parallel (SIMD groups over rows) -> simd (lanes over a row's nonzeros,
// Fig 8 cyclic) with SPMD or generic execution of the parallel region
// (simd_batch) -- with the memory traffic decoupled from the loop nest:
//
//   * warp 0 of every team is a PRODUCER.  It walks the team's contiguous
//     block of rows in chunks sized by NONZEROS: a chunk is the longest run of
//     rows (at most RMAX) whose nonzeros fit one stage of NB entries.  For each
//     chunk it copies rowptr into the stage, issues 1D bulk asynchronous
//     copies (cp.async.bulk, the TMA engine: SASS UBLKCP) of the chunk's
//     colind and val, and of the newly needed tail of the x window into a ring
//     buffer, and signals a "full" mbarrier (expect_tx).  NS stages are in
//     flight; a stage is refilled after every consumer warp arrived on its
//     "empty" mbarrier.
//   * warps 1..kGatherWarps are GATHERERS: once a chunk has landed they scan
//     its colind and, for every column outside the x window [r0 - H, r1 + H),
//     fetch xv[q] = x[col[q]] with an asynchronous 8-byte copy (cp.async)
//     into the stage, then signal a second mbarrier ("gathered") through
//     arrivals that fire when their copies complete -- no warp ever waits on a
//     global-memory gather.
//   * the remaining warps are CONSUMERS: the SIMD groups.  They run the
//     three-level loop nest over the staged rows, G*U rows per batch, with
//     acc = fma(val[q], x[col[q]], acc) in Fig 8's cyclic order, x from the
//     ring (window) or the gathered copy (far): all operands in shared memory.  A row longer than a stage is read from global memory.
//     Results are identical to nest_kernel for any H, NB, NS (same per-lane
//     order, same fma, same butterfly).
//
// Every consumer warp runs the same number of batches per chunk, so the group
// collectives are warp-uniform (SimdGroup<S, true>).
#pragma once

#include "bodies/bodies.cuh"
#include "device/ptx.cuh"

namespace nest {

// Chunk header written by the producer (rows < 0 marks the end of the team's rows).
struct ChunkHdr {
    int64_t r0;
    int64_t cb;          // first staged nonzero (multiple of 4); stage entry q holds nonzero cb + q
    int64_t staged_end;  // nonzeros [cb, staged_end) are in the stage
    int32_t rows;        // rows in the chunk; < 0: end of the team's rows
    int32_t lo, hi;      // x window [lo, hi)
    int32_t pad;
};

struct StagedLoop {
    int32_t trip;
    int32_t kl;      // first nonzero of the row, relative to the stage (cb)
    int64_t k0;      // first nonzero of the row, global index
};

// Body, fast path: the whole row is in the stage; x from the ring when the
// column is in the window, else from the stage's gathered copy.
struct SpmvStagedBody {
    using Acc = double;
    using Loop = StagedLoop;
    static constexpr int kLoopUnroll = 1;   // shared-memory operands: no MLP to gain, less code
    struct Step {
        int64_t i;
    };
    double* y;
    const double* s_val;
    const int32_t* s_col;
    const double* s_xv;
    const double* ring;
    int32_t lo;
    uint32_t span;
    uint32_t lo_slot;   // ring slot of column lo
    uint32_t xw;

    template <int OP>
    __device__ __forceinline__ double accum(const Loop& L, int32_t j, double acc) const {
        const int32_t q = L.kl + j;
        const int32_t c = s_col[q];
        const uint32_t d = (uint32_t)(c - lo);
        double xv;
        if (d < span) {
            uint32_t sl = d + lo_slot;
            sl = sl >= xw ? sl - xw : sl;
            xv = ring[sl];
        } else {
            xv = s_xv[q];
        }
        return Red<OP, double>::accum(acc, s_val[q], xv);
    }
    __device__ __forceinline__ void epilogue(const Step& st, double total) const { y[st.i] = total; }
};

// Body, overflow path: a row longer than a stage, everything from global memory.
struct SpmvStagedOvfBody : SpmvStagedBody {
    const int32_t* col;
    const double* val;
    const double* x;
    template <int OP>
    __device__ __forceinline__ double accum(const Loop& L, int32_t j, double acc) const {
        const int64_t k = L.k0 + j;
        return Red<OP, double>::accum(acc, __ldg(val + k), __ldg(x + __ldg(col + k)));
    }
};

// Warps that gather x for the staged nonzeros (between the producer and the consumers).
constexpr int kGatherWarps = 2;

__device__ __forceinline__ void cp_async8_s(void* smem_dst, const void* gsrc) {
    asm volatile("cp.async.ca.shared.global [%0], [%1], 8;\n" ::"r"(smem_u32(smem_dst)), "l"(gsrc) : "memory");
}
// mbarrier arrival that fires once all prior cp.async of this thread completed
__device__ __forceinline__ void cp_async_mbar_arrive_noinc(uint64_t* bar) {
    asm volatile("cp.async.mbarrier.arrive.noinc.shared::cta.b64 [%0];\n" ::"r"(smem_u32(bar)) : "memory");
}

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
    int32_t rmax;        // rows per chunk at most
    int32_t slot_bytes;  // generic sharing-space slot
    unsigned long long* trace;   // developer tracing (NEST_TRACE): pipeline timestamps of team 0
    unsigned char* gfallback;
};

__device__ __forceinline__ unsigned long long gtimer() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
    return t;
}

// Shared-memory layout (offsets 16-byte aligned).
struct StagedLayout {
    uint32_t stage0, stage_stride, xv_off, col_off, rp_off, hdr_off, bars, sharing, total;
};
__host__ __device__ __forceinline__ StagedLayout staged_layout(int32_t xw, int32_t nb, int32_t ns, int32_t rmax,
                                                            int32_t sharing_bytes) {
    auto al = [](uint32_t v) { return (v + 15u) & ~15u; };
    StagedLayout l;
    l.stage0 = al((uint32_t)xw * 8u);
    l.xv_off = al((uint32_t)nb * 8u);
    l.col_off = l.xv_off + al((uint32_t)nb * 8u);
    l.rp_off = l.col_off + al((uint32_t)nb * 4u);
    l.hdr_off = l.rp_off + al((uint32_t)(rmax + 1) * 8u);
    l.stage_stride = l.hdr_off + al((uint32_t)sizeof(ChunkHdr));
    l.bars = l.stage0 + (uint32_t)ns * l.stage_stride;
    l.sharing = al(l.bars + (uint32_t)ns * 24u);   // full, gathered, empty
    l.total = l.sharing + (uint32_t)sharing_bytes;
    return l;
}

template <int S, int MODE, int OP, int U>
__global__ void __launch_bounds__(1024, 1) spmv_staged_kernel(const StagedArgs a) {
    using Loop = StagedLoop;
    using Step = SpmvStagedBody::Step;
    extern __shared__ __align__(16) unsigned char smem[];
    const int nconsumer = (int)blockDim.x - 32 * (1 + kGatherWarps);
    const int G = nconsumer / S;                 // consumer SIMD groups per team
    const int B = G * U;                         // rows per batch
    const int32_t sharing_bytes = MODE == MODE_GENERIC_SMEM ? a.slot_bytes * G : 0;
    const StagedLayout lay = staged_layout(a.xw, a.nb, a.ns, a.rmax, sharing_bytes);
    double* ring = reinterpret_cast<double*>(smem);
    uint64_t* full = reinterpret_cast<uint64_t*>(smem + lay.bars);
    uint64_t* gathered = full + a.ns;
    uint64_t* empty = gathered + a.ns;
    auto stage = [&](int s) { return smem + lay.stage0 + (uint32_t)s * lay.stage_stride; };

    int64_t per_team = (a.nrows + gridDim.x - 1) / gridDim.x;
    per_team = (per_team + 1) & ~(int64_t)1;   // even: 16-byte aligned rowptr / x copies
    const int64_t rb0 = (int64_t)blockIdx.x * per_team;
    const int64_t rb = rb0 < a.nrows ? rb0 : a.nrows;
    const int64_t re = rb + per_team < a.nrows ? rb + per_team : a.nrows;
    const int warp = (int)(threadIdx.x >> 5), lane = (int)(threadIdx.x & 31);

    if (threadIdx.x == 0) {
        for (int s = 0; s < a.ns; ++s) {
            mbar_init(full + s, 1);
            mbar_init(gathered + s, 2u * 32u * kGatherWarps);
            mbar_init(empty + s, (uint32_t)(nconsumer / 32 + kGatherWarps));
        }
        mbar_fence_init();
    }
    __syncthreads();

    if (warp == 0) {
        // ------------------------------------------------------------ producer
        // Chunks of R rows (R, H and the team's first row are even, so every
        // bulk copy below is 16-byte aligned except at the very end of an array).
        const int R = a.rmax;
        int64_t r0 = rb, xdone = 0;
        int64_t b = r0 < re ? __ldg(a.rowptr + r0) : 0;
        // chunk ends rowptr[r0 + (k+1)R] for 32 chunks per warp-wide load, two windows ahead,
        // so the producer never waits on a dependent global load
        auto chunk_end = [&](int64_t kk) {
            const int64_t r = rb + (kk + 1) * (int64_t)R;
            return __ldg(a.rowptr + (r < re ? r : re));
        };
        int64_t ends_cur = rb < re ? chunk_end(lane) : 0;
        int64_t ends_nxt = rb < re ? chunk_end(32 + lane) : 0;
        for (int k = 0;; ++k) {
            const int s = k % a.ns;
            const int rows = (int)(re - r0 < R ? re - r0 : R);
            if (k > 0 && (k & 31) == 0) {
                ends_cur = ends_nxt;
                if (r0 < re) ends_nxt = chunk_end(k + 32 + lane);
            }
            const int64_t e = __shfl_sync(0xffffffffu, ends_cur, k & 31);
            if (k >= a.ns) mbar_wait(empty + s, (uint32_t)((k / a.ns) - 1) & 1u);
            if (a.trace && blockIdx.x == 0 && lane == 0 && k < 64) a.trace[k] = gtimer();
            unsigned char* st = stage(s);
            ChunkHdr* hdr = reinterpret_cast<ChunkHdr*>(st + lay.hdr_off);
            if (r0 >= re) {
                if (lane == 0) {
                    hdr->rows = -1;
                    mbar_arrive(full + s);
                }
                break;
            }
            int64_t* rp = reinterpret_cast<int64_t*>(st + lay.rp_off);
            // nonzeros [cb, cb + n4) by bulk copy (16-byte granules, at most NB), plus the
            // last < 4 entries of the arrays by hand when the chunk reaches them
            const int64_t cb = b & ~(int64_t)3;
            int64_t ce4 = (e + 3) & ~(int64_t)3;
            if (ce4 > cb + a.nb) ce4 = cb + a.nb;
            const int64_t cmax = a.nnz & ~(int64_t)3;
            int64_t n4 = (ce4 < cmax ? ce4 : cmax) - cb;
            if (n4 < 0) n4 = 0;
            int64_t staged_end = cb + n4;
            if (ce4 > cmax && e > cmax && e - cb <= a.nb) {
                // by the arriving lane itself, so its release covers these stores
                if (lane == 0)
                    for (int64_t tk = cmax; tk < e; ++tk) {
                        reinterpret_cast<int32_t*>(st + lay.col_off)[tk - cb] = __ldg(a.col + tk);
                        reinterpret_cast<double*>(st)[tk - cb] = __ldg(a.val + tk);
                    }
                staged_end = e;
            }
            // rowptr[r0 .. r0+rows]: even-length bulk part, the rest by hand
            const int nrp = rows & ~1;
            if (lane == 0) {
                rp[rows] = e;
                if (rows & 1) rp[rows - 1] = __ldg(a.rowptr + r0 + rows - 1);
            }
            // x window [lo, hi); new tail [xa, xb)
            int64_t lo = 0, hi = 0, xa2 = 0, xb2 = 0;
            if (a.xw > 0) {
                lo = r0 - a.halo > 0 ? r0 - a.halo : 0;
                hi = r0 + rows + a.halo < a.ncols ? r0 + rows + a.halo : a.ncols;
                const int64_t xa = xdone > lo ? xdone : lo;
                const int64_t xb = hi > xa ? hi : xa;
                xdone = xb;
                xa2 = (xa + 1) & ~(int64_t)1;
                xb2 = xb & ~(int64_t)1;
                if (xb2 < xa2) xb2 = xa2;
                if (lane == 0 && (xa & 1) && xa < xb) ring[(uint32_t)(xa % a.xw)] = __ldg(a.x + xa);
                if (lane == 0 && (xb & 1) && xb - 1 >= xa) ring[(uint32_t)((xb - 1) % a.xw)] = __ldg(a.x + xb - 1);
            }
            if (lane == 0) {
                hdr->r0 = r0;
                hdr->cb = cb;
                hdr->staged_end = staged_end;
                hdr->rows = rows;
                hdr->lo = (int32_t)lo;
                hdr->hi = (int32_t)hi;
            }
            __syncwarp();
            if (lane == 0) {
                const uint32_t xbytes = (uint32_t)(xb2 - xa2) * 8u;
                mbar_arrive_expect_tx(full + s, (uint32_t)n4 * 12u + (uint32_t)nrp * 8u + xbytes);
                if (nrp) bulk_g2s(rp, a.rowptr + r0, (uint32_t)nrp * 8u, full + s);
                if (n4) {
                    bulk_g2s(st, a.val + cb, (uint32_t)n4 * 8u, full + s);
                    bulk_g2s(st + lay.col_off, a.col + cb, (uint32_t)n4 * 4u, full + s);
                }
                if (xbytes) {
                    const uint32_t slot = (uint32_t)(xa2 % a.xw);
                    const uint32_t n = (uint32_t)(xb2 - xa2);
                    const uint32_t n1 = slot + n <= (uint32_t)a.xw ? n : (uint32_t)a.xw - slot;
                    bulk_g2s(ring + slot, a.x + xa2, n1 * 8u, full + s);
                    if (n1 < n) bulk_g2s(ring, a.x + xa2 + n1, (n - n1) * 8u, full + s);
                }
            }
            r0 += rows;
            b = e;
        }
        return;
    }

    if (warp <= kGatherWarps) {
        // ----------------------------------------------------------- gatherers
        const int gt = (warp - 1) * 32 + lane;
        for (int k = 0;; ++k) {
            const int s = k % a.ns;
            mbar_wait(full + s, (uint32_t)(k / a.ns) & 1u);
            if (a.trace && blockIdx.x == 0 && gt == 0 && k < 64) a.trace[64 + k] = gtimer();
            unsigned char* st = stage(s);
            const ChunkHdr& h = *reinterpret_cast<const ChunkHdr*>(st + lay.hdr_off);
            const int rows = h.rows;
            if (rows >= 0) {
                const int64_t* rp = reinterpret_cast<const int64_t*>(st + lay.rp_off);
                const int64_t e = rp[rows] < h.staged_end ? rp[rows] : h.staged_end;
                const int32_t q1 = e > h.cb ? (int32_t)(e - h.cb) : 0;
                const int32_t* sc = reinterpret_cast<const int32_t*>(st + lay.col_off);
                double* xv = reinterpret_cast<double*>(st + lay.xv_off);
                const int32_t lo = h.lo;
                const uint32_t span = (uint32_t)(h.hi - h.lo);
#pragma unroll 4
                for (int32_t q = (int32_t)(rp[0] - h.cb) + gt; q < q1; q += 32 * kGatherWarps) {
                    const int32_t c = sc[q];
                    if ((uint32_t)(c - lo) >= span) cp_async8_s(xv + q, a.x + c);   // outside the window
                }
            }
            mbar_arrive(gathered + s);
            cp_async_mbar_arrive_noinc(gathered + s);  // fires when this lane's copies landed
            if (rows < 0) break;
            __syncwarp();
            if (lane == 0) mbar_arrive(empty + s);     // done reading colind / the ring
        }
        return;
    }

    // -------------------------------------------------------------- consumers
    const SimdGroup<S, true> g;
    const int cg = g.group() - 32 * (1 + kGatherWarps) / S;   // consumer group index
    const int64_t gid = (int64_t)blockIdx.x * G + cg;
    Slot<Loop, U>* slot = group_slot<MODE, Loop, U>(smem + lay.sharing, a.slot_bytes, a.gfallback, cg, gid);
    SpmvStagedOvfBody body;
    body.y = a.y;
    body.ring = ring;
    body.xw = (uint32_t)a.xw;
    body.col = a.col;
    body.val = a.val;
    body.x = a.x;
    for (int k = 0;; ++k) {
        const int s = k % a.ns;
        mbar_wait(gathered + s, (uint32_t)(k / a.ns) & 1u);
        if (a.trace && blockIdx.x == 0 && threadIdx.x == 32 * (1 + kGatherWarps) && k < 64)
            a.trace[128 + k] = gtimer();
        const unsigned char* st = stage(s);
        const ChunkHdr hdr = *reinterpret_cast<const ChunkHdr*>(st + lay.hdr_off);
        if (hdr.rows < 0) break;
        const int64_t* rp = reinterpret_cast<const int64_t*>(st + lay.rp_off);
        body.s_val = reinterpret_cast<const double*>(st);
        body.s_col = reinterpret_cast<const int32_t*>(st + lay.col_off);
        body.s_xv = reinterpret_cast<const double*>(st + lay.xv_off);
        body.lo = hdr.lo;
        body.span = (uint32_t)(hdr.hi - hdr.lo);
        body.lo_slot = a.xw > 0 ? (uint32_t)(hdr.lo % a.xw) : 0u;
        // a chunk whose nonzeros did not all fit the stage (rows longer than NB, rare)
        // takes the global path; the choice is chunk-uniform
        const bool ovf = rp[hdr.rows] > hdr.staged_end;
        for (int base = 0; base < hdr.rows; base += B) {
            auto gather = [&](Loop (&L)[U], Step (&sp)[U], bool) {
                int n = 0;
#pragma unroll
                for (int u = 0; u < U; ++u) {
                    const int off = base + u * G + cg;
                    if (off < hdr.rows) {
                        const int64_t bb = rp[off];
                        L[u] = Loop{(int32_t)(rp[off + 1] - bb), (int32_t)(bb - hdr.cb), bb};
                        sp[u].i = hdr.r0 + off;
                        ++n;
                    } else {
                        L[u].trip = 0;
                    }
                }
                return n;   // an empty batch keeps the workers in step; never ends the region
            };
            if (!ovf)
                simd_batch<S, MODE, OP, U>(static_cast<const SpmvStagedBody&>(body), g, slot, gather);
            else
                simd_batch<S, MODE, OP, U>(body, g, slot, gather);
        }
        __syncwarp();
        if (lane == 0) mbar_arrive(empty + s);
        if (a.trace && blockIdx.x == 0 && threadIdx.x == 32 * (1 + kGatherWarps) && k < 64)
            a.trace[192 + k] = gtimer();
    }
    auto done = [&](Loop (&L)[U], Step (&)[U], bool) {
#pragma unroll
        for (int u = 0; u < U; ++u) L[u].trip = 0;
        return -1;
    };
    simd_batch<S, MODE, OP, U>(static_cast<const SpmvStagedBody&>(body), g, slot, done);
}

}  // namespace nest
