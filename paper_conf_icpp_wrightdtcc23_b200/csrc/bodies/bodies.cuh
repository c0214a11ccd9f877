// bodies.cuh -- the fixed device loop bodies (a8, a9, a10, probe).
//
// Each body is the compile-time analogue of the outlined WorkFn plus the
// sequential code of its parallel region (the loop body is
// outlined into a function taking (iv, payload); the B200 build instantiates
// it as a template instead of a function pointer -- the if-cascade of
// PAPER.md:794-800 resolved at compile time).  Contract used by engine.cuh:
//   Acc                         accumulator type of the simd reduction
//   Loop {trip, ...}            loop state the SIMD main posts (generic payload)
//   Step                        main-private state needed by the epilogue
//   TeamShared                  per-team shared state (team_begin/team_end)
//   steps(body)                 simd loops per outer iteration (K)
//   prologue(i, r, st, fx, tsh) sequential code before simd loop r of outer
//                               iteration i; side effects only if fx
//   accum<OP>(L, j, acc)        WorkFn(j, args) folded into the accumulator
//   epilogue(st, total)         sequential code after the loop (SIMD main)
#pragma once

#include <cstdint>

#include "device/engine.cuh"

#ifndef NEST_VEC_UNROLL
#define NEST_VEC_UNROLL 1
#endif
// float4 tuples per lane issued as one predicated block by the batched 128-bit body
#ifndef NEST_SCALAR_HEAD
#define NEST_SCALAR_HEAD -1   // -1: per simdlen (SpmvBody::head_for); 0: none
#endif
#ifndef NEST_BVEC_HEAD
#define NEST_BVEC_HEAD -1   // -1: per simdlen (BatchedVecBody::head_for)
#endif
// tuples per lane issued as one predicated block by the 128-bit SpMV body
#ifndef NEST_VEC_HEAD
#define NEST_VEC_HEAD 2
#endif

namespace nest {

// Streaming loads: L1 no-allocate + L2 evict-first policy (read once).
__device__ __forceinline__ int32_t ld_stream(const int32_t* p) { return __ldcs(p); }
__device__ __forceinline__ double ld_stream(const double* p) { return __ldcs(p); }

// L2 cache-policy loads (L1 behaviour unchanged): the streamed matrix is
// evict-first, the gathered x evict-last, so x stays in L2 while the matrix
// streams through it.
__device__ __forceinline__ uint64_t l2_policy_evict_first() {
    uint64_t p;
    asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ uint64_t l2_policy_evict_last() {
    uint64_t p;
    asm("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ int2 ld_pol(const int2* a, uint64_t pol) {
    int2 r;
    asm volatile("ld.global.nc.L2::cache_hint.v2.s32 {%0, %1}, [%2], %3;" : "=r"(r.x), "=r"(r.y) : "l"(a), "l"(pol));
    return r;
}
__device__ __forceinline__ int4 ld_pol(const int4* a, uint64_t pol) {
    int4 r;
    asm volatile("ld.global.nc.L2::cache_hint.v4.s32 {%0, %1, %2, %3}, [%4], %5;"
                 : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(a), "l"(pol));
    return r;
}
__device__ __forceinline__ double2 ld_pol(const double2* a, uint64_t pol) {
    double2 r;
    asm volatile("ld.global.nc.L2::cache_hint.v2.f64 {%0, %1}, [%2], %3;" : "=d"(r.x), "=d"(r.y) : "l"(a), "l"(pol));
    return r;
}
// L1 no-allocate loads for data read exactly once (keeps L1 for the x gathers)
__device__ __forceinline__ int2 ld_na(const int2* a) {
    int2 r;
    asm volatile("ld.global.nc.L1::no_allocate.v2.s32 {%0, %1}, [%2];" : "=r"(r.x), "=r"(r.y) : "l"(a));
    return r;
}
__device__ __forceinline__ int4 ld_na(const int4* a) {
    int4 r;
    asm volatile("ld.global.nc.L1::no_allocate.v4.s32 {%0, %1, %2, %3}, [%4];"
                 : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(a));
    return r;
}
__device__ __forceinline__ double2 ld_na(const double2* a) {
    double2 r;
    asm volatile("ld.global.nc.L1::no_allocate.v2.f64 {%0, %1}, [%2];" : "=d"(r.x), "=d"(r.y) : "l"(a));
    return r;
}
__device__ __forceinline__ double ld_pol(const double* a, uint64_t pol) {
    double r;
    asm volatile("ld.global.nc.L2::cache_hint.f64 %0, [%1], %2;" : "=d"(r) : "l"(a), "l"(pol));
    return r;
}

// ------------------------------------------------------- x access policies
// How the SpMV's simd loop reads x[c] (c a global column index).
// XLocal: x is one array in this GPU's memory (single GPU, or the all-gathered
// x_full of the row-partitioned SpMV).
struct XLocal {
    const double* p;
    __device__ __forceinline__ double operator()(int32_t c) const { return __ldg(p + c); }
};

// Unsigned 32-bit division by a run-time constant d >= 1 (round-up multiplier:
// q = (t + ((n - t) >> 1)) >> (l - 1), t = umulhi(n, m), l = ceil(log2 d)).
struct FastDivU32 {
    uint32_t d, m, s;   // s = l (0 when d == 1)
    static FastDivU32 make(uint32_t d) {
        FastDivU32 f{d, 0u, 0u};
        if (d > 1) {
            uint32_t l = 0;
            while (l < 32 && (1ull << l) < d) ++l;
            f.m = (uint32_t)(((1ull << 32) * ((1ull << l) - d)) / d + 1);
            f.s = l;
        }
        return f;
    }
    __device__ __forceinline__ uint32_t div(uint32_t n) const {
        if (s == 0) return n;
        const uint32_t t = __umulhi(n, m);
        return (t + ((n - t) >> 1)) >> (s - 1);
    }
};

// XPeer (NEXT-4, comm-free row-partitioned SpMV): x stays distributed -- rank
// o owns columns [o*chunk, (o+1)*chunk) in its own memory -- and the simd loop
// gathers x[c] straight from the owner's slice through its peer mapping
// (NVLink loads from the simd lanes; no all-gather).
struct XPeer {
    const double* const* slices;   // device array: nranks peer-mapped slice pointers
    FastDivU32 chunk;
    const double* own;             // this rank's slice (columns [own_lo, own_lo + chunk.d))
    uint32_t own_lo;
    __device__ __forceinline__ double operator()(int32_t c) const {
        const uint32_t d = (uint32_t)c - own_lo;   // the banded columns of local rows: no owner lookup
        if (d < chunk.d) return __ldg(own + d);
        const uint32_t o = chunk.div((uint32_t)c);
        const double* s = reinterpret_cast<const double*>(
            __ldg(reinterpret_cast<const unsigned long long*>(slices) + o));
        return __ldg(s + ((uint32_t)c - o * chunk.d));
    }
};

// ---------------------------------------------------------------- a8 SpMV
// sparse_matvec: outer loop over rows on "teams distribute
// parallel for", inner loop over the row's nonzeros on "simd".  The product is
// reduced in-group (R2) instead of the paper's atomic update.
template <bool HINTS, class I = int64_t, class XA = XLocal>
struct SpmvBody {
    using Acc = double;
    using OuterIndex = I;   // launcher: I = int32_t only when spmv_index32()
    // I: index type of rows and nonzeros (int32_t when they fit: fewer registers)
    struct Loop {
        I trip;   // nonzeros in the row (TripCount)
        I base;   // rowptr[i]
    };
    struct Step {
        I i;
    };
    static constexpr bool kTeamState = false;
    struct TeamShared {
        int unused;
    };
    const int64_t* rowptr;
    const int32_t* col;
    const double* val;
    XA x;   // x access (XLocal: x[c]; XPeer: the owner rank's slice; XRing: the staged window)
    double* y;
    int64_t nnz = 0;

    // the simd loop of the row [b, e): the loop state the sequential code computes
    static __device__ __forceinline__ Loop loop_of(int64_t b, int64_t e) { return Loop{(I)(e - b), (I)b}; }

    static __device__ __forceinline__ int steps(const SpmvBody&) { return 1; }
    static constexpr bool kOneStep = true;
    static __device__ __forceinline__ void team_begin(TeamShared&) {}
    static __device__ __forceinline__ void team_end(const SpmvBody&, TeamShared&) {}

    __device__ __forceinline__ Loop prologue(int64_t i, int, Step& st, bool, TeamShared&) const {
        st.i = (I)i;
        return loop_of(__ldg(rowptr + i), __ldg(rowptr + i + 1));
    }
    template <int OP>
    __device__ __forceinline__ double accum(const Loop& L, I j, double acc) const {
        const I k = L.base + j;
        const int32_t c = HINTS ? ld_stream(col + k) : __ldg(col + k);
        const double v = HINTS ? ld_stream(val + k) : __ldg(val + k);
        return Red<OP, double>::accum(acc, v, x(c));
    }
    // the lane's first head_for(S) nonzeros (j = id, id + S, ...) as one predicated
    // block: every colind/val load, then every x gather, then the folds in order
    // (engine.cuh head_iters; same per-lane order, bit-identical)
    static constexpr int head_for(int S) {
        return NEST_SCALAR_HEAD >= 0 ? NEST_SCALAR_HEAD : (S <= 8 ? 2 : 1);   // 4 at S <= 2 needs 40 registers
    }
    template <int OP, int S>
    __device__ __forceinline__ double accum_head(const Loop& L, int32_t id, double acc) const {
        constexpr int H = head_for(S) > 0 ? head_for(S) : 1;
        int32_t c[H];
        double v[H], xv[H];
#pragma unroll
        for (int h = 0; h < H; ++h) {
            const I j = (I)id + (I)(h * S);
            const I k = L.base + j;
            c[h] = j < L.trip ? (HINTS ? ld_stream(col + k) : __ldg(col + k)) : 0;
            v[h] = j < L.trip ? (HINTS ? ld_stream(val + k) : __ldg(val + k)) : 0.0;
        }
#pragma unroll
        for (int h = 0; h < H; ++h) xv[h] = (I)id + (I)(h * S) < L.trip ? x(c[h]) : 0.0;
#pragma unroll
        for (int h = 0; h < H; ++h)
            if ((I)id + (I)(h * S) < L.trip) acc = Red<OP, double>::accum(acc, v[h], xv[h]);
        return acc;
    }
    __device__ __forceinline__ void epilogue(const Step& st, double total) const { y[st.i] = total; }
};

// ------------------------------------------------- a8 SpMV, 128-bit loads
// NEST_F_VEC128 (V = 2) / NEST_F_VEC128 | NEST_F_VEC_QUAD (V = 4): the simd loop
// runs over V-tuples of nonzeros -- tuple P holds entries VP .. VP+V-1, read
// with 128-bit loads (V = 2: one double2 of val + one int2 of colind; V = 4:
// two double2 + one int4) -- and lane l takes the row's tuples l, l+S, ...
// ("blocked-cyclic", R1: a fixed order different from Fig 8's, so
// real results differ from the scalar path by rounding only).  Entries of a
// boundary tuple that belong to a neighbouring row are skipped; a tuple that
// would read past nnz falls back to scalar loads.
template <bool HINTS, int V, class I = int64_t, class XA = XLocal>
struct SpmvVecBody {
    static_assert(V == 2 || V == 4, "tuple width");
    // I: index type of rows and nonzeros (int32_t when nnz and nrows < 2^31:
    // fewer registers, so two teams of 1024 fit an SM)
    using Acc = double;
    using OuterIndex = I;   // launcher: I = int32_t only when spmv_index32()
    // engine.cuh two_teams_per_sm (U = 1): cap registers at 32 for two teams of 1024
    // per SM -- except quads at simdlen 1, which would spill (measured slower)
    static constexpr bool two_teams_for(int S) { return !(V == 4 && S == 1); }
    static constexpr int kLoopUnroll = NEST_VEC_UNROLL;   // V nonzeros per iteration already
    struct Loop {
        I base;         // rowptr[i]
        int32_t trip;   // tuples covering the row (the simd loop's TripCount)
        int32_t len;    // nonzeros in the row
    };
    struct Step {
        I i;
    };
    static constexpr bool kTeamState = false;
    struct TeamShared {
        int unused;
    };
    const int64_t* rowptr;
    const int32_t* col;
    const double* val;
    XA x;   // x access (XLocal: x[c]; XPeer: the owner rank's slice)
    double* y;
    int64_t nnz;

    static __device__ __forceinline__ int steps(const SpmvVecBody&) { return 1; }
    static constexpr bool kOneStep = true;
    static __device__ __forceinline__ void team_begin(TeamShared&) {}
    static __device__ __forceinline__ void team_end(const SpmvVecBody&, TeamShared&) {}

    // the simd loop of the row [b, e): tuples covering it, from the aligned tuple holding b
    static __device__ __forceinline__ Loop loop_of(int64_t b64, int64_t e64) {
        const I b = (I)b64, e = (I)e64;
        constexpr int kLog = V == 2 ? 1 : 2;
        return Loop{b, e > b ? (int32_t)(((e + V - 1) >> kLog) - (b >> kLog)) : 0, (int32_t)(e - b)};
    }
    __device__ __forceinline__ Loop prologue(int64_t i, int, Step& st, bool, TeamShared&) const {
        st.i = (I)i;
        return loop_of(__ldg(rowptr + i), __ldg(rowptr + i + 1));
    }
    // the tuple starting at entry k0: 128-bit loads, scalar at the end of the arrays
    __device__ __forceinline__ void load_tuple(I k0, int32_t (&c)[V], double (&v)[V]) const {
        if (k0 + V <= (I)nnz) {
            if constexpr (V == 2) {
                const int2 cc = HINTS ? ld_na(reinterpret_cast<const int2*>(col + k0))
                                      : __ldg(reinterpret_cast<const int2*>(col + k0));
                const double2 vv = HINTS ? ld_na(reinterpret_cast<const double2*>(val + k0))
                                         : __ldg(reinterpret_cast<const double2*>(val + k0));
                c[0] = cc.x, c[1] = cc.y, v[0] = vv.x, v[1] = vv.y;
            } else {
                const int4 cc = HINTS ? ld_na(reinterpret_cast<const int4*>(col + k0))
                                      : __ldg(reinterpret_cast<const int4*>(col + k0));
                c[0] = cc.x, c[1] = cc.y, c[2] = cc.z, c[3] = cc.w;
                // the quad's four values in ONE 256-bit load (sm_100 LDG.256; k0 is a
                // multiple of 4, so val + k0 is 32-byte aligned): one L1 tag lookup per
                // 32 bytes of a lane instead of two 128-bit loads
                asm("ld.global.nc.v4.f64 {%0, %1, %2, %3}, [%4];"
                    : "=d"(v[0]), "=d"(v[1]), "=d"(v[2]), "=d"(v[3])
                    : "l"(val + k0));
            }
        } else if constexpr (V == 2) {   // the last entry of the arrays
            c[0] = __ldg(col + k0), v[0] = __ldg(val + k0), c[1] = c[0], v[1] = 0.0;
        } else {
#pragma unroll
            for (int q = 0; q < V; ++q) {
                const I kq = k0 + q < (I)nnz ? k0 + q : k0;
                c[q] = __ldg(col + kq);
                v[q] = __ldg(val + kq);
            }
        }
    }
    template <int OP>
    __device__ __forceinline__ double accum(const Loop& L, int32_t j, double acc) const {
        const I b = L.base;
        const I e = b + L.len;
        constexpr int kLog = V == 2 ? 1 : 2;
        const I k0 = ((b >> kLog) + j) << kLog;   // first entry of the tuple
        int32_t c[V];
        double v[V];
        load_tuple(k0, c, v);
#pragma unroll
        for (int q = 0; q < V; ++q)
            if (k0 + q >= b && k0 + q < e)
                acc = Red<OP, double>::accum(acc, v[q], x(c[q]));
        return acc;
    }
    // the lane's first kHeadIters tuples (j = id, id + S, ...) as one predicated
    // block: all tuple loads, then all x gathers, then the folds in order
    // (engine.cuh head_iters; measured 0.313 -> 0.293 ms on cfg2 at S = 2).
    static constexpr int kHeadIters = V == 2 ? NEST_VEC_HEAD : 1;   // quads: 2 would spill (32 registers)
    template <int OP, int S>
    __device__ __forceinline__ double accum_head(const Loop& L, int32_t id, double acc) const {
        constexpr int H = kHeadIters > 0 ? kHeadIters : 1;
        const I b = L.base;
        const I e = b + L.len;
        constexpr int kLog = V == 2 ? 1 : 2;
        int32_t c[H][V];
        double v[H][V];
#pragma unroll
        for (int h = 0; h < H; ++h) {
            const int32_t j = id + h * S;
            const I k0 = ((b >> kLog) + j) << kLog;
            if (j < L.trip && k0 + V <= (I)nnz) {   // one branch: the 128-bit tuple
                load_tuple(k0, c[h], v[h]);
            } else {                                         // predicated scalar loads (array end / idle)
#pragma unroll
                for (int q = 0; q < V; ++q) {
                    const I kq = k0 + q < (I)nnz ? k0 + q : (I)nnz - 1;
                    c[h][q] = j < L.trip ? __ldg(col + kq) : 0;
                    v[h][q] = j < L.trip ? __ldg(val + kq) : 0.0;
                }
            }
        }
        double xv[H][V];
#pragma unroll
        for (int h = 0; h < H; ++h) {
            const int32_t j = id + h * S;
            const I k0 = ((b >> kLog) + j) << kLog;
#pragma unroll
            for (int q = 0; q < V; ++q) xv[h][q] = (j < L.trip && k0 + q >= b && k0 + q < e) ? x(c[h][q]) : 0.0;
        }
#pragma unroll
        for (int h = 0; h < H; ++h) {
            const int32_t j = id + h * S;
            const I k0 = ((b >> kLog) + j) << kLog;
#pragma unroll
            for (int q = 0; q < V; ++q)
                if (j < L.trip && k0 + q >= b && k0 + q < e) acc = Red<OP, double>::accum(acc, v[h][q], xv[h][q]);
        }
        return acc;
    }
    __device__ __forceinline__ void epilogue(const Step& st, double total) const { y[st.i] = total; }
};

// ------------------------------------------------------- a9 batched matvec
// SU3_bench stand-in: outer loop over batches, a
// sequential loop over the m rows inside the parallel region, a simd loop of
// n iterations (the dot product) per row.
struct BatchedBody {
    using Acc = float;
    struct Loop {
        int64_t trip;    // n
        int64_t base;    // (b*m + r)*n
        int64_t xbase;   // b*n
    };
    struct Step {
        int64_t out;     // b*m + r
    };
    static constexpr bool kTeamState = false;
    struct TeamShared {
        int unused;
    };
    const float* A;
    const float* x;
    float* y;
    int32_t m, n;

    static __device__ __forceinline__ int steps(const BatchedBody& b) { return b.m; }
    static __device__ __forceinline__ void team_begin(TeamShared&) {}
    static __device__ __forceinline__ void team_end(const BatchedBody&, TeamShared&) {}

    __device__ __forceinline__ Loop prologue(int64_t b, int r, Step& st, bool, TeamShared&) const {
        st.out = b * m + r;
        return Loop{n, (b * m + r) * (int64_t)n, b * (int64_t)n};
    }
    template <int OP>
    __device__ __forceinline__ float accum(const Loop& L, int64_t j, float acc) const {
        return Red<OP, float>::accum(acc, __ldg(A + L.base + j), __ldg(x + L.xbase + j));
    }
    __device__ __forceinline__ void epilogue(const Step& st, float total) const { y[st.out] = total; }
};

// NEST_F_VEC128 for the batched body: the simd loop over k runs over float4
// tuples (lane l takes tuples l, l+S, ...: blocked-cyclic, R1).
// Requires n % 4 == 0 and 16-byte aligned A and x (checked on the host).
struct BatchedVecBody {
    using Acc = float;
    static constexpr int kLoopUnroll = 1;
    struct Loop {
        int64_t base;    // (b*m + r)*n / 4   (float4 index)
        int64_t xbase;   // b*n / 4
        int32_t trip;    // n / 4
        int32_t pad;
    };
    struct Step {
        int64_t out;
    };
    static constexpr bool kTeamState = false;
    struct TeamShared {
        int unused;
    };
    const float4* A;
    const float4* x;
    float* y;
    int32_t m, n;

    static __device__ __forceinline__ int steps(const BatchedVecBody& b) { return b.m; }
    static __device__ __forceinline__ void team_begin(TeamShared&) {}
    static __device__ __forceinline__ void team_end(const BatchedVecBody&, TeamShared&) {}

    __device__ __forceinline__ Loop prologue(int64_t b, int r, Step& st, bool, TeamShared&) const {
        st.out = b * m + r;
        const int32_t n4 = n >> 2;
        return Loop{(b * m + r) * (int64_t)n4, b * (int64_t)n4, n4, 0};
    }
    template <int OP>
    __device__ __forceinline__ float accum(const Loop& L, int32_t j, float acc) const {
        const float4 a = __ldg(A + L.base + j);
        const float4 v = __ldg(x + L.xbase + j);
        acc = Red<OP, float>::accum(acc, a.x, v.x);
        acc = Red<OP, float>::accum(acc, a.y, v.y);
        acc = Red<OP, float>::accum(acc, a.z, v.z);
        return Red<OP, float>::accum(acc, a.w, v.w);
    }
    // the lane's first head_for(S) float4 tuples as one predicated block (engine.cuh
    // head_iters): every load in flight before the first fold; same fold order.
    // Sized for the 64-wide rows of cfg4 (16 tuples: S = 4 -> the whole row);
    // measured on cfg4 at U = 1: S = 4 5253 -> 6215 GB/s, S = 8 4614 -> 6084 GB/s.
    static constexpr int head_for(int S) {
        return NEST_BVEC_HEAD >= 0 ? NEST_BVEC_HEAD : (S == 1 || S == 4 ? 4 : S <= 8 ? 2 : 0);
    }
    template <int OP, int S>
    __device__ __forceinline__ float accum_head(const Loop& L, int32_t id, float acc) const {
        constexpr int H = head_for(S) > 0 ? head_for(S) : 1;
        float4 a[H], v[H];
#pragma unroll
        for (int h = 0; h < H; ++h) {
            const int32_t j = id + h * S;
            if (j < L.trip) {
                a[h] = __ldg(A + L.base + j);
                v[h] = __ldg(x + L.xbase + j);
            } else {
                a[h] = v[h] = make_float4(0.f, 0.f, 0.f, 0.f);
            }
        }
#pragma unroll
        for (int h = 0; h < H; ++h) {
            if (id + h * S < L.trip) {
                acc = Red<OP, float>::accum(acc, a[h].x, v[h].x);
                acc = Red<OP, float>::accum(acc, a[h].y, v[h].y);
                acc = Red<OP, float>::accum(acc, a[h].z, v[h].z);
                acc = Red<OP, float>::accum(acc, a[h].w, v[h].w);
            }
        }
        return acc;
    }
    __device__ __forceinline__ void epilogue(const Step& st, float total) const { y[st.out] = total; }
};

// ---------------------------------------------- a10 nested stencil loop
// "Benchmark kernel" stand-in with a data-dependent
// sequential prologue and a non-idempotent side effect
// that SPMD mode must guard: visits += 1.
// The counter is aggregated per team in shared memory (one global atomic per
// team); the count is still exactly one per outer iteration.
struct StencilBody {
    using Acc = double;
    struct Loop {
        int64_t trip;   // L, or 0 when w[i] == 0
        int64_t base;   // 1 + i*L
    };
    struct Step {
        int64_t i;
        double scale;
        int64_t skip;
    };
    static constexpr bool kTeamState = true;
    struct TeamShared {
        unsigned long long visits;
    };
    const double* in;
    const double* coef;
    const double* w;
    double* out;
    unsigned long long* visits;
    int32_t L;

    static __device__ __forceinline__ int steps(const StencilBody&) { return 1; }
    static constexpr bool kOneStep = true;
    static __device__ __forceinline__ void team_begin(TeamShared& t) {
        if (threadIdx.x == 0) t.visits = 0ull;
    }
    static __device__ __forceinline__ void team_end(const StencilBody& b, TeamShared& t) {
        if (threadIdx.x == 0 && b.visits && t.visits) atomicAdd(b.visits, t.visits);
    }

    __device__ __forceinline__ Loop prologue(int64_t i, int, Step& st, bool side_effects,
                                             TeamShared& tsh) const {
        const double scale = __ldg(w + i);
        if (side_effects) atomicAdd_block(&tsh.visits, 1ull);
        st.i = i;
        st.scale = scale;
        st.skip = (scale == 0.0);
        return Loop{st.skip ? 0 : (int64_t)L, 1 + i * (int64_t)L};
    }
    template <int OP>
    __device__ __forceinline__ double accum(const Loop& Lp, int64_t j, double acc) const {
        const double* p = in + Lp.base + j;
        const double t = (__ldg(p - 1) + 2.0 * __ldg(p)) + __ldg(p + 1);
        return Red<OP, double>::accum(acc, __ldg(coef + j), t);
    }
    __device__ __forceinline__ void epilogue(const Step& st, double total) const {
        out[st.i] = st.skip ? +0.0 : st.scale * total;
    }
};

// a10 with 128-bit tuples (NEST_F_VEC128, even L, 16-byte aligned in/coef):
// simd unit = a pair of consecutive inner iterations (j = 2t, 2t+1).  The
// pair's four neighbours in[p-1 .. p+2] are two aligned double2 loads (p - 1 =
// i*L + 2t is even) and its coefficients one, against eight scalar loads for
// two elements in StencilBody; each element's t and fma are StencilBody's, in
// the same j order within the lane (the lanes' partial sums cover different j
// sets, so real-valued results match the oracle to the R3 tolerance and
// integer-valued ones bit for bit).  Measured motivation: the SPMD stencil is
// issue-bound at S >= 8 (profiles/r01s3_mode_study.md).
struct StencilVecBody : StencilBody {
    __device__ __forceinline__ Loop prologue(int64_t i, int k, Step& st, bool side_effects,
                                             TeamShared& tsh) const {
        Loop l = StencilBody::prologue(i, k, st, side_effects, tsh);
        l.trip >>= 1;   // L / 2 pairs
        return l;
    }
    template <int OP>
    __device__ __forceinline__ double accum(const Loop& Lp, int64_t t, double acc) const {
        const int64_t j = 2 * t;
        const double* p = in + Lp.base + j;
        const double2 a = __ldg(reinterpret_cast<const double2*>(p - 1));   // in[p-1], in[p]
        const double2 b = __ldg(reinterpret_cast<const double2*>(p + 1));   // in[p+1], in[p+2]
        const double2 c = __ldg(reinterpret_cast<const double2*>(coef + j));
        const double t0 = (a.x + 2.0 * a.y) + b.x;
        const double t1 = (a.y + 2.0 * b.x) + b.y;
        acc = Red<OP, double>::accum(acc, c.x, t0);
        return Red<OP, double>::accum(acc, c.y, t1);
    }
    // The lane's first H pairs (t = id, id + S, ...) as one block (engine.cuh head_iters,
    // U = 1).  Their loads are predicated on the STATIC length L/2, not on the loop's
    // trip count, so they do not wait for w[i] (the prologue's load that decides trip
    // = 0 for w == 0): the in / coef loads of an outer iteration issue together with
    // its w load -- one memory latency per outer iteration instead of two.  Loads of
    // a skipped row are issued and discarded (they are within in[0 .. N*L+2), counted
    // in the algorithmic bytes); the folds run only for t < trip, in t order: the
    // per-lane order of accum, so results are bit-identical.
    // (a head of 4 pairs at S <= 4 measured slower: L = 16/32/64 flushed 3070/4038/4578
    // vs 3686/4352/5005 GB/s with 2)
    static constexpr int kHeadIters = 2;
    template <int OP, int S>
    __device__ __forceinline__ double accum_head(const Loop& Lp, int32_t id, double acc) const {
        constexpr int H = kHeadIters;
        const int64_t half = L >> 1;   // pairs of the row, whatever w[i] is
        double2 a[H], b[H], c[H];
#pragma unroll
        for (int h = 0; h < H; ++h) {
            const int64_t t = id + h * S;
            const double* p = in + Lp.base + 2 * t;
            if (t < half) {
                a[h] = __ldg(reinterpret_cast<const double2*>(p - 1));
                b[h] = __ldg(reinterpret_cast<const double2*>(p + 1));
                c[h] = __ldg(reinterpret_cast<const double2*>(coef + 2 * t));
            }
        }
#pragma unroll
        for (int h = 0; h < H; ++h) {
            if (id + h * S < Lp.trip) {
                const double t0 = (a[h].x + 2.0 * a[h].y) + b[h].x;
                const double t1 = (a[h].y + 2.0 * b[h].x) + b[h].y;
                acc = Red<OP, double>::accum(acc, c[h].x, t0);
                acc = Red<OP, double>::accum(acc, c[h].y, t1);
            }
        }
        return acc;
    }
};

// ------------------------------------------------ NEXT-2 laplace3d
// 3-D heat-diffusion step (the Fig 10 cost study):
// teams distribute + parallel for over the (i, j) lines of the interior, simd
// over k -- a simd loop WITHOUT a reduction (kReduce = false).  The prologue
// (line base offset) is the sequential code between the parallel and the simd
// loop that decides SPMD vs generic.  Each point:
//   lap = (((((u[z-1] + u[z+1]) + u[y-1]) + u[y+1]) + u[x-1]) + u[x+1]) - 6 u
//   out = u + alpha * lap
// with round-to-nearest intrinsics (no contraction), so every mode and simdlen
// is bit-identical to the oracle.
struct LaplaceBody {
    using Acc = double;
    static constexpr bool kReduce = false;
    struct Loop {
        int64_t trip;   // nx - 2
        int64_t base;   // index of (i, j, 1)
    };
    struct Step {
        int64_t i;
    };
    static constexpr bool kTeamState = false;
    struct TeamShared {
        int unused;
    };
    const double* u;
    double* out;
    int64_t ny, nx;
    double alpha;

    static __device__ __forceinline__ int steps(const LaplaceBody&) { return 1; }
    static __device__ __forceinline__ void team_begin(TeamShared&) {}
    static __device__ __forceinline__ void team_end(const LaplaceBody&, TeamShared&) {}

    __device__ __forceinline__ Loop prologue(int64_t o, int, Step& st, bool, TeamShared&) const {
        st.i = o;
        int64_t i, j;
        if (o < ((int64_t)1 << 32) && ny - 2 < ((int64_t)1 << 32)) {   // 32-bit division when it fits
            const uint32_t q = (uint32_t)o / (uint32_t)(ny - 2);
            i = 1 + (int64_t)q;
            j = 1 + (int64_t)((uint32_t)o - q * (uint32_t)(ny - 2));
        } else {
            i = 1 + o / (ny - 2), j = 1 + o % (ny - 2);
        }
        return Loop{nx - 2, (i * ny + j) * nx + 1};
    }
    __device__ __forceinline__ void apply(const Loop& L, int64_t j) const {
        const int64_t c = L.base + j;
        const int64_t sz = ny * nx;
        double lap = __dadd_rn(__ldg(u + c - sz), __ldg(u + c + sz));
        lap = __dadd_rn(lap, __ldg(u + c - nx));
        lap = __dadd_rn(lap, __ldg(u + c + nx));
        lap = __dadd_rn(lap, __ldg(u + c - 1));
        lap = __dadd_rn(lap, __ldg(u + c + 1));
        const double uc = __ldg(u + c);
        lap = __dsub_rn(lap, __dmul_rn(6.0, uc));
        out[c] = __dadd_rn(uc, __dmul_rn(alpha, lap));
    }
    template <int OP>
    __device__ __forceinline__ double accum(const Loop&, int64_t, double acc) const { return acc; }
    __device__ __forceinline__ void epilogue(const Step&, double) const {}
};

// NEXT-2 with 128-bit pairs (NEST_F_VEC128, even nx, 16-byte aligned u/out):
// the simd unit is the aligned pair k = 2t, 2t+1 of a line (t < nx/2), so every
// neighbour pair (z-1, z+1, y-1, y+1, the centres) is one double2 load and only
// u[k-1], u[k+2] are scalar: 7 loads per two points against 14.  Each point's
// arithmetic is LaplaceBody's, operand for operand (bit-identical to the
// oracle); the line's boundary points k = 0 and nx-1 are computed from valid
// neighbouring memory (interior lines only) and not stored.
#ifndef NEST_LAPLACE_2PM
#define NEST_LAPLACE_2PM 0   // A/B switch: 2 teams of 1024 per SM (32-register cap) at U = 1
#endif
struct LaplaceVecBody : LaplaceBody {
    static constexpr bool two_teams_for(int) { return NEST_LAPLACE_2PM != 0; }
    __device__ __forceinline__ Loop prologue(int64_t o, int k, Step& st, bool se, TeamShared& t) const {
        Loop l = LaplaceBody::prologue(o, k, st, se, t);
        return Loop{nx >> 1, l.base - 1};   // pairs over the whole line, base = line start
    }
    static __device__ __forceinline__ double point(double zm, double zp, double ym, double yp, double xm,
                                                   double xp, double uc, double alpha) {
        double lap = __dadd_rn(zm, zp);
        lap = __dadd_rn(lap, ym);
        lap = __dadd_rn(lap, yp);
        lap = __dadd_rn(lap, xm);
        lap = __dadd_rn(lap, xp);
        lap = __dsub_rn(lap, __dmul_rn(6.0, uc));
        return __dadd_rn(uc, __dmul_rn(alpha, lap));
    }
    __device__ __forceinline__ void apply(const Loop& L, int64_t t) const {
        const int64_t k0 = 2 * t;
        const int64_t c = L.base + k0;
        const int64_t sz = ny * nx;
        const double2 zm = __ldg(reinterpret_cast<const double2*>(u + c - sz));
        const double2 zp = __ldg(reinterpret_cast<const double2*>(u + c + sz));
        const double2 ym = __ldg(reinterpret_cast<const double2*>(u + c - nx));
        const double2 yp = __ldg(reinterpret_cast<const double2*>(u + c + nx));
        const double2 uc = __ldg(reinterpret_cast<const double2*>(u + c));
        const double xm = __ldg(u + c - 1), xp = __ldg(u + c + 2);
        const double o0 = point(zm.x, zp.x, ym.x, yp.x, xm, uc.y, uc.x, alpha);
        const double o1 = point(zm.y, zp.y, ym.y, yp.y, uc.x, xp, uc.y, alpha);
        if (k0 >= 1 && k0 + 1 <= nx - 2) {
            *reinterpret_cast<double2*>(out + c) = make_double2(o0, o1);
        } else {
            if (k0 >= 1 && k0 <= nx - 2) out[c] = o0;
            if (k0 + 1 >= 1 && k0 + 1 <= nx - 2) out[c + 1] = o1;
        }
    }
};

// ---------------------------------------------------------------- probe
// One outer iteration per group; the simd loop body records coverage (hits),
// the executing lane (owner, group 0 only) and counts iterations through the
// reduction (totals[i] == trip under SUM).
struct ProbeBody {
    using Acc = double;
    struct Loop {
        int64_t trip;
        int64_t base;   // the outer iteration (group) index
    };
    struct Step {
        int64_t i;
    };
    static constexpr bool kTeamState = false;
    struct TeamShared {
        int unused;
    };
    int32_t* hits;
    int32_t* owner;
    double* totals;
    int64_t trip;

    static __device__ __forceinline__ int steps(const ProbeBody&) { return 1; }
    static __device__ __forceinline__ void team_begin(TeamShared&) {}
    static __device__ __forceinline__ void team_end(const ProbeBody&, TeamShared&) {}

    __device__ __forceinline__ Loop prologue(int64_t i, int, Step& st, bool, TeamShared&) const {
        st.i = i;
        return Loop{trip, i};
    }
    template <int OP>
    __device__ __forceinline__ double accum(const Loop& L, int64_t j, double acc) const {
        if (hits) atomicAdd(hits + j, 1);
        if (owner && L.base == 0) owner[j] = (int32_t)(threadIdx.x & 31u);
        return Red<OP, double>::accum(acc, 1.0, 1.0);
    }
    __device__ __forceinline__ void epilogue(const Step& st, double total) const {
        if (totals) totals[st.i] = total;
    }
};

}  // namespace nest
