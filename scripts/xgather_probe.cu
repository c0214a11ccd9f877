// xgather_probe.cu -- developer micro-benchmark (not part of the library):
// which path should the headline SpMV's x gathers take on B200?  The headline
// (blocked teams of 1024, simdlen 2, quad tuples) sits at the L1TEX data-pipe
// wall of its x gathers (~1 LSU wavefront per 8-byte gather).
// Variants of the gather, everything else identical:
//   ldg      __ldg (LDG.E.CONSTANT) -- the library's path
//   tex      tex1Dfetch<int2> on a linear texture object (TEX pipe of L1TEX)
//   mix      the tuple's entries 0,2 via LDG and 1,3 via TEX
//   noX      diagnostic: no gather (col as the value) -- the floor
// Matrix: cfg2/G100-shaped (U{4..12} nnz/row, band +-4096, 1/16 far), same
// generator as l2x_probe.cu.  Median of 10 launches, L2 flushed before each.
// nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -lineinfo -o scripts/xgather_probe scripts/xgather_probe.cu
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <vector>

#define CK(x)                                                                                  \
    do {                                                                                       \
        cudaError_t e_ = (x);                                                                  \
        if (e_ != cudaSuccess) {                                                               \
            fprintf(stderr, "%s:%d %s: %s\n", __FILE__, __LINE__, #x, cudaGetErrorString(e_)); \
            exit(1);                                                                           \
        }                                                                                      \
    } while (0)

__host__ __device__ inline uint64_t mix(uint64_t z) {
    z += 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

__global__ void gen_cols(const int64_t* rp, int n, int* col, double* val, int W, int far_den, uint64_t seed) {
    int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= n) return;
    int64_t b = rp[i];
    int len = (int)(rp[i + 1] - b);
    int c[32];
    for (int k = 0; k < len; ++k) {
        uint64_t h = mix(seed ^ ((uint64_t)i * 0x9E3779B97F4A7C15ull) ^ ((uint64_t)(k + 1) * 0xBF58476D1CE4E5B9ull));
        uint64_t h2 = mix(h);
        int cc;
        if ((int)(h % far_den) == 0) {
            cc = (int)((h2 & 0xffffffffull) * (uint64_t)n >> 32);
        } else {
            int lo = max(0, i - W), hi = min(n - 1, i + W);
            cc = lo + (int)((h2 & 0xffffffffull) * (uint64_t)(hi - lo + 1) >> 32);
        }
        c[k] = cc;
        val[b + k] = (double)(int64_t)(h2 >> 40) * 0x1p-23 - 1.0;
    }
    for (int a = 1; a < len; ++a)
        for (int q = a; q > 0 && c[q - 1] > c[q]; --q) {
            int t = c[q];
            c[q] = c[q - 1];
            c[q - 1] = t;
        }
    for (int k = 0; k < len; ++k) col[b + k] = c[k];
}

__device__ cudaTextureObject_t g_xtex;

// XM: 0 ldg, 1 tex, 2 mix (odd entries tex), 3 no gather, 4 ld.global (no .nc), 5 ld.global.nc.L1::evict_last
template <int XM>
__device__ __forceinline__ double ldx(const double* x, int c, int q) {
    if constexpr (XM == 0) {
        return __ldg(x + c);
    } else if constexpr (XM == 1) {
        const int2 t = tex1Dfetch<int2>(g_xtex, c);
        return __hiloint2double(t.y, t.x);
    } else if constexpr (XM == 2) {
        if (q & 1) {
            const int2 t = tex1Dfetch<int2>(g_xtex, c);
            return __hiloint2double(t.y, t.x);
        }
        return __ldg(x + c);
    } else if constexpr (XM == 3) {
        return (double)c;
    } else if constexpr (XM == 4) {
        double r;
        asm volatile("ld.global.f64 %0, [%1];" : "=d"(r) : "l"(x + c));
        return r;
    } else if constexpr (XM == 5) {
        double r;
        asm volatile("ld.global.nc.L1::evict_last.f64 %0, [%1];" : "=d"(r) : "l"(x + c));
        return r;
    } else if constexpr (XM == 8) {   // diagnostic: every gather an L1 hit (32 KB of x), distinct lines as before
        return __ldg(x + (c & 4095));
    } else if constexpr (XM == 9) {   // diagnostic: every gather an L1 hit, one line per 32 lanes (no line spread)
        return __ldg(x + (c & 15));
    } else if constexpr (XM == 6) {
        double r;
        asm volatile("ld.global.nc.L1::evict_first.f64 %0, [%1];" : "=d"(r) : "l"(x + c));
        return r;
    } else {
        uint64_t pl;
        asm("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pl));
        double r;
        asm volatile("ld.global.nc.L2::cache_hint.f64 %0, [%1], %2;" : "=d"(r) : "l"(x + c), "l"(pl));
        return r;
    }
}

// the headline's structure: blocked teams, group of S lanes per row, quad tuples
// (int4 colind + one 256-bit val load), lane l takes tuples l, l+S, ...
// PC (CSR tuple loads): 0 __ldg, 1 L2::evict_first, 2 L1::evict_last + L2::evict_first,
// 3 L1::no_allocate + L2::evict_first, 4 L2::evict_first on half the lines (fractional 0.5)
template <int PC>
__device__ __forceinline__ void ld_quad(const int* col, const double* val, uint64_t pol, int (&c)[4], double (&v)[4]) {
    if constexpr (PC == 0) {
        const int4 cc = __ldg(reinterpret_cast<const int4*>(col));
        c[0] = cc.x, c[1] = cc.y, c[2] = cc.z, c[3] = cc.w;
        asm("ld.global.nc.v4.f64 {%0, %1, %2, %3}, [%4];" : "=d"(v[0]), "=d"(v[1]), "=d"(v[2]), "=d"(v[3]) : "l"(val));
    } else if constexpr (PC == 9) {   // L1::evict_first only (CSR lines leave L1 before the x band)
        asm("ld.global.nc.L1::evict_first.v4.s32 {%0, %1, %2, %3}, [%4];"
            : "=r"(c[0]), "=r"(c[1]), "=r"(c[2]), "=r"(c[3]) : "l"(col));
        asm("ld.global.nc.L1::evict_first.v4.f64 {%0, %1, %2, %3}, [%4];"
            : "=d"(v[0]), "=d"(v[1]), "=d"(v[2]), "=d"(v[3]) : "l"(val));
    } else if constexpr (PC == 7) {   // L1::no_allocate only (L1 kept for the x band)
        asm("ld.global.nc.L1::no_allocate.v4.s32 {%0, %1, %2, %3}, [%4];"
            : "=r"(c[0]), "=r"(c[1]), "=r"(c[2]), "=r"(c[3]) : "l"(col));
        asm("ld.global.nc.L1::no_allocate.v4.f64 {%0, %1, %2, %3}, [%4];"
            : "=d"(v[0]), "=d"(v[1]), "=d"(v[2]), "=d"(v[3]) : "l"(val));
    } else if constexpr (PC == 8) {   // val L1::no_allocate only
        const int4 cc = __ldg(reinterpret_cast<const int4*>(col));
        c[0] = cc.x, c[1] = cc.y, c[2] = cc.z, c[3] = cc.w;
        asm("ld.global.nc.L1::no_allocate.v4.f64 {%0, %1, %2, %3}, [%4];"
            : "=d"(v[0]), "=d"(v[1]), "=d"(v[2]), "=d"(v[3]) : "l"(val));
    } else if constexpr (PC == 5) {   // colind evict-first only
        asm("ld.global.nc.L2::cache_hint.v4.s32 {%0, %1, %2, %3}, [%4], %5;"
            : "=r"(c[0]), "=r"(c[1]), "=r"(c[2]), "=r"(c[3]) : "l"(col), "l"(pol));
        asm("ld.global.nc.v4.f64 {%0, %1, %2, %3}, [%4];" : "=d"(v[0]), "=d"(v[1]), "=d"(v[2]), "=d"(v[3]) : "l"(val));
    } else if constexpr (PC == 6) {   // val evict-first only
        const int4 cc = __ldg(reinterpret_cast<const int4*>(col));
        c[0] = cc.x, c[1] = cc.y, c[2] = cc.z, c[3] = cc.w;
        asm("ld.global.nc.L2::cache_hint.v4.f64 {%0, %1, %2, %3}, [%4], %5;"
            : "=d"(v[0]), "=d"(v[1]), "=d"(v[2]), "=d"(v[3]) : "l"(val), "l"(pol));
    } else if constexpr (PC == 1 || PC == 4) {
        asm("ld.global.nc.L2::cache_hint.v4.s32 {%0, %1, %2, %3}, [%4], %5;"
            : "=r"(c[0]), "=r"(c[1]), "=r"(c[2]), "=r"(c[3]) : "l"(col), "l"(pol));
        asm("ld.global.nc.L2::cache_hint.v4.f64 {%0, %1, %2, %3}, [%4], %5;"
            : "=d"(v[0]), "=d"(v[1]), "=d"(v[2]), "=d"(v[3]) : "l"(val), "l"(pol));
    } else if constexpr (PC == 2) {
        asm("ld.global.nc.L1::evict_last.L2::cache_hint.v4.s32 {%0, %1, %2, %3}, [%4], %5;"
            : "=r"(c[0]), "=r"(c[1]), "=r"(c[2]), "=r"(c[3]) : "l"(col), "l"(pol));
        asm("ld.global.nc.L1::evict_last.L2::cache_hint.v4.f64 {%0, %1, %2, %3}, [%4], %5;"
            : "=d"(v[0]), "=d"(v[1]), "=d"(v[2]), "=d"(v[3]) : "l"(val), "l"(pol));
    } else {
        asm("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.s32 {%0, %1, %2, %3}, [%4], %5;"
            : "=r"(c[0]), "=r"(c[1]), "=r"(c[2]), "=r"(c[3]) : "l"(col), "l"(pol));
        asm("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.f64 {%0, %1, %2, %3}, [%4], %5;"
            : "=d"(v[0]), "=d"(v[1]), "=d"(v[2]), "=d"(v[3]) : "l"(val), "l"(pol));
    }
}

template <int S, int XM, int PC = 0, int PF = 0>
__global__ void __launch_bounds__(1024, 2)
    spmv_q(const int64_t* __restrict__ rp, const int* __restrict__ col, const double* __restrict__ val,
           const double* __restrict__ x, double* __restrict__ y, int n, int chunk, int nnz) {
    if constexpr (PF) {
        // PF 1: the team's 1/grid share of x (far columns); PF 2: the team's own band
        // [row0 - 4096, row1 + 4096); bulk L2 prefetches of <= 32 KB by warp 0
        const int64_t xbytes = (int64_t)n * 8;
        int64_t b0, e0;
        if constexpr (PF == 1) {
            const int64_t per = ((xbytes + gridDim.x - 1) / gridDim.x + 15) & ~(int64_t)15;
            b0 = per * blockIdx.x, e0 = min(xbytes, b0 + per);
        } else {
            b0 = (int64_t)max(0, (int)blockIdx.x * chunk - 4096) * 8 & ~(int64_t)15;
            e0 = min(xbytes, (int64_t)min(n, ((int)blockIdx.x + 1) * chunk + 4096) * 8);
        }
        if (threadIdx.x < 32)
            for (int64_t o = b0 + (int64_t)threadIdx.x * 32768; o < e0; o += 32 * 32768) {
                const uint32_t sz = (uint32_t)min((int64_t)32768, e0 - o) & ~15u;
                if (sz)
                    asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(reinterpret_cast<const char*>(x) + o),
                                 "r"(sz) : "memory");
            }
    }
    const int G = blockDim.x / S;
    const int g = threadIdx.x / S, lane = threadIdx.x % S;
    const int cs = blockIdx.x * chunk;
    const int ce = min(n, cs + chunk);
    uint64_t pol = 0;
    if constexpr (PC == 4) {
        asm("createpolicy.fractional.L2::evict_first.L2::evict_unchanged.b64 %0, 0.5;" : "=l"(pol));
    } else if constexpr (PC != 0) {
        asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
    }
    for (int i = cs + g; i < ce; i += G) {
        const int b = (int)__ldg(rp + i), e = (int)__ldg(rp + i + 1);
        const int trip = e > b ? ((e + 3) >> 2) - (b >> 2) : 0;
        double acc = 0.0;
        for (int t = lane; t < trip; t += S) {
            const int k0 = ((b >> 2) + t) << 2;
            int c[4];
            double v[4];
            if (k0 + 4 <= nnz) {
                ld_quad<PC>(col + k0, val + k0, pol, c, v);
            } else {
#pragma unroll
                for (int q = 0; q < 4; ++q) {
                    const int kq = k0 + q < nnz ? k0 + q : k0;
                    c[q] = __ldg(col + kq);
                    v[q] = __ldg(val + kq);
                }
            }
#pragma unroll
            for (int q = 0; q < 4; ++q)
                if (k0 + q >= b && k0 + q < e) acc = fma(v[q], ldx<XM>(x, c[q], q), acc);
        }
#pragma unroll
        for (int off = S / 2; off >= 1; off >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, off);
        if (lane == 0) y[i] = acc;
    }
}

// Diagnostic for the DRAM side: the same nonzeros and gathers as the SpMV, but the
// CSR stream read in full lines (warp-coalesced, lane = nonzero) with a chosen L2
// policy, the x gathers with another; one sum per thread (no rows).  Does L2 keep
// x (80-100 MB) while 1-1.3 GB of CSR streams through it?  ncu dram__bytes tells.
// PC: 0 normal, 1 L2::evict_first, 2 L1::no_allocate + L2::evict_first
// PX: 0 normal, 1 L2::evict_last
template <int PC, int PX>
__global__ void __launch_bounds__(1024, 2)
    stream_gather(const int* __restrict__ col, const double* __restrict__ val, const double* __restrict__ x,
                  int nnz, double* sink) {
    uint64_t pf, pl;
    asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pf));
    asm("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pl));
    double acc = 0.0;
    const int stride = gridDim.x * blockDim.x;
    // blocked: each CTA sweeps a contiguous range (like the blocked teams)
    const int per = (nnz + gridDim.x - 1) / gridDim.x;
    const int b0 = blockIdx.x * per, e0 = min(nnz, b0 + per);
    (void)stride;
    for (int k = b0 + threadIdx.x; k < e0; k += blockDim.x) {
        int c;
        double v, xv;
        if constexpr (PC == 0) {
            c = __ldg(col + k), v = __ldg(val + k);
        } else if constexpr (PC == 1) {
            asm volatile("ld.global.nc.L2::cache_hint.s32 %0, [%1], %2;" : "=r"(c) : "l"(col + k), "l"(pf));
            asm volatile("ld.global.nc.L2::cache_hint.f64 %0, [%1], %2;" : "=d"(v) : "l"(val + k), "l"(pf));
        } else {
            asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.s32 %0, [%1], %2;" : "=r"(c) : "l"(col + k), "l"(pf));
            asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.f64 %0, [%1], %2;" : "=d"(v) : "l"(val + k), "l"(pf));
        }
        if constexpr (PX == 0) {
            xv = __ldg(x + c);
        } else {
            asm volatile("ld.global.nc.L2::cache_hint.f64 %0, [%1], %2;" : "=d"(xv) : "l"(x + c), "l"(pl));
        }
        acc = fma(v, xv, acc);
    }
    if (acc == 1234.5) sink[0] = acc;
}

// ----------------------------------------------------------------------------
// Warp-staged CSR (experiment): warp = 32/S groups = a batch of RB = 32/S
// consecutive rows of the team's range.  The warp loads the batch's rowptr slice
// (one coalesced load) and its whole colind/val range in 4-nonzero units with
// full-line loads (POL 1: L1::no_allocate + L2::evict_first, so x stays in L2),
// stores them to its shared stage, and each group runs its row's simd loop from
// the stage: lane id takes nonzeros id, id+S, ... (Fig 8 order, scalar).  A batch
// whose range exceeds the stage falls back to direct loads.
template <int POL>
__device__ __forceinline__ void ld_unit(const int* col, const double* val, uint64_t pol, int4& c, double (&v)[4]) {
    if constexpr (POL == 0) {
        c = __ldg(reinterpret_cast<const int4*>(col));
        asm volatile("ld.global.nc.v4.f64 {%0, %1, %2, %3}, [%4];" : "=d"(v[0]), "=d"(v[1]), "=d"(v[2]), "=d"(v[3]) : "l"(val));
    } else {
        asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.s32 {%0, %1, %2, %3}, [%4], %5;"
                     : "=r"(c.x), "=r"(c.y), "=r"(c.z), "=r"(c.w) : "l"(col), "l"(pol));
        asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.f64 {%0, %1, %2, %3}, [%4], %5;"
                     : "=d"(v[0]), "=d"(v[1]), "=d"(v[2]), "=d"(v[3]) : "l"(val), "l"(pol));
    }
}

template <int S, int CAPU, int H, int TPB, int MINB, int POL, bool RPF>
__global__ void __launch_bounds__(TPB, MINB)
    spmv_ws(const int64_t* __restrict__ rp, const int* __restrict__ col, const double* __restrict__ val,
            const double* __restrict__ x, double* __restrict__ y, int n, int chunk, int nnz) {
    constexpr int RB = 32 / S;
    extern __shared__ __align__(16) unsigned char sm_raw[];
    const int W = TPB / 32, w = threadIdx.x >> 5, lane = threadIdx.x & 31;
    int* scol = reinterpret_cast<int*>(sm_raw) + w * CAPU * 4;
    double* sval = reinterpret_cast<double*>(sm_raw + (size_t)W * CAPU * 16) + w * CAPU * 4;
    uint64_t pol = 0;
    if constexpr (POL == 1) asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
    const int g = lane / S, id = lane % S;
    const int cs = blockIdx.x * chunk;
    const int ce = min(n, cs + chunk);
    const int nb = (ce - cs + RB - 1) / RB;
    int m = w;
    long long rpn = 0;
    if (RPF && m < nb) {
        const int r = cs + m * RB + lane;
        if (lane <= RB) rpn = __ldg(rp + min(r, ce));
    }
    for (; m < nb; m += W) {
        const int r0 = cs + m * RB;
        const int nr = min(RB, ce - r0);
        long long rpl;
        if constexpr (RPF) {
            rpl = rpn;
            const int r = cs + (m + W) * RB + lane;
            if (m + W < nb && lane <= RB) rpn = __ldg(rp + min(r, ce));
        } else {
            rpl = lane <= RB ? __ldg(rp + min(r0 + lane, ce)) : 0;
        }
        const int kb = (int)__shfl_sync(0xffffffffu, rpl, 0);
        const int ke = (int)__shfl_sync(0xffffffffu, rpl, nr);
        const int b = (int)__shfl_sync(0xffffffffu, rpl, min(g, nr));
        const int e = (int)__shfl_sync(0xffffffffu, rpl, min(g + 1, nr));
        const int u0 = kb >> 2;
        const int nu = ((ke + 3) >> 2) - u0;
        double acc = 0.0;
        if (nu <= CAPU) {
            for (int u = lane; u < nu; u += 32) {
                const int k0 = (u0 + u) << 2;
                int4 c;
                double v[4];
                if (k0 + 4 <= nnz) {
                    ld_unit<POL>(col + k0, val + k0, pol, c, v);
                } else {
                    c.x = __ldg(col + k0);
                    c.y = k0 + 1 < nnz ? __ldg(col + k0 + 1) : 0;
                    c.z = k0 + 2 < nnz ? __ldg(col + k0 + 2) : 0;
                    c.w = k0 + 3 < nnz ? __ldg(col + k0 + 3) : 0;
#pragma unroll
                    for (int q = 0; q < 4; ++q) v[q] = k0 + q < nnz ? __ldg(val + k0 + q) : 0.0;
                }
                reinterpret_cast<int4*>(scol)[u] = c;
                reinterpret_cast<double2*>(sval)[2 * u] = make_double2(v[0], v[1]);
                reinterpret_cast<double2*>(sval)[2 * u + 1] = make_double2(v[2], v[3]);
            }
            __syncwarp();
            const int o = b - (u0 << 2);
            const int len = e - b;
            // head block of H iterations: smem loads, then gathers, then folds (Fig 8 order)
            int cc[H];
            double vv[H], xv[H];
#pragma unroll
            for (int h = 0; h < H; ++h) {
                const int j = id + h * S;
                cc[h] = j < len ? scol[o + j] : 0;
                vv[h] = j < len ? sval[o + j] : 0.0;
            }
#pragma unroll
            for (int h = 0; h < H; ++h) xv[h] = id + h * S < len ? __ldg(x + cc[h]) : 0.0;
#pragma unroll
            for (int h = 0; h < H; ++h)
                if (id + h * S < len) acc = fma(vv[h], xv[h], acc);
            for (int j = id + H * S; j < len; j += S) acc = fma(sval[o + j], __ldg(x + scol[o + j]), acc);
            __syncwarp();
        } else {
            for (int j = id; j < e - b; j += S) acc = fma(__ldg(val + b + j), __ldg(x + __ldg(col + b + j)), acc);
        }
#pragma unroll
        for (int off = S / 2; off >= 1; off >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, off);
        if (id == 0 && g < nr) y[r0 + g] = acc;
    }
}

// reference for the staged kernels' order: scalar Fig 8 (lane id: id, id+S, ...)
template <int S>
__global__ void __launch_bounds__(1024, 2)
    spmv_s(const int64_t* __restrict__ rp, const int* __restrict__ col, const double* __restrict__ val,
           const double* __restrict__ x, double* __restrict__ y, int n, int chunk, int nnz) {
    const int G = blockDim.x / S;
    const int g = threadIdx.x / S, id = threadIdx.x % S;
    const int cs = blockIdx.x * chunk;
    const int ce = min(n, cs + chunk);
    for (int i = cs + g; i < ce; i += G) {
        const int b = (int)__ldg(rp + i), e = (int)__ldg(rp + i + 1);
        double acc = 0.0;
        for (int j = id; j < e - b; j += S) acc = fma(__ldg(val + b + j), __ldg(x + __ldg(col + b + j)), acc);
#pragma unroll
        for (int off = S / 2; off >= 1; off >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, off);
        if (id == 0) y[i] = acc;
    }
}

// Co-located teams (diagnostic): the two teams resident on an SM sweep ONE region of
// rows together (rounds of 2G consecutive rows, team slot s taking the s-th half), so
// the SM's L1 holds one band of x instead of two.  Region = %smid; slot = parity of a
// per-SM launch counter (exactly two teams per SM per launch: grid = 2 x SMs at an
// occupancy of 2 -- checked by comparing y with the headline, bit for bit).
__device__ int g_sm_ctr[256];
template <int S>
__global__ void __launch_bounds__(1024, 2)
    spmv_colo(const int64_t* __restrict__ rp, const int* __restrict__ col, const double* __restrict__ val,
              const double* __restrict__ x, double* __restrict__ y, int n, int chunk_unused, int nnz) {
    __shared__ int s_slot, s_sm;
    if (threadIdx.x == 0) {
        int sm;
        asm volatile("mov.u32 %0, %%smid;" : "=r"(sm));
        s_sm = sm;
        s_slot = atomicAdd(&g_sm_ctr[sm], 1) & 1;
    }
    __syncthreads();
    const int nsm = gridDim.x / 2;
    const int G = blockDim.x / S;
    const int g = threadIdx.x / S, lane = threadIdx.x % S;
    int per = (n + nsm - 1) / nsm;
    per = (per + 2 * G - 1) / (2 * G) * (2 * G);
    const int cs = s_sm * per;
    const int ce = min(n, cs + per);
    for (int i = cs + s_slot * G + g; i < ce; i += 2 * G) {
        const int b = (int)__ldg(rp + i), e = (int)__ldg(rp + i + 1);
        const int trip = e > b ? ((e + 3) >> 2) - (b >> 2) : 0;
        double acc = 0.0;
        for (int t = lane; t < trip; t += S) {
            const int k0 = ((b >> 2) + t) << 2;
            int c[4];
            double v[4];
            if (k0 + 4 <= nnz) {
                ld_quad<0>(col + k0, val + k0, 0, c, v);
            } else {
#pragma unroll
                for (int q = 0; q < 4; ++q) {
                    const int kq = k0 + q < nnz ? k0 + q : k0;
                    c[q] = __ldg(col + kq);
                    v[q] = __ldg(val + kq);
                }
            }
#pragma unroll
            for (int q = 0; q < 4; ++q)
                if (k0 + q >= b && k0 + q < e) acc = fma(v[q], __ldg(x + c[q]), acc);
        }
#pragma unroll
        for (int off = S / 2; off >= 1; off >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, off);
        if (lane == 0) y[i] = acc;
    }
}

// ----------------------------------------------------------------------------
// Static x window per team (experiment): non-persistent grid, team = C consecutive
// rows; thread 0 bulk-copies x[lo, hi) = [r0 - H, r0 + C + H) (clipped, 16-byte
// aligned) into shared memory at team start on one mbarrier; every warp loads its
// first row's bounds and tuples BEFORE waiting on it (the copy hides behind the CSR
// latency).  Gathers inside the window read shared memory, the rest global memory.
__device__ __forceinline__ uint32_t sptr(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

template <int S, int C, int H>
__global__ void __launch_bounds__(1024, 2)
    spmv_win(const int64_t* __restrict__ rp, const int* __restrict__ col, const double* __restrict__ val,
             const double* __restrict__ x, double* __restrict__ y, int n, int chunk_unused, int nnz) {
    extern __shared__ __align__(16) double win[];
    __shared__ __align__(8) uint64_t bar;
    const int r0 = blockIdx.x * C;
    const int r1 = min(n, r0 + C);
    const int lo = max(0, r0 - H) & ~1;
    const int hi = min(n, ((r1 + H) + 1) & ~1);   // n even in these matrices
    const uint32_t bytes = (uint32_t)(hi - lo) * 8u;
    if (threadIdx.x == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(sptr(&bar)));
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(sptr(&bar)), "r"(bytes) : "memory");
        for (uint32_t o = 0; o < bytes; o += 16384) {
            const uint32_t sz = min(16384u, bytes - o);
            asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                         ::"r"(sptr(win) + o), "l"(reinterpret_cast<const char*>(x + lo) + o), "r"(sz), "r"(sptr(&bar))
                         : "memory");
        }
    }
    const int G = blockDim.x / S;
    const int g = threadIdx.x / S, lane = threadIdx.x % S;
    const unsigned wlen = (unsigned)(hi - lo);
    bool waited = false;
    for (int i = r0 + g; i < r1; i += G) {
        const int b = (int)__ldg(rp + i), e = (int)__ldg(rp + i + 1);
        const int trip = e > b ? ((e + 3) >> 2) - (b >> 2) : 0;
        double acc = 0.0;
        for (int t = lane; t < trip; t += S) {
            const int k0 = ((b >> 2) + t) << 2;
            int c[4];
            double v[4];
            if (k0 + 4 <= nnz) {
                ld_quad<0>(col + k0, val + k0, 0, c, v);
            } else {
#pragma unroll
                for (int q = 0; q < 4; ++q) {
                    const int kq = k0 + q < nnz ? k0 + q : k0;
                    c[q] = __ldg(col + kq);
                    v[q] = __ldg(val + kq);
                }
            }
            if (!waited) {
                asm volatile("{\n .reg .pred p;\n W: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], 0;\n @!p bra W;\n}"
                             ::"r"(sptr(&bar)) : "memory");
                waited = true;
            }
            double xv[4];
#pragma unroll
            for (int q = 0; q < 4; ++q) {   // branch-free: one predicated shared and one predicated global load
                const unsigned off = (unsigned)(c[q] - lo);
                const uint32_t sa = sptr(win) + (off < wlen ? off : 0u) * 8u;
                asm volatile("{\n .reg .pred p;\n setp.lt.u32 p, %1, %2;\n @p ld.shared.f64 %0, [%3];\n"
                             " @!p ld.global.nc.f64 %0, [%4];\n}"
                             : "=d"(xv[q]) : "r"(off), "r"(wlen), "r"(sa), "l"(x + c[q]));
            }
#pragma unroll
            for (int q = 0; q < 4; ++q)
                if (k0 + q >= b && k0 + q < e) acc = fma(v[q], xv[q], acc);
        }
#pragma unroll
        for (int off = S / 2; off >= 1; off >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, off);
        if (lane == 0) y[i] = acc;
    }
    if (!waited)   // never leave a bulk copy in flight into a released shared-memory block
        asm volatile("{\n .reg .pred p;\n W2: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], 0;\n @!p bra W2;\n}"
                     ::"r"(sptr(&bar)) : "memory");
}

// Head block of H quads per lane (all tuple loads, then all gathers, then the folds in
// order), then the plain loop; launch bounds (TB, MINB) set the register budget.
template <int S, int H, int TB, int MINB>
__global__ void __launch_bounds__(TB, MINB)
    spmv_qh(const int64_t* __restrict__ rp, const int* __restrict__ col, const double* __restrict__ val,
            const double* __restrict__ x, double* __restrict__ y, int n, int chunk, int nnz) {
    const int G = blockDim.x / S;
    const int g = threadIdx.x / S, lane = threadIdx.x % S;
    const int cs = blockIdx.x * chunk;
    const int ce = min(n, cs + chunk);
    for (int i = cs + g; i < ce; i += G) {
        const int b = (int)__ldg(rp + i), e = (int)__ldg(rp + i + 1);
        const int trip = e > b ? ((e + 3) >> 2) - (b >> 2) : 0;
        double acc = 0.0;
        int c[H][4];
        double v[H][4];
#pragma unroll
        for (int h = 0; h < H; ++h) {
            const int t = lane + h * S;
            const int k0 = ((b >> 2) + t) << 2;
            if (t < trip && k0 + 4 <= nnz) {
                ld_quad<0>(col + k0, val + k0, 0, c[h], v[h]);
            } else {
#pragma unroll
                for (int q = 0; q < 4; ++q) {
                    const int kq = min(k0 + q, nnz - 1);
                    c[h][q] = t < trip ? __ldg(col + kq) : 0;
                    v[h][q] = t < trip ? __ldg(val + kq) : 0.0;
                }
            }
        }
        double xv[H][4];
#pragma unroll
        for (int h = 0; h < H; ++h) {
            const int t = lane + h * S;
            const int k0 = ((b >> 2) + t) << 2;
#pragma unroll
            for (int q = 0; q < 4; ++q) xv[h][q] = (t < trip && k0 + q >= b && k0 + q < e) ? __ldg(x + c[h][q]) : 0.0;
        }
#pragma unroll
        for (int h = 0; h < H; ++h) {
            const int t = lane + h * S;
            const int k0 = ((b >> 2) + t) << 2;
#pragma unroll
            for (int q = 0; q < 4; ++q)
                if (t < trip && k0 + q >= b && k0 + q < e) acc = fma(v[h][q], xv[h][q], acc);
        }
        for (int t = lane + H * S; t < trip; t += S) {
            const int k0 = ((b >> 2) + t) << 2;
            int cc[4];
            double vv[4];
            if (k0 + 4 <= nnz) {
                ld_quad<0>(col + k0, val + k0, 0, cc, vv);
            } else {
#pragma unroll
                for (int q = 0; q < 4; ++q) {
                    const int kq = min(k0 + q, nnz - 1);
                    cc[q] = __ldg(col + kq);
                    vv[q] = __ldg(val + kq);
                }
            }
#pragma unroll
            for (int q = 0; q < 4; ++q)
                if (k0 + q >= b && k0 + q < e) acc = fma(vv[q], __ldg(x + cc[q]), acc);
        }
#pragma unroll
        for (int off = S / 2; off >= 1; off >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, off);
        if (lane == 0) y[i] = acc;
    }
}

// Per-team start / end times (%globaltimer, ns) of the headline structure: how much of the
// kernel is the tail after the median team has finished?
__device__ unsigned long long g_t0[1024], g_t1[1024];
template <int S, bool REV = false>
__global__ void __launch_bounds__(1024, 2)
    spmv_qt(const int64_t* __restrict__ rp, const int* __restrict__ col, const double* __restrict__ val,
            const double* __restrict__ x, double* __restrict__ y, int n, int chunk, int nnz) {
    unsigned long long t;
    if (threadIdx.x == 0) {
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
        g_t0[blockIdx.x] = t;
    }
    const int G = blockDim.x / S;
    const int g = threadIdx.x / S, lane = threadIdx.x % S;
    const int cs = (REV ? gridDim.x - 1 - blockIdx.x : blockIdx.x) * chunk;
    const int ce = min(n, cs + chunk);
    for (int i = cs + g; i < ce; i += G) {
        const int b = (int)__ldg(rp + i), e = (int)__ldg(rp + i + 1);
        const int trip = e > b ? ((e + 3) >> 2) - (b >> 2) : 0;
        double acc = 0.0;
        for (int tt = lane; tt < trip; tt += S) {
            const int k0 = ((b >> 2) + tt) << 2;
            int c[4];
            double v[4];
            if (k0 + 4 <= nnz) {
                ld_quad<0>(col + k0, val + k0, 0, c, v);
            } else {
#pragma unroll
                for (int q = 0; q < 4; ++q) {
                    const int kq = k0 + q < nnz ? k0 + q : k0;
                    c[q] = __ldg(col + kq);
                    v[q] = __ldg(val + kq);
                }
            }
#pragma unroll
            for (int q = 0; q < 4; ++q)
                if (k0 + q >= b && k0 + q < e) acc = fma(v[q], __ldg(x + c[q]), acc);
        }
#pragma unroll
        for (int off = S / 2; off >= 1; off >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, off);
        if (lane == 0) y[i] = acc;
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
        g_t1[blockIdx.x] = t;
    }
}

// Tail pool (experiment): team b's first (1 - F/100) of its chunk is processed as in the
// headline (static); the last F% of every chunk forms one global pool of 16-row warp
// blocks (round-robin over the teams), claimed by any warp that has finished its own part
// (one atomicAdd per block on g_pool, zeroed before every launch).  Results identical (a
// row is computed the same way by whichever warp takes it).
__device__ int g_pool;
template <int S, int F>
__global__ void __launch_bounds__(1024, 2)
    spmv_qpool(const int64_t* __restrict__ rp, const int* __restrict__ col, const double* __restrict__ val,
               const double* __restrict__ x, double* __restrict__ y, int n, int chunk, int nnz) {
    constexpr int RB = 32 / S;   // rows per warp block
    const int W = blockDim.x / 32, w = threadIdx.x / 32;
    const int gl = (threadIdx.x & 31) / S, lane = threadIdx.x % S;
    const int nblk_team = chunk / RB;                       // chunk is a multiple of G (so of RB)
    const int tail = (nblk_team * F / 100 + W - 1) / W * W; // pool blocks per team
    const int priv = nblk_team - tail;
    auto row_block = [&](int team, int j) {
        const int r0 = team * chunk + j * RB;
        const int i = r0 + gl;
        if (i >= n) return;
        const int b = (int)__ldg(rp + i), e = (int)__ldg(rp + i + 1);
        const int trip = e > b ? ((e + 3) >> 2) - (b >> 2) : 0;
        double acc = 0.0;
        for (int t = lane; t < trip; t += S) {
            const int k0 = ((b >> 2) + t) << 2;
            int c[4];
            double v[4];
            if (k0 + 4 <= nnz) {
                ld_quad<0>(col + k0, val + k0, 0, c, v);
            } else {
#pragma unroll
                for (int q = 0; q < 4; ++q) {
                    const int kq = k0 + q < nnz ? k0 + q : k0;
                    c[q] = __ldg(col + kq);
                    v[q] = __ldg(val + kq);
                }
            }
#pragma unroll
            for (int q = 0; q < 4; ++q)
                if (k0 + q >= b && k0 + q < e) acc = fma(v[q], __ldg(x + c[q]), acc);
        }
#pragma unroll
        for (int off = S / 2; off >= 1; off >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, off);
        if (lane == 0) y[i] = acc;
    };
    for (int j = w; j < priv; j += W) row_block(blockIdx.x, j);
    const int total = tail * gridDim.x;
    while (true) {
        int q = 0;
        if ((threadIdx.x & 31) == 0) q = atomicAdd(&g_pool, 1);
        q = __shfl_sync(0xffffffffu, q, 0);
        if (q >= total) break;
        row_block(q % gridDim.x, priv + q / gridDim.x);
    }
}

__global__ void zero_pool() { g_pool = 0; }

// Diagnostic (wrong values): the consumer side of a fully staged design -- row bounds
// from global rowptr (real), each nonzero's colind / val read from a static shared "stage"
// (k & 4095), x from a static shared window (c & 8191), and one nonzero in 16 gathering
// x from global memory at a scattered column (the far columns).  No CSR traffic from
// DRAM: what the consumers alone would cost if a producer kept the stages full.
template <int S, int FAR, int TB, int MINB, bool BAR = false>
__global__ void __launch_bounds__(TB, MINB)
    spmv_stagediag(const int64_t* __restrict__ rp, const int* __restrict__ col, const double* __restrict__ val,
                   const double* __restrict__ x, double* __restrict__ y, int n, int chunk, int nnz) {
    extern __shared__ __align__(16) unsigned char sm_raw[];
    int* scol = reinterpret_cast<int*>(sm_raw);                       // 4096 ints (16 KB)
    double* sval = reinterpret_cast<double*>(sm_raw + 16384);        // 4096 doubles (32 KB)
    double* xwin = reinterpret_cast<double*>(sm_raw + 16384 + 32768); // 8192 doubles (64 KB)
    for (int k = threadIdx.x; k < 4096; k += blockDim.x) {
        scol[k] = (int)((k * 2654435761u) & 0x7fffffff);
        sval[k] = (double)(k & 7) - 3.0;
    }
    for (int k = threadIdx.x; k < 8192; k += blockDim.x) xwin[k] = (double)(k & 15);
    __syncthreads();
    const int G = blockDim.x / S;
    const int g = threadIdx.x / S, lane = threadIdx.x % S;
    const int cs = blockIdx.x * chunk;
    const int ce = min(n, cs + chunk);
    const int rounds = (ce - cs + G - 1) / G;
    for (int rd = 0; rd < rounds; ++rd) {
        const int i = cs + rd * G + g;
        if (BAR) __syncthreads();   // team-synchronous rounds (a stage per round)
        if (i >= ce) continue;
        const int b = (int)__ldg(rp + i), e = (int)__ldg(rp + i + 1);
        double acc = 0.0;
        for (int k = b + lane; k < e; k += S) {
            int c;
            double v, xv;
            asm volatile("ld.shared.s32 %0, [%1];" : "=r"(c) : "r"(sptr(scol + (k & 4095))));
            asm volatile("ld.shared.f64 %0, [%1];" : "=d"(v) : "r"(sptr(sval + (k & 4095))));
            if (FAR && (k & 15) == 0)
                xv = __ldg(x + (unsigned)c % (unsigned)n);
            else
                asm volatile("ld.shared.f64 %0, [%1];" : "=d"(xv) : "r"(sptr(xwin + (c & 8191))));
            acc = fma(v, xv, acc);
        }
#pragma unroll
        for (int off = S / 2; off >= 1; off >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, off);
        if (lane == 0) y[i] = acc;
    }
}

__global__ void flush_kernel(int4* p, size_t n) {
    for (size_t k = blockIdx.x * (size_t)blockDim.x + threadIdx.x; k < n; k += (size_t)gridDim.x * blockDim.x)
        p[k] = make_int4((int)k, 1, 2, 3);
}

typedef void (*SpmvFn)(const int64_t*, const int*, const double*, const double*, double*, int, int, int);

int main(int argc, char** argv) {
    const int n = argc > 1 ? atoi(argv[1]) : 10000000;
    const int far_den = argc > 2 ? atoi(argv[2]) : 16;
    cudaDeviceProp prop;
    CK(cudaGetDeviceProperties(&prop, 0));
    const size_t flush_bytes = 512ull << 20;
    int4* fl;
    CK(cudaMalloc(&fl, flush_bytes));
    cudaEvent_t e0, e1;
    CK(cudaEventCreate(&e0));
    CK(cudaEventCreate(&e1));
    std::vector<int64_t> rp(n + 1);
    rp[0] = 0;
    for (int i = 0; i < n; ++i) rp[i + 1] = rp[i] + 4 + (int)(mix(20230809ull ^ (uint64_t)i * 77) % 9);
    const int nnz = (int)rp[n];
    int64_t* drp;
    int* dcol;
    double *dval, *dx, *dy, *dy0;
    CK(cudaMalloc(&drp, (n + 1) * 8ull));
    CK(cudaMalloc(&dcol, nnz * 4ull));
    CK(cudaMalloc(&dval, nnz * 8ull + 64));
    CK(cudaMalloc(&dx, n * 8ull));
    CK(cudaMalloc(&dy, n * 8ull));
    CK(cudaMalloc(&dy0, n * 8ull));
    CK(cudaMemcpy(drp, rp.data(), (n + 1) * 8ull, cudaMemcpyHostToDevice));
    gen_cols<<<(n + 255) / 256, 256>>>(drp, n, dcol, dval, 4096, far_den, 20230809ull);
    std::vector<double> hx(n);
    for (int i = 0; i < n; ++i) hx[i] = (double)(mix(i * 3ull + 1) >> 11) * 0x1p-53 * 2 - 1;
    CK(cudaMemcpy(dx, hx.data(), n * 8ull, cudaMemcpyHostToDevice));
    cudaResourceDesc rd;
    memset(&rd, 0, sizeof(rd));
    rd.resType = cudaResourceTypeLinear;
    rd.res.linear.devPtr = dx;
    rd.res.linear.desc = cudaCreateChannelDesc<int2>();
    rd.res.linear.sizeInBytes = n * 8ull;
    cudaTextureDesc td;
    memset(&td, 0, sizeof(td));
    td.readMode = cudaReadModeElementType;
    cudaTextureObject_t tex;
    CK(cudaCreateTextureObject(&tex, &rd, &td, nullptr));
    CK(cudaMemcpyToSymbol(g_xtex, &tex, sizeof(tex)));
    CK(cudaDeviceSynchronize());
    const double alg = nnz * 12.0 + (n + 1) * 8.0 + n * 8.0 + n * 8.0;
    printf("# %s n=%d nnz=%d far 1/%d alg %.3f GB maxTex1DLinear %d\n", prop.name, n, nnz, far_den, alg * 1e-9,
           prop.maxTexture1DLinear);
    struct V {
        const char* name;
        SpmvFn fn;
        int T = 1024;
        int smem = 0;
        const char* ref = nullptr;
        int apw = 0;   // set-aside MB of a persisting L2 access-policy window over x (reset before every launch)
        int rows_per_team = 0;   // > 0: non-persistent grid of ceil(n / rows_per_team) teams
    } vs[] = {
        {"S2 quads ldg (headline)", spmv_q<2, 0>, 1024, 0, "q"},
        {"S2 quads timed teams", spmv_qt<2>, 1024, 0, nullptr, 0},
        {"S2 quads timed teams apw", spmv_qt<2>, 1024, 0, nullptr, 63},
    };
    int k = 0;
    for (auto& v : vs) {
        ++k;
        int nb = 0;
        if (v.smem > 48 * 1024) CK(cudaFuncSetAttribute(v.fn, cudaFuncAttributeMaxDynamicSharedMemorySize, v.smem));
        CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, v.fn, v.T, v.smem));
        const int grid = v.rows_per_team ? (n + v.rows_per_team - 1) / v.rows_per_team : prop.multiProcessorCount * nb;
        int chunk = (n + grid - 1) / grid;
        chunk = (chunk + 31) / 32 * 32;
        std::vector<float> ts;
        cudaStream_t st = 0;
        if (v.apw) {
            CK(cudaStreamCreate(&st));
            const size_t setaside = std::min((size_t)prop.persistingL2CacheMaxSize, (size_t)v.apw << 20);
            CK(cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, setaside));
            cudaStreamAttrValue a;
            memset(&a, 0, sizeof(a));
            a.accessPolicyWindow.base_ptr = dx;
            a.accessPolicyWindow.num_bytes = std::min((size_t)n * 8, (size_t)prop.accessPolicyMaxWindowSize);
            a.accessPolicyWindow.hitRatio = std::min(1.0f, (float)setaside / (float)a.accessPolicyWindow.num_bytes);
            a.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
            a.accessPolicyWindow.missProp = cudaAccessPropertyNormal;
            CK(cudaStreamSetAttribute(st, cudaStreamAttributeAccessPolicyWindow, &a));
            printf("   apw: setaside %zu MB window %zu MB hitRatio %.2f\n", setaside >> 20,
                   (size_t)a.accessPolicyWindow.num_bytes >> 20, a.accessPolicyWindow.hitRatio);
        }
        for (int r = 0; r < 13; ++r) {
            if (v.apw) CK(cudaCtxResetPersistingL2Cache());
            flush_kernel<<<4 * prop.multiProcessorCount, 1024, 0, st>>>(fl, flush_bytes / 16);
            if (strstr(v.name, "pool")) zero_pool<<<1, 1, 0, st>>>();
            CK(cudaEventRecord(e0, st));
            v.fn<<<grid, v.T, v.smem, st>>>(drp, dcol, dval, dx, dy, n, chunk, nnz);
            CK(cudaEventRecord(e1, st));
            CK(cudaEventSynchronize(e1));
            float ms;
            CK(cudaEventElapsedTime(&ms, e0, e1));
            if (r >= 3) ts.push_back(ms);
        }
        CK(cudaGetLastError());
        if (v.apw) {
            cudaStreamAttrValue a;
            memset(&a, 0, sizeof(a));
            CK(cudaStreamSetAttribute(st, cudaStreamAttributeAccessPolicyWindow, &a));
            CK(cudaCtxResetPersistingL2Cache());
            CK(cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, 0));
            CK(cudaStreamSynchronize(st));
            CK(cudaStreamDestroy(st));
        }
        std::sort(ts.begin(), ts.end());
        const float med = ts[ts.size() / 2];
        const char* tag = "(ref)";
        if (v.ref) {
            CK(cudaMemcpy(dy0, dy, n * 8ull, cudaMemcpyDeviceToDevice));
        } else {
            std::vector<double> a(n), b(n);
            CK(cudaMemcpy(a.data(), dy, n * 8ull, cudaMemcpyDeviceToHost));
            CK(cudaMemcpy(b.data(), dy0, n * 8ull, cudaMemcpyDeviceToHost));
            tag = memcmp(a.data(), b.data(), n * 8ull) ? "differs" : "bit-identical";
        }
        printf("%2d %-28s grid %4d median %.4f ms min %.4f  %.0f GB/s alg  %s\n", k, v.name, grid, med, ts[0],
               alg / med * 1e-6, tag);
        if (strstr(v.name, "timed")) {
            std::vector<unsigned long long> t0(grid), t1(grid);
            CK(cudaMemcpyFromSymbol(t0.data(), g_t0, grid * 8));
            CK(cudaMemcpyFromSymbol(t1.data(), g_t1, grid * 8));
            const unsigned long long base = *std::min_element(t0.begin(), t0.end());
            std::vector<double> st(grid), en(grid);
            for (int q = 0; q < grid; ++q) st[q] = (t0[q] - base) * 1e-3, en[q] = (t1[q] - base) * 1e-3;
            std::sort(st.begin(), st.end());
            std::sort(en.begin(), en.end());
            if (getenv("XG_DUMP")) {
                char fn[512];
                snprintf(fn, sizeof fn, "%s_%d.txt", getenv("XG_DUMP"), k);
                FILE* f = fopen(fn, "w");
                for (int q = 0; q < grid; ++q) fprintf(f, "%d %.2f %.2f\n", q, (t0[q] - base) * 1e-3, (t1[q] - base) * 1e-3);
                fclose(f);
            }
            printf("   team start us: min %.1f median %.1f max %.1f | team end us: min %.1f p10 %.1f median %.1f p90 %.1f max %.1f\n",
                   st[0], st[grid / 2], st[grid - 1], en[0], en[grid / 10], en[grid / 2], en[grid * 9 / 10], en[grid - 1]);
        }
    }
    // ---- DRAM-side diagnostic (stream_gather); time here, bytes under ncu
    typedef void (*SgFn)(const int*, const double*, const double*, int, double*);
    struct W {
        const char* name;
        SgFn fn;
    } ws[] = {{"sg csr normal, x normal", stream_gather<0, 0>},
              {"sg csr evict_first, x normal", stream_gather<1, 0>},
              {"sg csr evict_first, x evict_last", stream_gather<1, 1>},
              {"sg csr L1na+evict_first, x evict_last", stream_gather<2, 1>},
              {"sg csr normal, x evict_last", stream_gather<0, 1>}};
    for (auto& w : ws) {
        std::vector<float> ts;
        for (int r = 0; r < 8; ++r) {
            flush_kernel<<<4 * prop.multiProcessorCount, 1024>>>(fl, flush_bytes / 16);
            CK(cudaEventRecord(e0));
            w.fn<<<2 * prop.multiProcessorCount, 1024>>>(dcol, dval, dx, nnz, dy);
            CK(cudaEventRecord(e1));
            CK(cudaEventSynchronize(e1));
            float ms;
            CK(cudaEventElapsedTime(&ms, e0, e1));
            if (r >= 3) ts.push_back(ms);
        }
        CK(cudaGetLastError());
        std::sort(ts.begin(), ts.end());
        printf("   %-40s median %.4f ms\n", w.name, ts[ts.size() / 2]);
    }
    return 0;
}
