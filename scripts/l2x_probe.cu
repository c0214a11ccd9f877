// l2x_probe.cu -- developer micro-benchmark (not part of the library):
// can x (80 MB of fp64) stay L2-resident while the 1.12 GB CSR matrix streams
// through L2?  The headline SpMV reads 1.54 GB of DRAM for 1.12 GB of
// algorithmic reads; the excess is far gathers of x that miss L2
// (profiles/r01_l2_traffic_experiments.md).  Two parts:
//   cap    warm random 8-byte gathers over footprints of 16..160 MB: where does
//          the effective L2 capacity for a random gather end?
//   spmv   a stand-alone copy of the headline kernel's structure (blocked teams
//          of 1024, simdlen 2, 128-bit pair loads) on a cfg2-shaped matrix,
//          with L1/L2 eviction-priority variants for the x gathers and the CSR
//          stream, an L2 prefetch of x at kernel start, and an access-policy
//          window (persisting) over x.
// nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -lineinfo -o scripts/l2x_probe scripts/l2x_probe.cu
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <string>
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

// ------------------------------------------------------------------ loads
template <int P>
__device__ __forceinline__ double ldx(const double* p, uint64_t pol) {
    double r;
    if constexpr (P == 0) {
        r = __ldg(p);
    } else if constexpr (P == 1) {
        asm volatile("ld.global.nc.L2::cache_hint.f64 %0, [%1], %2;" : "=d"(r) : "l"(p), "l"(pol));
    } else if constexpr (P == 2) {
        asm volatile("ld.global.nc.L1::evict_last.L2::cache_hint.f64 %0, [%1], %2;" : "=d"(r) : "l"(p), "l"(pol));
    } else {
        asm volatile("ld.global.nc.L1::evict_last.f64 %0, [%1];" : "=d"(r) : "l"(p));
    }
    return r;
}
template <int P>
__device__ __forceinline__ void ldcsr(const int* c, const double* v, uint64_t pol, int2& cc, double2& vv) {
    if constexpr (P == 0) {
        cc = __ldg(reinterpret_cast<const int2*>(c));
        vv = __ldg(reinterpret_cast<const double2*>(v));
    } else if constexpr (P == 1) {
        asm volatile("ld.global.nc.L1::no_allocate.v2.s32 {%0, %1}, [%2];" : "=r"(cc.x), "=r"(cc.y) : "l"(c));
        asm volatile("ld.global.nc.L1::no_allocate.v2.f64 {%0, %1}, [%2];" : "=d"(vv.x), "=d"(vv.y) : "l"(v));
    } else if constexpr (P == 2) {
        asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v2.s32 {%0, %1}, [%2], %3;"
                     : "=r"(cc.x), "=r"(cc.y) : "l"(c), "l"(pol));
        asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v2.f64 {%0, %1}, [%2], %3;"
                     : "=d"(vv.x), "=d"(vv.y) : "l"(v), "l"(pol));
    } else {
        asm volatile("ld.global.nc.L1::evict_first.v2.s32 {%0, %1}, [%2];" : "=r"(cc.x), "=r"(cc.y) : "l"(c));
        asm volatile("ld.global.nc.L1::evict_first.v2.f64 {%0, %1}, [%2];" : "=d"(vv.x), "=d"(vv.y) : "l"(v));
    }
}

// ------------------------------------------------------- capacity probe
__global__ void gather_kernel(const double* __restrict__ x, uint32_t n, int iters, uint64_t seed, double* sink) {
    uint64_t s = mix(seed ^ (blockIdx.x * 1024ull + threadIdx.x));
    double acc = 0;
    for (int it = 0; it < iters; ++it) {
        s = mix(s);
        acc += __ldg(x + (uint32_t)(((s & 0xffffffffull) * n) >> 32));
    }
    if (acc == 12345.678) sink[0] = acc;
}

// ----------------------------------------------------------- matrix gen
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
    for (int a = 1; a < len; ++a)   // insertion sort (duplicates allowed: traffic study only)
        for (int q = a; q > 0 && c[q - 1] > c[q]; --q) {
            int t = c[q];
            c[q] = c[q - 1];
            c[q - 1] = t;
        }
    for (int k = 0; k < len; ++k) col[b + k] = c[k];
}

// ------------------------------------------------------------ the SpMV
// Blocked teams: team b owns rows [b*chunk, (b+1)*chunk); its G = T/2 groups
// take them cyclically; lane l of a group takes tuples l, l+2, ... (pairs).
template <int XP, int CP, bool PF, int XM = 0>
__global__ void __launch_bounds__(1024, 2)
    spmv(const int64_t* __restrict__ rp, const int* __restrict__ col, const double* __restrict__ val,
         const double* __restrict__ x, double* __restrict__ y, int n, int chunk, int nnz, int64_t xbytes) {
    uint64_t polx = 0, polc = 0;
    if constexpr (XP == 1 || XP == 2) asm("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(polx));
    if constexpr (CP == 2) asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(polc));
    if constexpr (PF) {
        // the team's share of x, prefetched to L2 (evict_last) in 32 KB pieces by warp 0
        const int64_t per = ((xbytes + gridDim.x - 1) / gridDim.x + 15) & ~(int64_t)15;
        const int64_t b0 = per * blockIdx.x;
        const int64_t e0 = min(xbytes, b0 + per);
        uint64_t pl;
        asm("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pl));
        if (threadIdx.x < 32)
            for (int64_t o = b0 + (int64_t)threadIdx.x * 32768; o < e0; o += 32 * 32768) {
                const uint32_t sz = (uint32_t)min((int64_t)32768, e0 - o);
                asm volatile("cp.async.bulk.prefetch.L2.global.L2::cache_hint [%0], %1, %2;" ::"l"(
                                 reinterpret_cast<const char*>(x) + o),
                             "r"(sz & ~15u), "l"(pl)
                             : "memory");
            }
    }
    const int G = blockDim.x >> 1;
    const int g = threadIdx.x >> 1, lane = threadIdx.x & 1;
    const int cs = blockIdx.x * chunk;
    const int ce = min(n, cs + chunk);
    for (int i = cs + g; i < ce; i += G) {
        const int b = (int)__ldg(rp + i), e = (int)__ldg(rp + i + 1);
        const int trip = e > b ? ((e + 1) >> 1) - (b >> 1) : 0;
        double acc = 0.0;
        for (int t = lane; t < trip; t += 2) {
            const int k0 = ((b >> 1) + t) << 1;
            int2 cc;
            double2 vv;
            if (k0 + 2 <= nnz) {
                ldcsr<CP>(col + k0, val + k0, polc, cc, vv);
            } else {
                cc.x = col[k0], cc.y = cc.x, vv.x = val[k0], vv.y = 0.0;
            }
            if constexpr (XM == 1) {
                if (k0 >= b) acc = fma(vv.x, (double)cc.x, acc);
                if (k0 + 1 < e) acc = fma(vv.y, (double)cc.y, acc);
            } else if constexpr (XM == 2) {
                if (k0 >= b) acc = fma(vv.x, ldx<XP>(x + (cc.x & 1023), polx), acc);
                if (k0 + 1 < e) acc = fma(vv.y, ldx<XP>(x + (cc.y & 1023), polx), acc);
            } else {
                if (k0 >= b) acc = fma(vv.x, ldx<XP>(x + cc.x, polx), acc);
                if (k0 + 1 < e) acc = fma(vv.y, ldx<XP>(x + cc.y, polx), acc);
            }
        }
        acc += __shfl_xor_sync(0xffffffffu, acc, 1);
        if (lane == 0) y[i] = acc;
    }
}


// ---------------------------------------------- MLP variants (tuple body)
// Group of S lanes per row; tuples of V nonzeros (128-bit loads); lane l takes
// tuples l, l+S, ...  The first UNR iterations are issued as one predicated
// block (all tuple loads, then all x gathers, then the FMAs in iteration
// order -- same per-lane order as the plain loop), the rest in a plain loop.
template <int S, int V, int UNR, int MINB, int XL = 0, bool RPF = false, int TB = 1024, int XS = 0>
__global__ void __launch_bounds__(TB, MINB)
    spmv2(const int64_t* __restrict__ rp, const int* __restrict__ col, const double* __restrict__ val,
          const double* __restrict__ x, double* __restrict__ y, int n, int chunk, int nnz, int64_t) {
    constexpr int LG = V == 2 ? 1 : 2;
    const int G = blockDim.x / S;
    const int g = threadIdx.x / S, lane = threadIdx.x % S;
    const int cs = blockIdx.x * chunk;
    const int ce = min(n, cs + chunk);
    const unsigned mask = S == 32 ? 0xffffffffu : (((1u << S) - 1) << (S * ((threadIdx.x & 31) / S)));
    extern __shared__ double xs[];   // XS: diagnostic -- gathers from an 8192-double shared window (wrong values)
    if constexpr (XS) {
        for (int k = threadIdx.x; k < 8192; k += blockDim.x) xs[k] = x[k];
        __syncthreads();
    }
    int nb = 0, ne = 0;
    if (RPF && cs + g < ce) nb = (int)__ldg(rp + cs + g), ne = (int)__ldg(rp + cs + g + 1);
    const int rounds = (ce - cs + G - 1) / G;
    for (int k = 0; k < rounds; ++k) {
        const int i = cs + g + k * G;
        if constexpr (XS == 2) {
            if (k % 4 == 0) __syncthreads();   // diag: a team barrier every 4 rows per group
        }
        if constexpr (XS == 3) {
            if (k % 16 == 0) __syncthreads();
        }
        if (i >= ce) continue;
        int b, e;
        if constexpr (RPF) {
            b = nb, e = ne;
            if (i + G < ce) nb = (int)__ldg(rp + i + G), ne = (int)__ldg(rp + i + G + 1);
        } else {
            b = (int)__ldg(rp + i), e = (int)__ldg(rp + i + 1);
        }
        const int trip = e > b ? ((e + V - 1) >> LG) - (b >> LG) : 0;
        double acc = 0.0;
        int c[UNR][V];
        double v[UNR][V];
#pragma unroll
        for (int u = 0; u < UNR; ++u) {
            const int t = lane + u * S;
            const int k0 = ((b >> LG) + t) << LG;
            if (t < trip && k0 + V <= nnz) {
                if constexpr (V == 2) {
                    const int2 cc = __ldg(reinterpret_cast<const int2*>(col + k0));
                    const double2 vv = __ldg(reinterpret_cast<const double2*>(val + k0));
                    c[u][0] = cc.x, c[u][1] = cc.y, v[u][0] = vv.x, v[u][1] = vv.y;
                } else {
                    const int4 cc = __ldg(reinterpret_cast<const int4*>(col + k0));
                    const double2 v0 = __ldg(reinterpret_cast<const double2*>(val + k0));
                    const double2 v1 = __ldg(reinterpret_cast<const double2*>(val + k0 + 2));
                    c[u][0] = cc.x, c[u][1] = cc.y, c[u][2] = cc.z, c[u][3] = cc.w;
                    v[u][0] = v0.x, v[u][1] = v0.y, v[u][2] = v1.x, v[u][3] = v1.y;
                }
            } else {
#pragma unroll
                for (int q = 0; q < V; ++q) {
                    const int kq = k0 + q < nnz ? k0 + q : nnz - 1;
                    c[u][q] = t < trip ? __ldg(col + kq) : 0;
                    v[u][q] = t < trip ? __ldg(val + kq) : 0.0;
                }
            }
        }
        double xv[UNR][V];
#pragma unroll
        for (int u = 0; u < UNR; ++u) {
            const int k0 = ((b >> LG) + lane + u * S) << LG;
#pragma unroll
            for (int q = 0; q < V; ++q)
                xv[u][q] = (lane + u * S < trip && k0 + q >= b && k0 + q < e)
                               ? (XS ? xs[c[u][q] & 8191] : ldx<XL>(x + c[u][q], 0)) : 0.0;
        }
#pragma unroll
        for (int u = 0; u < UNR; ++u) {
            const int k0 = ((b >> LG) + lane + u * S) << LG;
#pragma unroll
            for (int q = 0; q < V; ++q)
                if (lane + u * S < trip && k0 + q >= b && k0 + q < e) acc = fma(v[u][q], xv[u][q], acc);
        }
        for (int t = lane + UNR * S; t < trip; t += S) {
            const int k0 = ((b >> LG) + t) << LG;
#pragma unroll
            for (int q = 0; q < V; ++q) {
                const int k = k0 + q;
                if (k >= b && k < e) acc = fma(__ldg(val + k), __ldg(x + __ldg(col + k)), acc);
            }
        }
#pragma unroll
        for (int off = S / 2; off >= 1; off >>= 1) acc += __shfl_xor_sync(mask, acc, off);
        if (lane == 0) y[i] = acc;
    }
}

__global__ void read_kernel(const int4* p, size_t n, double* sink) {
    int acc = 0;
    for (size_t k = blockIdx.x * (size_t)blockDim.x + threadIdx.x; k < n; k += (size_t)gridDim.x * blockDim.x)
        acc += __ldcg(p + n + k).x;   // the second half of the flush buffer
    if (acc == 0x7fffffff) sink[0] = acc;
}

__global__ void flush_kernel(int4* p, size_t n) {
    for (size_t k = blockIdx.x * (size_t)blockDim.x + threadIdx.x; k < n; k += (size_t)gridDim.x * blockDim.x)
        p[k] = make_int4((int)k, 1, 2, 3);
}

typedef void (*SpmvFn)(const int64_t*, const int*, const double*, const double*, double*, int, int, int, int64_t);

int main(int argc, char** argv) {
    const char* part = argc > 1 ? argv[1] : "all";
    int dev = 0;
    CK(cudaSetDevice(dev));
    cudaDeviceProp prop;
    CK(cudaGetDeviceProperties(&prop, dev));
    printf("# %s, %d SMs, L2 %d MB, persisting max %zu MB, accessPolicyMaxWindow %d MB\n", prop.name,
           prop.multiProcessorCount, prop.l2CacheSize >> 20, (size_t)prop.persistingL2CacheMaxSize >> 20,
           prop.accessPolicyMaxWindowSize >> 20);
    double* sink;
    CK(cudaMalloc(&sink, 64));
    cudaEvent_t e0, e1;
    CK(cudaEventCreate(&e0));
    CK(cudaEventCreate(&e1));
    const size_t flush_bytes = 512ull << 20;
    int4* fl;
    CK(cudaMalloc(&fl, flush_bytes));
    auto flush = [&]() { flush_kernel<<<4 * prop.multiProcessorCount, 1024>>>(fl, flush_bytes / 16); };
    // write flush followed by a 256 MB read: L2 ends clean (no dirty write-backs inside the timed kernel)
    auto flush_wr = [&]() {
        flush();
        read_kernel<<<4 * prop.multiProcessorCount, 1024>>>(fl, flush_bytes / 32, sink);
    };

    if (!strcmp(part, "all") || !strcmp(part, "cap")) {
        const size_t maxb = 192ull << 20;
        double* x;
        CK(cudaMalloc(&x, maxb));
        CK(cudaMemset(x, 0, maxb));
        const int blocks = prop.multiProcessorCount * 2, iters = 2048;
        const double ng = (double)blocks * 1024 * iters;
        for (int mb : {8, 16, 32, 48, 64, 72, 80, 88, 96, 112, 128, 160, 192}) {
            const uint32_t n = (uint32_t)(((size_t)mb << 20) / 8);
            for (int w = 0; w < 3; ++w) gather_kernel<<<blocks, 1024>>>(x, n, iters, 17 + w, sink);
            float best = 1e30f;
            for (int r = 0; r < 5; ++r) {
                CK(cudaEventRecord(e0));
                gather_kernel<<<blocks, 1024>>>(x, n, iters, 100 + r, sink);
                CK(cudaEventRecord(e1));
                CK(cudaEventSynchronize(e1));
                float ms;
                CK(cudaEventElapsedTime(&ms, e0, e1));
                best = std::min(best, ms);
            }
            printf("cap %4d MB  %.3f ms  %.2f G gathers/s  (%.0f GB/s of 32B sectors)\n", mb, best,
                   ng / best * 1e-6, ng * 32 / best * 1e-6);
        }
        CK(cudaFree(x));
    }
    if (!strcmp(part, "all") || !strcmp(part, "spmv")) {
        // argv[2] = "file:<prefix>": read <prefix>_rp.bin (int64), _col.bin (int32), _val.bin, _x.bin (f64)
        const bool from_file = argc > 2 && !strncmp(argv[2], "file:", 5);
        auto slurp = [](const std::string& fn, std::vector<char>& buf) {
            FILE* f = fopen(fn.c_str(), "rb");
            if (!f) { fprintf(stderr, "cannot open %s\n", fn.c_str()); exit(1); }
            fseek(f, 0, SEEK_END);
            buf.resize(ftell(f));
            fseek(f, 0, SEEK_SET);
            if (fread(buf.data(), 1, buf.size(), f) != buf.size()) exit(1);
            fclose(f);
        };
        std::vector<char> frp, fcol, fval, fx;
        if (from_file) {
            const std::string pre = argv[2] + 5;
            slurp(pre + "_rp.bin", frp), slurp(pre + "_col.bin", fcol), slurp(pre + "_val.bin", fval), slurp(pre + "_x.bin", fx);
        }
        const int n = from_file ? (int)(frp.size() / 8 - 1) : (argc > 2 ? atoi(argv[2]) : 10000000);
        const int far_den = argc > 3 ? atoi(argv[3]) : 16;
        std::vector<int64_t> rp(n + 1);
        rp[0] = 0;
        if (from_file) memcpy(rp.data(), frp.data(), frp.size());
        else for (int i = 0; i < n; ++i) rp[i + 1] = rp[i] + 4 + (int)(mix(20230809ull ^ (uint64_t)i * 77) % 9);
        const int nnz = (int)rp[n];
        int64_t* drp;
        int* dcol;
        double *dval, *dx, *dy, *dy0;
        CK(cudaMalloc(&drp, (n + 1) * 8ull));
        CK(cudaMalloc(&dcol, nnz * 4ull));
        CK(cudaMalloc(&dval, nnz * 8ull));
        CK(cudaMalloc(&dx, n * 8ull));
        CK(cudaMalloc(&dy, n * 8ull));
        CK(cudaMalloc(&dy0, n * 8ull));
        CK(cudaMemcpy(drp, rp.data(), (n + 1) * 8ull, cudaMemcpyHostToDevice));
        if (from_file) {
            CK(cudaMemcpy(dcol, fcol.data(), fcol.size(), cudaMemcpyHostToDevice));
            CK(cudaMemcpy(dval, fval.data(), fval.size(), cudaMemcpyHostToDevice));
            CK(cudaMemcpy(dx, fx.data(), fx.size(), cudaMemcpyHostToDevice));
        } else {
            gen_cols<<<(n + 255) / 256, 256>>>(drp, n, dcol, dval, 4096, far_den, 20230809ull);
            std::vector<double> hx(n);
            for (int i = 0; i < n; ++i) hx[i] = (double)(mix(i * 3ull + 1) >> 11) * 0x1p-53 * 2 - 1;
            CK(cudaMemcpy(dx, hx.data(), n * 8ull, cudaMemcpyHostToDevice));
        }
        CK(cudaDeviceSynchronize());
        const double alg = nnz * 12.0 + (n + 1) * 8.0 + n * 8.0 + n * 8.0;
        const int G = 32;   // chunk granularity (a multiple of every variant's groups per warp)
        printf("# spmv n=%d nnz=%d far 1/%d alg %.3f GB\n", n, nnz, far_den, alg * 1e-9);
        struct V {
            const char* name;
            SpmvFn fn;
            int apw;   // 1: persisting access-policy window over x
            int T = 1024;
        } vs[] = {
            {"base(nc/nc)", spmv<0, 0, false>, 0},
            {"x:L2last", spmv<1, 0, false>, 0},
            {"x:L1last+L2last", spmv<2, 0, false>, 0},
            {"x:L1last", spmv<3, 0, false>, 0},
            {"csr:L1noalloc", spmv<0, 1, false>, 0},
            {"csr:L1na+L2first", spmv<0, 2, false>, 0},
            {"csr:L1first", spmv<0, 3, false>, 0},
            {"x:L2last csr:L1na", spmv<1, 1, false>, 0},
            {"x:L2last csr:L1na+L2first", spmv<1, 2, false>, 0},
            {"pf x:L2last", spmv<1, 0, true>, 0},
            {"pf x:L2last csr:L1na", spmv<1, 1, true>, 0},
            {"pf x:L2last csr:L1na+L2first", spmv<1, 2, true>, 0},
            {"pf base", spmv<0, 0, true>, 0},
            {"apw(x persisting)", spmv<0, 0, false>, 1},
            {"apw + csr:L1na", spmv<0, 1, false>, 1},
            {"diag: no x gather", spmv<0, 0, false, 1>, 0},
            {"diag: x gather in 8 KB (L1)", spmv<0, 0, false, 2>, 0},
            {"base, write+read flush", spmv<0, 0, false>, 2},
            {"S2 V2 U1 (=base)", spmv2<2, 2, 1, 2>, 2},
            {"S2 V2 U2", spmv2<2, 2, 2, 2>, 2},
            {"S2 V2 U2 minb1", spmv2<2, 2, 2, 1>, 2},
            {"S2 V2 U3", spmv2<2, 2, 3, 2>, 2},
            {"S2 V2 U4", spmv2<2, 2, 4, 2>, 2},
            {"S2 V2 U2 x:L1last", spmv2<2, 2, 2, 2, 3>, 2},
            {"S2 V2 U2 rowptr prefetch", spmv2<2, 2, 2, 2, 0, true>, 2},
            {"S2 V2 U2 x:L1last rp-pf", spmv2<2, 2, 2, 2, 3, true>, 2},
            {"S2 V2 U2 (write-only flush)", spmv2<2, 2, 2, 2>, 0},
            {"S2 V2 U3 T768x2", spmv2<2, 2, 3, 2, 0, false, 768>, 2, 768},
            {"diag: S2 V2 U2, head gathers from smem", spmv2<2, 2, 2, 2, 0, false, 1024, 1>, 2, 1024},
            {"diag: smem gathers + barrier every 4 rows", spmv2<2, 2, 2, 2, 0, false, 1024, 2>, 2, 1024},
            {"diag: smem gathers + barrier every 16 rows", spmv2<2, 2, 2, 2, 0, false, 1024, 3>, 2, 1024},
            {"S2 V2 U2 T768x2", spmv2<2, 2, 2, 2, 0, false, 768>, 2, 768},
            {"S2 V2 U4 T512x3", spmv2<2, 2, 4, 3, 0, false, 512>, 2, 512},
            {"S2 V2 U3 T512x3", spmv2<2, 2, 3, 3, 0, false, 512>, 2, 512},
            {"S2 V2 U2 T512x4", spmv2<2, 2, 2, 4, 0, false, 512>, 2, 512},
            {"S4 V2 U2 T768x2", spmv2<4, 2, 2, 2, 0, false, 768>, 2, 768},
            {"S1 V2 U4 T768x2", spmv2<1, 2, 4, 2, 0, false, 768>, 2, 768},
            {"S4 V2 U1", spmv2<4, 2, 1, 2>, 2},
            {"S4 V2 U2", spmv2<4, 2, 2, 2>, 2},
            {"S2 V4 U1", spmv2<2, 4, 1, 2>, 2},
            {"S2 V4 U2", spmv2<2, 4, 2, 2>, 2},
            {"S4 V4 U1", spmv2<4, 4, 1, 2>, 2},
            {"S8 V2 U1", spmv2<8, 2, 1, 2>, 2},
            {"S1 V4 U2", spmv2<1, 4, 2, 2>, 2},
            {"S1 V4 U3", spmv2<1, 4, 3, 2>, 2},
            {"S1 V2 U4 minb1", spmv2<1, 2, 4, 1>, 2},
            {"diag: no x, write+read flush", spmv<0, 0, false, 1>, 2},
        };
        const char* only = getenv("L2X_ONLY");
        int k = 0;
        for (auto& v : vs) {
            ++k;
            if (only && atoi(only) != k) continue;
            cudaStream_t st = 0;
            if (v.apw == 1) {
                size_t setaside = prop.persistingL2CacheMaxSize;
                CK(cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, setaside));
                cudaStreamAttrValue a;
                memset(&a, 0, sizeof(a));
                a.accessPolicyWindow.base_ptr = dx;
                a.accessPolicyWindow.num_bytes = std::min((size_t)n * 8, (size_t)prop.accessPolicyMaxWindowSize);
                a.accessPolicyWindow.hitRatio = std::min(1.0f, (float)setaside / (float)(a.accessPolicyWindow.num_bytes));
                a.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
                a.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
                CK(cudaStreamSetAttribute(st, cudaStreamAttributeAccessPolicyWindow, &a));
            }
            int nb = 0;
            const int T = v.T;
            CK(cudaFuncSetAttribute(v.fn, cudaFuncAttributeMaxDynamicSharedMemorySize, 65536));
            const size_t dsm = strstr(v.name, "smem") ? 65536 : 0;
            CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, v.fn, T, dsm));
            const int grid = prop.multiProcessorCount * nb;
            int chunk = (n + grid - 1) / grid;
            chunk = (chunk + G - 1) / G * G;
            std::vector<float> ts;
            for (int r = 0; r < 13; ++r) {
                if (v.apw == 1) CK(cudaCtxResetPersistingL2Cache());
                if (v.apw == 2) flush_wr(); else flush();
                CK(cudaEventRecord(e0, st));
                v.fn<<<grid, T, dsm, st>>>(drp, dcol, dval, dx, dy, n, chunk, nnz, (int64_t)n * 8);
                CK(cudaEventRecord(e1, st));
                CK(cudaEventSynchronize(e1));
                float ms;
                CK(cudaEventElapsedTime(&ms, e0, e1));
                if (r >= 3) ts.push_back(ms);
            }
            CK(cudaGetLastError());
            if (v.apw == 1) {
                cudaStreamAttrValue a;
                memset(&a, 0, sizeof(a));
                CK(cudaStreamSetAttribute(st, cudaStreamAttributeAccessPolicyWindow, &a));
                CK(cudaCtxResetPersistingL2Cache());
                CK(cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, 0));
            }
            std::sort(ts.begin(), ts.end());
            const float med = ts[ts.size() / 2];
            bool same = true;
            if (k == 1) {
                CK(cudaMemcpy(dy0, dy, n * 8ull, cudaMemcpyDeviceToDevice));
            } else {
                std::vector<double> a(n), b(n);
                CK(cudaMemcpy(a.data(), dy, n * 8ull, cudaMemcpyDeviceToHost));
                CK(cudaMemcpy(b.data(), dy0, n * 8ull, cudaMemcpyDeviceToHost));
                same = !memcmp(a.data(), b.data(), n * 8ull);
            }
            printf("spmv %2d %-30s median %.4f ms min %.4f ms  %.0f GB/s alg  %s\n", k, v.name, med, ts[0],
                   alg / med * 1e-6, k == 1 ? "(ref)" : (same ? "bit-identical" : "DIFFERS"));
        }
    }
    return 0;
}
