// stream_probe.cu -- developer micro-benchmark (not part of the library):
// how fast can one CTA per SM stream a 1.2 GB array through shared memory
// with cp.async.bulk + mbarriers (NS stages of SB bytes), versus plain
// 128-bit loads?  Consumers only touch one word per stage.
// nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o scripts/stream_probe scripts/stream_probe.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t* b, uint32_t c) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(su32(b)), "r"(c) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* b) {
    asm volatile("{ .reg .b64 s; mbarrier.arrive.shared::cta.b64 s, [%0]; }" ::"r"(su32(b)) : "memory");
}
__device__ __forceinline__ void mbar_arrive_tx(uint64_t* b, uint32_t tx) {
    asm volatile("{ .reg .b64 s; mbarrier.arrive.expect_tx.shared::cta.b64 s, [%0], %1; }" ::"r"(su32(b)), "r"(tx) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* b, uint32_t par) {
    uint32_t done = 0;
    do {
        asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0,1,0,p; }"
                     : "=r"(done) : "r"(su32(b)), "r"(par) : "memory");
    } while (!done);
}
__device__ __forceinline__ void bulk(void* d, const void* s, uint32_t n, uint64_t* b) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                 ::"r"(su32(d)), "l"(s), "r"(n), "r"(su32(b)) : "memory");
}

__global__ void tma_stream(const char* src, size_t bytes, int ns, int sb, int ncw, double* sink) {
    extern __shared__ __align__(16) unsigned char sm[];
    uint64_t* full = (uint64_t*)(sm + (size_t)ns * sb);
    uint64_t* empty = full + ns;
    const size_t per = (bytes / gridDim.x) & ~(size_t)15;
    const char* base = src + per * blockIdx.x;
    const int nst = (int)(per / sb);
    if (threadIdx.x == 0) {
        for (int s = 0; s < ns; ++s) { mbar_init(full + s, 1); mbar_init(empty + s, ncw); }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (warp == 0) {
        if (lane == 0)
            for (int k = 0; k < nst; ++k) {
                int s = k % ns;
                if (k >= ns) mbar_wait(empty + s, ((k / ns) - 1) & 1);
                mbar_arrive_tx(full + s, sb);
                bulk(sm + (size_t)s * sb, base + (size_t)k * sb, sb, full + s);
            }
        return;
    }
    double acc = 0;
    for (int k = 0; k < nst; ++k) {
        int s = k % ns;
        mbar_wait(full + s, (k / ns) & 1);
        const double* p = (const double*)(sm + (size_t)s * sb);
        for (int i = threadIdx.x - 32; i < sb / 8; i += blockDim.x - 32) acc += p[i];
        __syncwarp();
        if (lane == 0) mbar_arrive(empty + s);
    }
    if (acc == 12345.678) sink[0] = acc;
}

__global__ void ldg_stream(const double2* src, size_t n2, double* sink) {
    double a = 0, b = 0;
    size_t stride = (size_t)gridDim.x * blockDim.x;
    size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
    for (; i + 3 * stride < n2; i += 4 * stride) {
        double2 v0 = __ldcs(src + i), v1 = __ldcs(src + i + stride), v2 = __ldcs(src + i + 2 * stride), v3 = __ldcs(src + i + 3 * stride);
        a += v0.x + v1.x + v2.x + v3.x;
        b += v0.y + v1.y + v2.y + v3.y;
    }
    for (; i < n2; i += stride) { double2 v = src[i]; a += v.x; b += v.y; }
    if (a + b == 12345.678) sink[0] = a;
}

int main() {
    const size_t bytes = 1200ull << 20;
    char* buf; double* sink;
    cudaMalloc(&buf, bytes + 4096);
    cudaMalloc(&sink, 8);
    cudaMemset(buf, 0, bytes);
    int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    auto timeit = [&](auto fn) {
        fn(); cudaDeviceSynchronize();
        float best = 1e9;
        for (int r = 0; r < 5; ++r) { cudaEventRecord(e0); fn(); cudaEventRecord(e1); cudaEventSynchronize(e1);
            float ms; cudaEventElapsedTime(&ms, e0, e1); if (ms < best) best = ms; }
        return best;
    };
    float ms = timeit([&] { ldg_stream<<<sms * 8, 256>>>((const double2*)buf, bytes / 16, sink); });
    printf("ldg128 stream: %.3f ms  %.0f GB/s\n", ms, bytes / ms / 1e6);
    int cfgs[][3] = {{2, 32768, 1024}, {4, 32768, 1024}, {6, 32768, 1024}, {3, 65536, 1024}, {4, 49152, 1024},
                     {8, 16384, 1024}, {12, 16384, 1024}, {4, 32768, 256}, {6, 32768, 512}, {2, 98304, 1024}};
    for (auto& c : cfgs) {
        int ns = c[0], sb = c[1], T = c[2];
        size_t smem = (size_t)ns * sb + ns * 16;
        if (smem > 227 * 1024) continue;
        cudaFuncSetAttribute(tma_stream, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        int ncw = T / 32 - 1;
        int per_sm = (int)((228 * 1024) / (smem + 1024));
        if (per_sm > 2048 / T) per_sm = 2048 / T;
        for (int g : {sms, sms * per_sm}) {
            ms = timeit([&] { tma_stream<<<g, T, smem>>>(buf, bytes, ns, sb, ncw, sink); });
            printf("bulk ns=%d stage=%dKB T=%d grid=%d: %.3f ms  %.0f GB/s  (%s)\n", ns, sb / 1024, T, g, ms,
                   bytes / ms / 1e6, cudaGetErrorString(cudaGetLastError()));
        }
    }
    return 0;
}
