// xpeer.cu -- NEXT-4: the row-partitioned SpMV without an
// all-gather.  Each rank's x slice lives in a library-owned buffer that every
// peer maps (CUDA IPC over NVLink/NVSwitch); the simd lanes gather x[c] from
// the owning rank's slice (bodies.cuh XPeer), so the exchange step of a12
// (north_star: "an NCCL all-gather of x") is fused into the SpMV's loads and
// overlaps the matrix stream tile by tile.  Ordering between ranks: a flag
// barrier in peer memory (system-scope release stores / acquire loads).
#include <cuda_runtime.h>

#include <cstring>
#include <new>
#include <vector>

#include "dispatch.cuh"
#include "internal.h"

struct nest_xpeer {
    int32_t nranks = 0;
    int32_t rank = 0;
    int64_t ncols = 0;
    int64_t xchunk = 0;
    bool local = false;                  // nest_xpeer_create_local: no IPC, no barrier
    bool opened = false;
    double* x_own = nullptr;             // this rank's slice (IPC mode, library-owned)
    const double* own_slice = nullptr;   // this rank's slice as the kernel reads it (either form)
    uint64_t* flags_own = nullptr;       // barrier flags written by the peers (nranks)
    const double** d_slices = nullptr;   // device: nranks slice pointers
    uint64_t** d_peer_flags = nullptr;   // device: nranks pointers to each rank's flags
    std::vector<void*> ipc_opened;       // peer mappings to close
    uint64_t epoch = 0;
};

namespace nest {

template <class Body>
static int32_t xpeer_payload(int32_t U) {
    switch (U) {
        case 1: return payload_bytes<Body, 1>();
        case 2: return payload_bytes<Body, 2>();
        case 4: return payload_bytes<Body, 4>();
    }
    return -1;
}

nest_status launch_spmv_xpeer_vec(const Plan& p, const int64_t* rowptr, const int32_t* col, const double* val,
                                  XPeer xa, double* y, unsigned char* fb, cudaStream_t st, int64_t nnz);

__device__ __forceinline__ void st_release_sys(uint64_t* p, uint64_t v) {
    asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ uint64_t ld_acquire_sys(const uint64_t* p) {
    uint64_t v;
    asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}

// One team: lane r posts `epoch` into rank r's flag slot for this rank, then
// waits until every rank has posted it here.  Work ordered before the barrier
// on each rank's stream is visible to all peers after it (kernel boundary +
// system-scope fence and release/acquire).
__global__ void xpeer_barrier_kernel(uint64_t* const* peer_flags, const uint64_t* my_flags, int32_t rank,
                                     int32_t nranks, uint64_t epoch) {
    const int r = threadIdx.x;
    if (r < nranks) {
        __threadfence_system();
        st_release_sys(peer_flags[r] + rank, epoch);
        // bounded wait: a peer that never arrives (lost process, broken mapping)
        // traps after 120 s instead of hanging the stream forever
        uint64_t t0, t;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
        while (ld_acquire_sys(my_flags + r) < epoch) {
            __nanosleep(64);
            asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
            if (t - t0 > 120000000000ull) __trap();
        }
    }
    __syncthreads();
}

}  // namespace nest

using namespace nest;

static constexpr size_t kIpcBytes = sizeof(cudaIpcMemHandle_t);

static nest_status xpeer_free(nest_xpeer* xp) {
    cudaError_t first = cudaSuccess;
    auto keep = [&](cudaError_t e) {
        if (first == cudaSuccess && e != cudaSuccess) first = e;
    };
    for (void* p : xp->ipc_opened) keep(cudaIpcCloseMemHandle(p));
    if (xp->d_slices) keep(cudaFree(const_cast<double**>(xp->d_slices)));
    if (xp->d_peer_flags) keep(cudaFree(xp->d_peer_flags));
    if (xp->x_own) keep(cudaFree(xp->x_own));
    if (xp->flags_own) keep(cudaFree(xp->flags_own));
    delete xp;
    return first == cudaSuccess ? NEST_OK : cuda_fail(first, "nest_xpeer_destroy");
}

static nest_status xpeer_new(int32_t nranks, int32_t rank, int64_t ncols, nest_xpeer** out) {
    if (!out) return fail(NEST_ERR_INVALID_ARG, "out is NULL");
    *out = nullptr;
    if (nranks <= 0 || nranks > 1024 || rank < 0 || rank >= nranks)
        return fail(NEST_ERR_INVALID_ARG, "bad xpeer arguments (nranks %d, rank %d)", nranks, rank);
    if (ncols < 0 || ncols > INT32_MAX) return fail(NEST_ERR_INVALID_ARG, "ncols_global %lld", (long long)ncols);
    nest_xpeer* xp = new (std::nothrow) nest_xpeer;
    if (!xp) return fail(NEST_ERR_NO_MEMORY, "nest_xpeer");
    xp->nranks = nranks;
    xp->rank = rank;
    xp->ncols = ncols;
    xp->xchunk = (ncols + nranks - 1) / nranks;
    *out = xp;
    return NEST_OK;
}

NEST_API size_t nest_xpeer_handle_bytes(void) { return 2 * kIpcBytes; }

NEST_API nest_status nest_xpeer_create(int32_t nranks, int32_t rank, int64_t ncols_global, nest_xpeer** out,
                                       uint8_t* handle) {
    if (!handle) return fail(NEST_ERR_INVALID_ARG, "handle is NULL");
    nest_xpeer* xp = nullptr;
    nest_status s = xpeer_new(nranks, rank, ncols_global, &xp);
    if (s != NEST_OK) return s;
    cudaError_t e;
    cudaIpcMemHandle_t hx, hf;
    const size_t xbytes = (size_t)(xp->xchunk > 0 ? xp->xchunk : 1) * sizeof(double);
    if ((e = cudaMalloc(&xp->x_own, xbytes)) != cudaSuccess ||
        (e = cudaMalloc(&xp->flags_own, (size_t)nranks * sizeof(uint64_t))) != cudaSuccess ||
        (e = cudaMemset(xp->x_own, 0, xbytes)) != cudaSuccess ||
        (e = cudaMemset(xp->flags_own, 0, (size_t)nranks * sizeof(uint64_t))) != cudaSuccess ||
        (e = cudaIpcGetMemHandle(&hx, xp->x_own)) != cudaSuccess ||
        (e = cudaIpcGetMemHandle(&hf, xp->flags_own)) != cudaSuccess ||
        (e = cudaDeviceSynchronize()) != cudaSuccess) {
        xpeer_free(xp);
        return cuda_fail(e, "nest_xpeer_create");
    }
    std::memcpy(handle, &hx, kIpcBytes);
    std::memcpy(handle + kIpcBytes, &hf, kIpcBytes);
    *out = xp;
    return NEST_OK;
}

NEST_API nest_status nest_xpeer_open(nest_xpeer* xp, const uint8_t* all) {
    if (!xp || !all) return fail(NEST_ERR_INVALID_ARG, "xpeer/handles is NULL");
    if (xp->local || xp->opened) return fail(NEST_ERR_INVALID_ARG, "xpeer already open");
    const int P = xp->nranks;
    std::vector<const double*> slices(P);
    std::vector<uint64_t*> flags(P);
    for (int r = 0; r < P; ++r) {
        if (r == xp->rank) {
            slices[r] = xp->x_own;
            flags[r] = xp->flags_own;
            continue;
        }
        cudaIpcMemHandle_t hx, hf;
        std::memcpy(&hx, all + (size_t)r * 2 * kIpcBytes, kIpcBytes);
        std::memcpy(&hf, all + (size_t)r * 2 * kIpcBytes + kIpcBytes, kIpcBytes);
        void *px = nullptr, *pf = nullptr;
        cudaError_t e = cudaIpcOpenMemHandle(&px, hx, cudaIpcMemLazyEnablePeerAccess);
        if (e != cudaSuccess) return cuda_fail(e, "cudaIpcOpenMemHandle(x slice)");
        xp->ipc_opened.push_back(px);
        e = cudaIpcOpenMemHandle(&pf, hf, cudaIpcMemLazyEnablePeerAccess);
        if (e != cudaSuccess) return cuda_fail(e, "cudaIpcOpenMemHandle(flags)");
        xp->ipc_opened.push_back(pf);
        slices[r] = static_cast<const double*>(px);
        flags[r] = static_cast<uint64_t*>(pf);
    }
    cudaError_t e;
    if ((e = cudaMalloc(&xp->d_slices, P * sizeof(double*))) != cudaSuccess ||
        (e = cudaMalloc(&xp->d_peer_flags, P * sizeof(uint64_t*))) != cudaSuccess ||
        (e = cudaMemcpy(xp->d_slices, slices.data(), P * sizeof(double*), cudaMemcpyHostToDevice)) != cudaSuccess ||
        (e = cudaMemcpy(xp->d_peer_flags, flags.data(), P * sizeof(uint64_t*), cudaMemcpyHostToDevice)) !=
            cudaSuccess)
        return cuda_fail(e, "nest_xpeer_open");
    xp->opened = true;
    return NEST_OK;
}

NEST_API nest_status nest_xpeer_create_local(int32_t nranks, int32_t rank, int64_t ncols_global,
                                             const double* const* slices, nest_xpeer** out) {
    if (!slices) return fail(NEST_ERR_INVALID_ARG, "slices is NULL");
    nest_xpeer* xp = nullptr;
    nest_status s = xpeer_new(nranks, rank, ncols_global, &xp);
    if (s != NEST_OK) return s;
    for (int r = 0; r < nranks; ++r)
        if (!slices[r] && xp->xchunk > 0) {
            xpeer_free(xp);
            return fail(NEST_ERR_INVALID_ARG, "slice %d is NULL", r);
        }
    cudaError_t e;
    if ((e = cudaMalloc(&xp->d_slices, nranks * sizeof(double*))) != cudaSuccess ||
        (e = cudaMemcpy(xp->d_slices, slices, nranks * sizeof(double*), cudaMemcpyHostToDevice)) != cudaSuccess) {
        xpeer_free(xp);
        return cuda_fail(e, "nest_xpeer_create_local");
    }
    xp->local = true;
    xp->opened = true;
    xp->own_slice = slices[rank];
    *out = xp;
    return NEST_OK;
}

NEST_API double* nest_xpeer_local_x(nest_xpeer* xp) { return xp ? xp->x_own : nullptr; }
NEST_API int64_t nest_xpeer_xchunk(const nest_xpeer* xp) { return xp ? xp->xchunk : -1; }

NEST_API nest_status nest_xpeer_set_x(nest_xpeer* xp, const double* x_local, int64_t n, void* stream) {
    if (!xp || !xp->x_own) return fail(NEST_ERR_INVALID_ARG, "xpeer is NULL or has no own slice");
    if (n < 0 || (n > 0 && !x_local)) return fail(NEST_ERR_INVALID_ARG, "bad x_local");
    int64_t len = xp->ncols - (int64_t)xp->rank * xp->xchunk;
    if (len > xp->xchunk) len = xp->xchunk;
    if (len < 0) len = 0;
    if (n > len) n = len;
    if (n == 0) return NEST_OK;
    const cudaError_t e = cudaMemcpyAsync(xp->x_own, x_local, (size_t)n * sizeof(double), cudaMemcpyDeviceToDevice,
                                          static_cast<cudaStream_t>(stream));
    return e == cudaSuccess ? NEST_OK : cuda_fail(e, "nest_xpeer_set_x");
}

NEST_API nest_status nest_xpeer_barrier(nest_xpeer* xp, void* stream) {
    if (!xp || !xp->opened) return fail(NEST_ERR_INVALID_ARG, "xpeer is NULL or not open");
    if (xp->local || xp->nranks == 1) return NEST_OK;
    const int threads = (xp->nranks + 31) / 32 * 32;
    xpeer_barrier_kernel<<<1, threads, 0, static_cast<cudaStream_t>(stream)>>>(
        xp->d_peer_flags, xp->flags_own, xp->rank, xp->nranks, ++xp->epoch);
    const cudaError_t e = cudaGetLastError();
    return e == cudaSuccess ? NEST_OK : cuda_fail(e, "xpeer barrier launch");
}

NEST_API nest_status nest_spmv_csr_f64_xpeer(const nest_desc* desc, nest_xpeer* xp, int64_t nrows_global,
                                             int64_t nrows_local, int64_t nnz, const int64_t* rowptr,
                                             const int32_t* colind, const double* val, double* y,
                                             void* stream) {
    if (!xp || !xp->opened) return fail(NEST_ERR_INVALID_ARG, "xpeer is NULL or not open");
    if (nrows_global < 0 || nrows_local < 0 || nnz < 0) return fail(NEST_ERR_INVALID_ARG, "negative extent");
    const int64_t chunk = (nrows_global + xp->nranks - 1) / xp->nranks;
    int64_t b = (int64_t)xp->rank * chunk;
    if (b > nrows_global) b = nrows_global;
    const int64_t e_ = b + chunk < nrows_global ? b + chunk : nrows_global;
    if (nrows_local != e_ - b)
        return fail(NEST_ERR_INVALID_ARG, "rank %d owns %lld rows, got nrows_local %lld", xp->rank,
                    (long long)(e_ - b), (long long)nrows_local);
    Plan p;
    nest_status s = make_plan(desc, nrows_local, 1, spmv_payload, &p, true);
    if (s != NEST_OK) return s;
    if (desc->mode == NEST_MODE_TEAMS_GENERIC || (p.flags & (NEST_F_VEC_QUAD | NEST_F_X_L2_PERSIST)) || p.x_halo > 0)
        return fail(NEST_ERR_UNSUPPORTED,
                    "nest_spmv_csr_f64_xpeer: cyclic/blocked schedules with scalar or pair loads only");
    if (nrows_local > 0 && (!rowptr || !y)) return fail(NEST_ERR_INVALID_ARG, "rowptr/y is NULL");
    if (nnz > 0 && (!colind || !val)) return fail(NEST_ERR_INVALID_ARG, "colind/val is NULL");
    const bool vec = (p.flags & NEST_F_VEC128) != 0;
    const bool i32 = spmv_index32(p, nnz);
    if (vec && !i32) return fail(NEST_ERR_UNSUPPORTED, "NEST_F_VEC128 (xpeer) needs nnz_local < 2^31, nrows_local < 2^30");
    // the generic payload of the body that runs (the kernel follows the plan's fallback decision)
    const int32_t payload = vec ? xpeer_payload<SpmvVecBody<false, 2, int32_t, XPeer>>(p.unroll)
                                : xpeer_payload<SpmvBody<false, int64_t, XPeer>>(p.unroll);
    if (payload != p.payload_bytes && (s = make_plan_fixed(desc, nrows_local, 1, payload, &p, true)) != NEST_OK)
        return s;
    if (vec && ((reinterpret_cast<uintptr_t>(val) & 15) || (reinterpret_cast<uintptr_t>(colind) & 7)))
        return fail(NEST_ERR_UNSUPPORTED, "NEST_F_VEC128 needs 16-byte aligned val and 8-byte aligned colind");
    unsigned char* fb = nullptr;
    if ((s = prepare_fallback(p, &fb, stream)) != NEST_OK) return s;
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    // every rank's slice is written before anyone gathers from it
    if ((s = nest_xpeer_barrier(xp, stream)) != NEST_OK) return s;
    if (nrows_local > 0) {
        const XPeer xa{xp->d_slices, FastDivU32::make((uint32_t)(xp->xchunk > 0 ? xp->xchunk : 1)),
                       xp->local ? xp->own_slice : xp->x_own, (uint32_t)((int64_t)xp->rank * xp->xchunk)};
        if (vec) {
            s = launch_spmv_xpeer_vec(p, rowptr, colind, val, xa, y, fb, st, nnz);
        } else {
            SpmvBody<false, int64_t, XPeer> body{rowptr, colind, val, xa, y};
            body.nnz = nnz;
            s = dispatch(p, body, fb, st);
        }
    }
    // nobody overwrites its slice while a peer may still read it.  Posted even when
    // the launch failed (e.g. the variant's thread limit), so every rank's barrier
    // epochs stay in step and no peer waits for an epoch this rank never posts.
    const nest_status sb = nest_xpeer_barrier(xp, stream);
    return s != NEST_OK ? s : sb;
}

NEST_API nest_status nest_xpeer_destroy(nest_xpeer* xp) {
    if (!xp) return NEST_OK;
    cudaDeviceSynchronize();
    return xpeer_free(xp);
}
