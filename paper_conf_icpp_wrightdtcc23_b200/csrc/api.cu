// api.cu -- the C ABI of include/nest.h: validation, the a1 planner, the
// library-owned sharing-space fallback and the single-GPU entry points.
#include <cstdlib>
#include <cuda_runtime.h>

#include <algorithm>
#include <atomic>
#include <climits>
#include <cstdint>
#include <cstdarg>
#include <cstdio>
#include <map>
#include <mutex>
#include <utility>

#include "internal.h"

namespace nest {

static thread_local char g_err[512] = "";

nest_status fail(nest_status s, const char* fmt, ...) {
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(g_err, sizeof(g_err), fmt, ap);
    va_end(ap);
    return s;
}

nest_status cuda_fail(cudaError_t e, const char* what) {
    cudaGetLastError();   // clear a sticky-free error so the next call starts clean
    return fail(NEST_ERR_CUDA, "%s: %s (%s)", what, cudaGetErrorName(e), cudaGetErrorString(e));
}

static nest_status sm_count(int* out) {
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return cuda_fail(e, "cudaGetDevice");
    e = cudaDeviceGetAttribute(out, cudaDevAttrMultiProcessorCount, dev);
    if (e != cudaSuccess) return cuda_fail(e, "cudaDeviceGetAttribute(SM count)");
    return NEST_OK;
}

static bool valid_simdlen(int32_t s) {
    return s == 1 || s == 2 || s == 4 || s == 8 || s == 16 || s == 32;
}

static constexpr int32_t kDefaultThreads = 256;
static constexpr int32_t kDefaultSharing = 2048;
static constexpr int32_t kMaxSharing = 48 * 1024;       // static-carveout dynamic smem
static constexpr int32_t kMaxBlocksPerSm = 32;
static constexpr int32_t kMaxThreadsPerSm = 2048;
static constexpr int32_t kSmemPerSm = 228 * 1024;
static constexpr int32_t kSmemReservedPerBlock = 1024;

// Descriptor validation (groups are equal,
// inside one warp, and divide the team evenly).
static nest_status validate_desc(const nest_desc* d, int32_t* T, int32_t* sharing, int32_t* U) {
    if (!d) return fail(NEST_ERR_INVALID_ARG, "desc is NULL");
    if (d->abi_version != NEST_ABI_VERSION)
        return fail(NEST_ERR_INVALID_ARG, "abi_version %u != %u", d->abi_version, NEST_ABI_VERSION);
    *T = d->threads_per_team ? d->threads_per_team : kDefaultThreads;
    if (*T < 32 || *T > 1024 || *T % 32)
        return fail(NEST_ERR_INVALID_ARG, "threads_per_team %d: need a multiple of 32 in [32,1024]", *T);
    if (!valid_simdlen(d->simdlen))
        return fail(NEST_ERR_INVALID_ARG, "simdlen %d: need 1, 2, 4, 8, 16 or 32", d->simdlen);
    if (d->mode < NEST_MODE_SPMD || d->mode > NEST_MODE_TEAMS_GENERIC)
        return fail(NEST_ERR_INVALID_ARG, "mode %d", d->mode);
    if (d->mode == NEST_MODE_TEAMS_GENERIC && d->simdlen != 1)
        return fail(NEST_ERR_INVALID_ARG, "NEST_MODE_TEAMS_GENERIC is the two-level baseline: simdlen must be 1");
    if (d->mode == NEST_MODE_TEAMS_GENERIC && *T > 992)
        return fail(NEST_ERR_INVALID_ARG, "NEST_MODE_TEAMS_GENERIC: threads_per_team (workers) <= 992 (+ the main warp)");
    if (d->reduce < NEST_REDUCE_SUM || d->reduce > NEST_REDUCE_MIN)
        return fail(NEST_ERR_INVALID_ARG, "reduce %d", d->reduce);
    *sharing = d->sharing_bytes ? d->sharing_bytes : kDefaultSharing;
    if (*sharing < 0 || *sharing > kMaxSharing)
        return fail(NEST_ERR_INVALID_ARG, "sharing_bytes %d: need [0, %d]", d->sharing_bytes, kMaxSharing);
    if (d->num_teams < 0) return fail(NEST_ERR_INVALID_ARG, "num_teams %d < 0", d->num_teams);
    *U = d->outer_unroll ? d->outer_unroll : 1;
    if (*U != 1 && *U != 2 && *U != 4)
        return fail(NEST_ERR_INVALID_ARG, "outer_unroll %d: need 1, 2 or 4", d->outer_unroll);
    if (d->flags & ~(uint32_t)(NEST_F_PERSISTENT_GRID | NEST_F_STREAM_HINTS | NEST_F_BLOCKED |
                               NEST_F_VEC128 | NEST_F_VEC_QUAD | NEST_F_X_L2_PERSIST))
        return fail(NEST_ERR_INVALID_ARG, "unknown flags 0x%x", d->flags);
    if (d->teams_per_sm < 0 || d->teams_per_sm > 2)
        return fail(NEST_ERR_INVALID_ARG, "teams_per_sm %d: need 0, 1 or 2", d->teams_per_sm);
    if (d->teams_per_sm && d->x_halo <= 0)
        return fail(NEST_ERR_INVALID_ARG, "teams_per_sm applies to the x ring (x_halo > 0) only");
    if (d->team_chunk < 0) return fail(NEST_ERR_INVALID_ARG, "team_chunk %d < 0", d->team_chunk);
    if (d->team_chunk > 0 && !(d->flags & NEST_F_BLOCKED))
        return fail(NEST_ERR_INVALID_ARG, "team_chunk needs NEST_F_BLOCKED");
    return NEST_OK;
}

nest_status resident_blocks(int32_t T, int32_t smem, int64_t* out) {
    int sms = 0;
    nest_status s = sm_count(&sms);
    if (s != NEST_OK) return s;
    int32_t per_sm = kMaxBlocksPerSm;
    if (kMaxThreadsPerSm / T < per_sm) per_sm = kMaxThreadsPerSm / T;
    if (smem > 0) {
        const int32_t by_smem = kSmemPerSm / (smem + kSmemReservedPerBlock);
        if (by_smem < per_sm) per_sm = by_smem;
    }
    *out = (int64_t)sms * (per_sm > 0 ? per_sm : 1);
    return NEST_OK;
}

static nest_status plan_core(const nest_desc* d, int64_t outer, int32_t K, int32_t T,
                             int32_t sharing, int32_t U, int32_t payload, Plan* p, bool spmv_window) {
    if (outer < 0) return fail(NEST_ERR_INVALID_ARG, "outer iterations %lld < 0", (long long)outer);
    if (d->x_halo < 0) return fail(NEST_ERR_INVALID_ARG, "x_halo %d < 0", d->x_halo);
    if (d->x_halo > 0 && !spmv_window)
        return fail(NEST_ERR_INVALID_ARG, "x_halo applies to the CSR SpMV only (nest_spmv_plan)");
    if (d->mode == NEST_MODE_TEAMS_GENERIC && !spmv_window)
        return fail(NEST_ERR_INVALID_ARG, "NEST_MODE_TEAMS_GENERIC applies to the CSR SpMV only");
    if ((d->flags & NEST_F_VEC_QUAD) && !spmv_window)
        return fail(NEST_ERR_INVALID_ARG, "NEST_F_VEC_QUAD applies to the CSR SpMV only");
    if ((d->flags & NEST_F_X_L2_PERSIST) && !spmv_window)
        return fail(NEST_ERR_INVALID_ARG, "NEST_F_X_L2_PERSIST applies to the CSR SpMV only");
    if ((d->flags & NEST_F_VEC_QUAD) && !(d->flags & NEST_F_VEC128))
        return fail(NEST_ERR_INVALID_ARG, "NEST_F_VEC_QUAD needs NEST_F_VEC128");
    if (K <= 0) K = 1;
    const int32_t S = d->simdlen;
    const bool smem_mode = d->mode == NEST_MODE_GENERIC_SMEM && S > 1;
    Plan q;
    q.block = T;
    q.simdlen = S;
    q.mode = S == 1 ? NEST_MODE_SPMD : d->mode;
    q.reduce = d->reduce;
    q.groups = T / S;
    q.slot_bytes = (sharing / q.groups) & ~7;           // split evenly, 8-B aligned (R8)
    q.payload_bytes = payload;
    q.fallback = smem_mode && payload > q.slot_bytes;
    q.unroll = U;
    q.smem_bytes = smem_mode ? sharing : 0;             // SPMD needs no sharing space
    q.flags = d->flags;
    q.outer = outer;
    // one batch of U steps spans ceil(U/K) outer iterations of a group
    const int64_t per_group = (U + K - 1) / K;
    const int64_t denom = (int64_t)q.groups * per_group;
    int64_t needed = (outer + denom - 1) / denom;
    if (d->x_halo > 0) {
        q.x_halo = d->x_halo;   // the x ring: sized by plan_spmv_ring (needs nnz)
        q.grid = d->num_teams;
    } else if (d->num_teams > 0) {
        q.grid = d->num_teams;
    } else if ((d->flags & (NEST_F_PERSISTENT_GRID | NEST_F_BLOCKED)) || q.fallback) {
        int64_t resident = 0;
        nest_status s = resident_blocks(T, q.smem_bytes, &resident);
        if (s != NEST_OK) return s;
        q.grid = (int32_t)(needed < resident ? needed : resident);
    } else {
        if (needed > INT32_MAX) needed = INT32_MAX;
        q.grid = (int32_t)needed;
    }
    if ((d->flags & NEST_F_BLOCKED) && q.grid > 0) {
        // team chunks: the requested size, or one contiguous range per team;
        // rounded up to a multiple of G so every group starts inside its chunk
        int64_t c = d->team_chunk > 0 ? d->team_chunk : (outer + q.grid - 1) / q.grid;
        if (c < 1) c = 1;
        q.chunk = (c + q.groups - 1) / q.groups * q.groups;
    }
    *p = q;
    return NEST_OK;
}

nest_status make_plan(const nest_desc* d, int64_t outer, int32_t K, PayloadFn payload_of, Plan* p,
                      bool spmv_window) {
    int32_t T = 0, sharing = 0, U = 1;   // set by validate_desc on success
    nest_status s = validate_desc(d, &T, &sharing, &U);
    if (s != NEST_OK) return s;
    return plan_core(d, outer, K, T, sharing, U, payload_of(U), p, spmv_window);
}

nest_status make_plan_fixed(const nest_desc* d, int64_t outer, int32_t K, int32_t payload, Plan* p,
                            bool spmv_window) {
    int32_t T = 0, sharing = 0, U = 1;   // set by validate_desc on success
    nest_status s = validate_desc(d, &T, &sharing, &U);
    if (s != NEST_OK) return s;
    if (payload < 0) return fail(NEST_ERR_INVALID_ARG, "payload_bytes %d < 0", payload);
    return plan_core(d, outer, K, T, sharing, U, payload, p, spmv_window);
}

// ------------------------------------------------ sharing-space fallback
struct Scratch {
    unsigned char* ptr = nullptr;
    size_t bytes = 0;
};
// One buffer per (device, stream): launches on different streams may run
// concurrently and must not share slots; launches on one stream are ordered.
static std::mutex g_scratch_mu;
static std::map<std::pair<int, void*>, Scratch> g_scratch;

nest_status fallback_scratch(size_t bytes, unsigned char** out, void* stream) {
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return cuda_fail(e, "cudaGetDevice");
    std::lock_guard<std::mutex> lk(g_scratch_mu);
    Scratch& s = g_scratch[std::make_pair(dev, stream)];
    if (s.bytes < bytes) {
        if (s.ptr) {
            e = cudaFree(s.ptr);   // synchronises: only on growth, never in steady state
            s.ptr = nullptr;
            s.bytes = 0;
            if (e != cudaSuccess) return cuda_fail(e, "cudaFree(fallback)");
        }
        e = cudaMalloc(&s.ptr, bytes);
        if (e != cudaSuccess) {
            cudaGetLastError();
            return fail(NEST_ERR_NO_MEMORY, "fallback scratch of %zu bytes", bytes);
        }
        s.bytes = bytes;
    }
    *out = s.ptr;
    return NEST_OK;
}

nest_status prepare_fallback(const Plan& p, unsigned char** fb, void* stream) {
    *fb = nullptr;
    if (!p.fallback) return NEST_OK;
    const size_t bytes = (size_t)p.grid * (size_t)p.groups * (size_t)p.payload_bytes;
    return fallback_scratch(bytes, fb, stream);
}

// ------------------------------------------- NEST_F_X_L2_PERSIST (x in L2)
// Set-aside the library asks for: half of L2 (63 MB on B200), capped by the
// device's maximum persisting size (79 MB).  Measured on cfg2 / G100 (x = 80 /
// 100 MB, profiles/r02s3_x_l2_persist.md): 63-71 MB beat 47 MB and the 79 MB
// maximum (which leaves too little L2 for the streamed CSR lines).
static std::mutex g_persist_mu;
static std::map<int, size_t> g_persist_orig;       // device -> the limit before this library raised it
static std::atomic<bool> g_persist_used{false};    // a persisting launch happened (nest_util_l2_flush resets)

nest_status x_persist_window(Plan* p, const double* x, int64_t ncols, bool apply) {
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return cuda_fail(e, "cudaGetDevice");
    int max_persist = 0, l2 = 0, max_win = 0;
    if ((e = cudaDeviceGetAttribute(&max_persist, cudaDevAttrMaxPersistingL2CacheSize, dev)) != cudaSuccess ||
        (e = cudaDeviceGetAttribute(&l2, cudaDevAttrL2CacheSize, dev)) != cudaSuccess ||
        (e = cudaDeviceGetAttribute(&max_win, cudaDevAttrMaxAccessPolicyWindowSize, dev)) != cudaSuccess)
        return cuda_fail(e, "cudaDeviceGetAttribute(L2 persistence)");
    if (max_persist <= 0 || max_win <= 0)
        return fail(NEST_ERR_UNSUPPORTED, "NEST_F_X_L2_PERSIST: the device has no persisting L2");
    size_t cur = 0;
    if ((e = cudaDeviceGetLimit(&cur, cudaLimitPersistingL2CacheSize)) != cudaSuccess)
        return cuda_fail(e, "cudaDeviceGetLimit(persisting L2)");
    const int64_t want = std::min<int64_t>(max_persist, (int64_t)l2 / 2);
    p->l2_win_bytes = std::min<int64_t>(ncols * 8, max_win);
    p->l2_setaside = std::max<int64_t>((int64_t)cur, want);
    if (!apply) return NEST_OK;
    if ((int64_t)cur < want) {
        std::lock_guard<std::mutex> lk(g_persist_mu);
        g_persist_orig.emplace(dev, cur);   // first raise only: nest_shutdown restores it
        if ((e = cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, (size_t)want)) != cudaSuccess ||
            (e = cudaDeviceGetLimit(&cur, cudaLimitPersistingL2CacheSize)) != cudaSuccess)   // granularity
            return cuda_fail(e, "cudaDeviceSetLimit(persisting L2)");
        p->l2_setaside = (int64_t)cur;
    }
    g_persist_used = true;
    p->l2_win = x;
    return NEST_OK;
}

// --------------------------------------------------------- device utilities
__global__ void csr_validate_kernel(int64_t nrows, int64_t ncols, int64_t nnz,
                                    const int64_t* __restrict__ rowptr,
                                    const int32_t* __restrict__ col, int32_t* __restrict__ bad) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    const int64_t t0 = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (t0 == 0 && (rowptr[0] != 0 || rowptr[nrows] != nnz)) atomicOr(bad, 1);
    for (int64_t i = t0; i < nrows; i += stride)
        if (rowptr[i + 1] < rowptr[i]) atomicOr(bad, 2);
    for (int64_t k = t0; k < nnz; k += stride)
        if (col[k] < 0 || (int64_t)col[k] >= ncols) atomicOr(bad, 4);
}

__global__ void l2_flush_kernel(uint4* __restrict__ buf, size_t n16, uint32_t salt) {
    const size_t stride = (size_t)gridDim.x * blockDim.x;
    for (size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x; i < n16; i += stride)
        buf[i] = make_uint4(salt, (uint32_t)i, salt ^ 0x9e3779b9u, (uint32_t)(i >> 32));
}

// Second flush phase: read the first half of the buffer (written earliest, so
// no longer resident) -- L2 ends up holding only clean lines, and the dirty
// lines of the write phase are written back here rather than inside the next
// (timed) kernel.
__global__ void l2_clean_kernel(const uint4* __restrict__ buf, size_t n16, uint32_t* sink) {
    const size_t stride = (size_t)gridDim.x * blockDim.x;
    uint32_t acc = 0;
    for (size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x; i < n16; i += stride) acc ^= __ldcg(buf + i).y;
    if (acc == 0x9e3779b9u && sink) *sink = acc;
}

}  // namespace nest

using namespace nest;

static cudaStream_t as_stream(void* s) { return reinterpret_cast<cudaStream_t>(s); }

NEST_API uint32_t nest_abi_version(void) { return NEST_ABI_VERSION; }

NEST_API const char* nest_status_str(nest_status s) {
    switch (s) {
        case NEST_OK: return "NEST_OK";
        case NEST_ERR_INVALID_ARG: return "NEST_ERR_INVALID_ARG";
        case NEST_ERR_UNSUPPORTED: return "NEST_ERR_UNSUPPORTED";
        case NEST_ERR_CUDA: return "NEST_ERR_CUDA";
        case NEST_ERR_NCCL: return "NEST_ERR_NCCL";
        case NEST_ERR_NO_MEMORY: return "NEST_ERR_NO_MEMORY";
    }
    return "NEST_ERR_UNKNOWN";
}

NEST_API const char* nest_last_error(void) { return nest::g_err; }

static void fill_plan_info(const Plan& p, int32_t kernel, int32_t index_bits, nest_plan_info* out) {
    out->grid = p.grid;
    out->block = p.block;
    out->groups_per_team = p.groups;
    out->slot_bytes = p.slot_bytes;
    out->payload_bytes = p.payload_bytes;
    out->uses_global_fallback = p.fallback;
    out->outer_unroll = p.unroll;
    out->smem_bytes = p.smem_bytes;
    out->kernel = kernel;
    out->index_bits = index_bits;
    out->ring_segments = p.ring_nseg;
    out->ring_row_slots = p.ring_nrp;
    out->chunk = (p.flags & NEST_F_BLOCKED) || p.x_halo > 0 ? p.chunk : 0;
    out->l2_window_bytes = p.l2_win_bytes;
    out->l2_setaside_bytes = p.l2_setaside;
}

NEST_API nest_status nest_plan(const nest_desc* desc, int64_t outer_iters, int32_t payload_bytes,
                               nest_plan_info* out) {
    if (!out) return fail(NEST_ERR_INVALID_ARG, "out is NULL");
    Plan p;
    nest_status s = make_plan_fixed(desc, outer_iters, 1, payload_bytes, &p, false);
    if (s != NEST_OK) return s;
    fill_plan_info(p, NEST_KERNEL_NEST, 64, out);
    return NEST_OK;
}

// The plan the CSR SpMV launches for this matrix shape (a1 for a8): the
// descriptor's geometry, the variant's own sizing (x ring, teams-generic), and
// the generic payload of the body that actually runs -- so the reported
// fallback is the kernel's (engine.cuh group_slot follows the plan).
static nest_status spmv_plan(const nest_desc* desc, int64_t nrows, int64_t ncols, int64_t nnz, Plan* p,
                             int32_t* kernel, int32_t* index_bits) {
    if (nrows < 0 || ncols < 0 || nnz < 0)
        return fail(NEST_ERR_INVALID_ARG, "negative extent (nrows %lld, ncols %lld, nnz %lld)",
                    (long long)nrows, (long long)ncols, (long long)nnz);
    if (ncols > INT32_MAX) return fail(NEST_ERR_INVALID_ARG, "ncols exceeds int32 column indices");
    nest_status s = make_plan(desc, nrows, 1, spmv_payload, p, true);
    if (s != NEST_OK) return s;
    if (desc->mode == NEST_MODE_TEAMS_GENERIC) {
        if ((p->flags & (NEST_F_VEC128 | NEST_F_BLOCKED | NEST_F_X_L2_PERSIST)) || p->x_halo > 0)
            return fail(NEST_ERR_UNSUPPORTED, "NEST_MODE_TEAMS_GENERIC takes no SpMV variant flags");
        if (desc->num_teams <= 0) {
            int64_t resident = 0;
            if ((s = resident_blocks(p->block + 32, 0, &resident)) != NEST_OK) return s;
            p->grid = (int32_t)std::max<int64_t>(1, std::min(nrows, resident));
        }
        *kernel = NEST_KERNEL_TEAMS_GENERIC;
        *index_bits = 64;
        return NEST_OK;
    }
    if (p->x_halo > 0) {
        *kernel = NEST_KERNEL_XRING;
        *index_bits = nnz < ((int64_t)1 << 31) - 8 && nrows < ((int64_t)1 << 31) - 8 ? 32 : 64;
        if ((s = plan_spmv_ring(p, nrows, nnz, desc->num_teams, desc->teams_per_sm)) != NEST_OK) return s;
        if ((p->flags & NEST_F_X_L2_PERSIST) && (s = x_persist_window(p, nullptr, ncols, false)) != NEST_OK)
            return s;
        return NEST_OK;
    }
    *kernel = NEST_KERNEL_NEST;
    const int32_t payload = spmv_body_payload(*p, nnz);
    if (payload != p->payload_bytes && (s = make_plan_fixed(desc, nrows, 1, payload, p, true)) != NEST_OK) return s;
    *index_bits = spmv_index32(*p, nnz) ? 32 : 64;
    if ((p->flags & NEST_F_X_L2_PERSIST) && (s = x_persist_window(p, nullptr, ncols, false)) != NEST_OK) return s;
    return NEST_OK;
}

NEST_API nest_status nest_spmv_plan(const nest_desc* desc, int64_t nrows, int64_t ncols, int64_t nnz,
                                    nest_plan_info* out) {
    if (!out) return fail(NEST_ERR_INVALID_ARG, "out is NULL");
    Plan p;
    int32_t kernel = 0, bits = 0;
    nest_status s = spmv_plan(desc, nrows, ncols, nnz, &p, &kernel, &bits);
    if (s != NEST_OK) return s;
    fill_plan_info(p, kernel, bits, out);
    return NEST_OK;
}

// Launch a planned SpMV on rows [0, nrows) of the given arrays (rowptr entries
// are absolute offsets into colind/val).
static nest_status spmv_launch(const Plan& p, int32_t kernel, int64_t nrows, int64_t ncols, int64_t nnz,
                               const int64_t* rowptr, const int32_t* colind, const double* val, const double* x,
                               double* y, unsigned char* fb, cudaStream_t st) {
    if (kernel == NEST_KERNEL_TEAMS_GENERIC) return launch_spmv_teams_generic(p, nrows, rowptr, colind, val, x, y, st);
    Plan q = p;
    if ((q.flags & NEST_F_X_L2_PERSIST) && ncols > 0) {   // the x window of this launch
        nest_status s = x_persist_window(&q, x, ncols, true);
        if (s != NEST_OK) return s;
    }
    if (kernel == NEST_KERNEL_XRING) return launch_spmv_ring(q, nrows, ncols, nnz, rowptr, colind, val, x, y, fb, st);
    return launch_spmv(q, (q.flags & NEST_F_STREAM_HINTS) != 0, nrows, rowptr, colind, val, x, y, fb, st, nnz);
}

// Alignment the variants need (checked before any launch).
static nest_status spmv_alignment(const Plan& p, int32_t kernel, const int64_t* rowptr, const int32_t* colind,
                                  const double* val, const double* x) {
    if (reinterpret_cast<uintptr_t>(rowptr) & 7) return fail(NEST_ERR_INVALID_ARG, "rowptr must be 8-byte aligned");
    const bool quad = (p.flags & NEST_F_VEC_QUAD) != 0;
    if ((p.flags & NEST_F_VEC128) &&
        ((reinterpret_cast<uintptr_t>(val) & (quad ? 31 : 15)) ||
         (reinterpret_cast<uintptr_t>(colind) & (quad ? 15 : 7))))
        return fail(NEST_ERR_UNSUPPORTED, "NEST_F_VEC128 needs %d-byte aligned val and %d-byte aligned colind",
                    quad ? 32 : 16, quad ? 16 : 8);
    if (kernel == NEST_KERNEL_XRING && (reinterpret_cast<uintptr_t>(x) & 15))
        return fail(NEST_ERR_UNSUPPORTED, "x_halo needs 16-byte aligned x (bulk copies of x segments)");
    return NEST_OK;
}

NEST_API nest_status nest_spmv_csr_f64(const nest_desc* desc, int64_t nrows, int64_t ncols,
                                       int64_t nnz, const int64_t* rowptr, const int32_t* colind,
                                       const double* val, const double* x, double* y,
                                       void* stream) {
    Plan p;
    int32_t kernel = 0, bits = 0;
    nest_status s = spmv_plan(desc, nrows, ncols, nnz, &p, &kernel, &bits);
    if (s != NEST_OK) return s;
    if (nrows == 0) return NEST_OK;
    if (!rowptr || !y) return fail(NEST_ERR_INVALID_ARG, "rowptr/y is NULL");
    if (nnz > 0 && (!colind || !val || !x)) return fail(NEST_ERR_INVALID_ARG, "colind/val/x is NULL");
    if ((s = spmv_alignment(p, kernel, rowptr, colind, val, x)) != NEST_OK) return s;
    unsigned char* fb = nullptr;
    if ((s = prepare_fallback(p, &fb, stream)) != NEST_OK) return s;
    return spmv_launch(p, kernel, nrows, ncols, nnz, rowptr, colind, val, x, y, fb, as_stream(stream));
}

static size_t align256(size_t b) { return (b + 255) & ~(size_t)255; }

NEST_API size_t nest_spmv_hostio_workspace_bytes(int64_t nrows, int64_t ncols, int64_t nnz) {
    if (nrows < 0 || ncols < 0 || nnz < 0) return 0;
    return align256((size_t)(nrows + 1) * 8) + align256((size_t)nnz * 4) + align256((size_t)nnz * 8) +
           align256((size_t)ncols * 8) + align256((size_t)nrows * 8);
}

// ---------------------------------------- a8 end to end: chunked pipeline
// The host->device copy of the matrix is the bound of the end-to-end call
// (PCIe, ~50 GB/s against ~4 TB/s for the SpMV itself).  Rows are split into
// chunks of about kHostioChunkNnz nonzeros: x first, then per chunk its rowptr
// slice, colind and val on an H2D stream; chunk c's SpMV runs on the caller's
// stream once the copies it reads have landed, and its y rows go back on a
// D2H stream while later chunks are still crossing the bus (the two PCIe
// directions are independent).  Same kernel, same per-row arithmetic as the
// single-shot path: results are bit-identical.
static constexpr int64_t kHostioChunkNnz = int64_t(8) << 20;
static constexpr int kHostioMaxChunks = 32;

static int hostio_chunks(int64_t nnz) {
    static const int forced = [] {
        const char* e = std::getenv("NEST_HOSTIO_CHUNKS");   // A/B experiments (1 = single shot)
        return e ? std::atoi(e) : 0;
    }();
    int64_t k = forced > 0 ? forced : (nnz + kHostioChunkNnz - 1) / kHostioChunkNnz;
    if (k < 1) k = 1;
    if (k > kHostioMaxChunks) k = kHostioMaxChunks;
    return (int)k;
}

struct HostioStreams {
    cudaStream_t h2d = nullptr, d2h = nullptr;
    cudaEvent_t ev[2 * kHostioMaxChunks + 2] = {};
};
static std::mutex g_hostio_mu;
static std::map<int, HostioStreams> g_hostio;

static void hostio_destroy(HostioStreams& h) {
    for (cudaEvent_t& ev : h.ev)
        if (ev) cudaEventDestroy(ev), ev = nullptr;
    if (h.h2d) cudaStreamDestroy(h.h2d), h.h2d = nullptr;
    if (h.d2h) cudaStreamDestroy(h.d2h), h.d2h = nullptr;
}

// caller holds g_hostio_mu
static nest_status hostio_streams(HostioStreams** out) {
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return cuda_fail(e, "cudaGetDevice");
    auto it = g_hostio.find(dev);
    if (it == g_hostio.end()) {
        HostioStreams h;
        if ((e = cudaStreamCreateWithFlags(&h.h2d, cudaStreamNonBlocking)) == cudaSuccess)
            e = cudaStreamCreateWithFlags(&h.d2h, cudaStreamNonBlocking);
        for (cudaEvent_t& ev : h.ev)
            if (e == cudaSuccess) e = cudaEventCreateWithFlags(&ev, cudaEventDisableTiming);
        if (e != cudaSuccess) {
            hostio_destroy(h);
            return cuda_fail(e, "hostio streams/events");
        }
        it = g_hostio.emplace(dev, h).first;
    }
    *out = &it->second;
    return NEST_OK;
}

static nest_status spmv_hostio_pipelined(const nest_desc* desc, int nchunks, int64_t nrows,
                                         int64_t ncols, int64_t nnz, const int64_t* h_rowptr,
                                         const int32_t* h_colind, const double* h_val, const double* h_x,
                                         double* h_y, int64_t* d_rowptr, int32_t* d_col, double* d_val,
                                         double* d_x, double* d_y, cudaStream_t st) {
    // chunk c = rows [r[c], r[c+1]) with nonzeros [h_rowptr[r[c]], h_rowptr[r[c+1]]);
    // boundaries at the rows where the nonzero count crosses c * nnz / nchunks
    int64_t r[kHostioMaxChunks + 1];
    r[0] = 0;
    for (int c = 1; c < nchunks; ++c) {
        const int64_t target = h_rowptr[0] + (nnz * c) / nchunks;
        int64_t lo = r[c - 1], hi = nrows;   // first row whose start >= target
        while (lo < hi) {
            const int64_t mid = lo + (hi - lo) / 2;
            if (h_rowptr[mid] < target) lo = mid + 1; else hi = mid;
        }
        r[c] = lo;
    }
    r[nchunks] = nrows;
    std::lock_guard<std::mutex> lk(g_hostio_mu);
    HostioStreams* h = nullptr;
    nest_status s = hostio_streams(&h);
    if (s != NEST_OK) return s;
    cudaEvent_t ev_start = h->ev[0], ev_done = h->ev[1];
    cudaEvent_t* ev_in = h->ev + 2;
    cudaEvent_t* ev_k = h->ev + 2 + kHostioMaxChunks;
    cudaError_t e;
    // everything earlier on the caller's stream (a previous call reading this workspace) first
    if ((e = cudaEventRecord(ev_start, st)) || (e = cudaStreamWaitEvent(h->h2d, ev_start, 0)) ||
        (e = cudaStreamWaitEvent(h->d2h, ev_start, 0)))
        return cuda_fail(e, "hostio start");
    if (ncols && (e = cudaMemcpyAsync(d_x, h_x, (size_t)ncols * 8, cudaMemcpyHostToDevice, h->h2d)))
        return cuda_fail(e, "host->device copy (x)");
    int64_t zb[kHostioMaxChunks + 1];   // nonzero boundaries, relative to the arrays
    for (int c = 0; c <= nchunks; ++c) zb[c] = h_rowptr[r[c]];
    for (int c = 0; c < nchunks; ++c) {
        // rowptr entries [r[c] + (c > 0), r[c+1]]: disjoint slices, chunk c's bounds all covered by copies <= c
        const int64_t p0r = r[c] + (c > 0), p1r = r[c + 1];
        if (p1r >= p0r && (e = cudaMemcpyAsync(d_rowptr + p0r, h_rowptr + p0r, (size_t)(p1r - p0r + 1) * 8,
                                               cudaMemcpyHostToDevice, h->h2d)))
            return cuda_fail(e, "host->device copy (rowptr)");
        const int64_t z0 = zb[c], z1 = zb[c + 1];
        if (z1 > z0 &&
            ((e = cudaMemcpyAsync(d_col + z0, h_colind + z0, (size_t)(z1 - z0) * 4, cudaMemcpyHostToDevice, h->h2d)) ||
             (e = cudaMemcpyAsync(d_val + z0, h_val + z0, (size_t)(z1 - z0) * 8, cudaMemcpyHostToDevice, h->h2d))))
            return cuda_fail(e, "host->device copy (colind/val)");
        if ((e = cudaEventRecord(ev_in[c], h->h2d))) return cuda_fail(e, "hostio event");
    }
    for (int c = 0; c < nchunks; ++c) {
        const int64_t rows = r[c + 1] - r[c];
        // 128-bit tuples read up to 3 entries past the chunk's last nonzero (unused):
        // wait for the copy that holds the last entry the chunk can touch
        const int64_t last = std::min<int64_t>(nnz, (zb[c + 1] + 3) & ~(int64_t)3) - 1;
        int j = c;
        while (j + 1 < nchunks && zb[j + 1] <= last) ++j;
        if ((e = cudaStreamWaitEvent(st, ev_in[j], 0))) return cuda_fail(e, "hostio wait");
        if (rows > 0) {
            Plan p;
            int32_t kernel = 0, bits = 0;
            unsigned char* fb = nullptr;
            if ((s = spmv_plan(desc, rows, ncols, nnz, &p, &kernel, &bits)) != NEST_OK ||
                (s = prepare_fallback(p, &fb, st)) != NEST_OK ||
                (s = spmv_launch(p, kernel, rows, ncols, nnz, d_rowptr + r[c], d_col, d_val, d_x, d_y + r[c], fb, st)) !=
                    NEST_OK)
                return s;
        }
        if ((e = cudaEventRecord(ev_k[c], st)) || (e = cudaStreamWaitEvent(h->d2h, ev_k[c], 0)))
            return cuda_fail(e, "hostio event");
        if (rows > 0 && (e = cudaMemcpyAsync(h_y + r[c], d_y + r[c], (size_t)rows * 8, cudaMemcpyDeviceToHost, h->d2h)))
            return cuda_fail(e, "device->host copy");
    }
    // the caller's stream completes only after the last y rows are on the host
    if ((e = cudaEventRecord(ev_done, h->d2h)) || (e = cudaStreamWaitEvent(st, ev_done, 0)))
        return cuda_fail(e, "hostio done");
    return NEST_OK;
}

NEST_API nest_status nest_spmv_csr_f64_hostio(const nest_desc* desc, int64_t nrows, int64_t ncols,
                                              int64_t nnz, const int64_t* h_rowptr,
                                              const int32_t* h_colind, const double* h_val,
                                              const double* h_x, double* h_y, void* d_workspace,
                                              size_t workspace_bytes, void* stream) {
    Plan p;
    int32_t kernel = 0, bits = 0;
    nest_status s = spmv_plan(desc, nrows, ncols, nnz, &p, &kernel, &bits);
    if (s != NEST_OK) return s;
    if (nrows == 0) return NEST_OK;
    if (kernel == NEST_KERNEL_TEAMS_GENERIC)
        return fail(NEST_ERR_UNSUPPORTED, "nest_spmv_csr_f64_hostio: use nest_spmv_csr_f64 for NEST_MODE_TEAMS_GENERIC");
    const size_t need = nest_spmv_hostio_workspace_bytes(nrows, ncols, nnz);
    if (!d_workspace || workspace_bytes < need)
        return fail(NEST_ERR_INVALID_ARG, "workspace %zu bytes < %zu", workspace_bytes, need);
    if (reinterpret_cast<uintptr_t>(d_workspace) & 255)
        return fail(NEST_ERR_INVALID_ARG, "workspace must be 256-byte aligned");
    if (!h_rowptr || !h_y || (nnz > 0 && (!h_colind || !h_val || !h_x)))
        return fail(NEST_ERR_INVALID_ARG, "host buffer is NULL");
    if (h_rowptr[0] != 0 || h_rowptr[nrows] != nnz)
        return fail(NEST_ERR_INVALID_ARG, "rowptr must run from 0 to nnz (%lld .. %lld, nnz %lld)",
                    (long long)h_rowptr[0], (long long)h_rowptr[nrows], (long long)nnz);
    unsigned char* w = static_cast<unsigned char*>(d_workspace);
    int64_t* d_rowptr = reinterpret_cast<int64_t*>(w);
    w += align256((size_t)(nrows + 1) * 8);
    int32_t* d_col = reinterpret_cast<int32_t*>(w);
    w += align256((size_t)nnz * 4);
    double* d_val = reinterpret_cast<double*>(w);
    w += align256((size_t)nnz * 8);
    double* d_x = reinterpret_cast<double*>(w);
    w += align256((size_t)ncols * 8);
    double* d_y = reinterpret_cast<double*>(w);
    cudaStream_t st = as_stream(stream);
    const int nchunks = hostio_chunks(nnz);
    if (nchunks > 1)
        return spmv_hostio_pipelined(desc, nchunks, nrows, ncols, nnz, h_rowptr, h_colind, h_val, h_x, h_y,
                                     d_rowptr, d_col, d_val, d_x, d_y, st);
    unsigned char* fb = nullptr;
    if ((s = prepare_fallback(p, &fb, stream)) != NEST_OK) return s;
    cudaError_t e;
    if ((e = cudaMemcpyAsync(d_rowptr, h_rowptr, (size_t)(nrows + 1) * 8, cudaMemcpyHostToDevice, st)) ||
        (nnz && (e = cudaMemcpyAsync(d_col, h_colind, (size_t)nnz * 4, cudaMemcpyHostToDevice, st))) ||
        (nnz && (e = cudaMemcpyAsync(d_val, h_val, (size_t)nnz * 8, cudaMemcpyHostToDevice, st))) ||
        (ncols && (e = cudaMemcpyAsync(d_x, h_x, (size_t)ncols * 8, cudaMemcpyHostToDevice, st))))
        return cuda_fail(e, "host->device copy");
    if ((s = spmv_launch(p, kernel, nrows, ncols, nnz, d_rowptr, d_col, d_val, d_x, d_y, fb, st)) != NEST_OK) return s;
    if ((e = cudaMemcpyAsync(h_y, d_y, (size_t)nrows * 8, cudaMemcpyDeviceToHost, st)))
        return cuda_fail(e, "device->host copy");
    return NEST_OK;
}

NEST_API nest_status nest_batched_matvec_f32(const nest_desc* desc, int64_t batch, int32_t m,
                                             int32_t n, const float* A, const float* x, float* y,
                                             void* stream) {
    if (batch < 0 || m < 0 || n < 0) return fail(NEST_ERR_INVALID_ARG, "negative extent");
    Plan p;
    nest_status s = make_plan(desc, batch, m, batched_payload, &p);
    if (s != NEST_OK) return s;
    if (batch == 0 || m == 0) return NEST_OK;
    if (!y || (n > 0 && (!A || !x))) return fail(NEST_ERR_INVALID_ARG, "A/x/y is NULL");
    if ((p.flags & NEST_F_VEC128) &&
        (n % 4 || (reinterpret_cast<uintptr_t>(A) & 15) || (reinterpret_cast<uintptr_t>(x) & 15)))
        return fail(NEST_ERR_UNSUPPORTED, "NEST_F_VEC128 (batched) needs n %% 4 == 0 and 16-byte aligned A and x");
    unsigned char* fb = nullptr;
    if ((s = prepare_fallback(p, &fb, stream)) != NEST_OK) return s;
    return launch_batched(p, batch, m, n, A, x, y, fb, as_stream(stream));
}

NEST_API nest_status nest_nested_stencil_f64(const nest_desc* desc, int64_t nouter, int32_t L,
                                             const double* in, const double* coef,
                                             const double* w, double* out,
                                             unsigned long long* visits, void* stream) {
    if (nouter < 0 || L < 0) return fail(NEST_ERR_INVALID_ARG, "negative extent");
    Plan p;
    nest_status s = make_plan(desc, nouter, 1, stencil_payload, &p);
    if (s != NEST_OK) return s;
    if (nouter == 0) return NEST_OK;
    if (!w || !out || (L > 0 && (!in || !coef))) return fail(NEST_ERR_INVALID_ARG, "in/coef/w/out is NULL");
    if ((p.flags & NEST_F_VEC128) &&
        ((L & 1) || (reinterpret_cast<uintptr_t>(in) & 15) || (reinterpret_cast<uintptr_t>(coef) & 15)))
        return fail(NEST_ERR_UNSUPPORTED, "NEST_F_VEC128 (stencil) needs an even L and 16-byte aligned in and coef");
    unsigned char* fb = nullptr;
    if ((s = prepare_fallback(p, &fb, stream)) != NEST_OK) return s;
    return launch_stencil(p, nouter, L, in, coef, w, out, visits, fb, as_stream(stream));
}

NEST_API nest_status nest_laplace3d_f64(const nest_desc* desc, int64_t nz, int64_t ny, int64_t nx,
                                        double alpha, const double* u, double* out, void* stream) {
    if (nz < 0 || ny < 0 || nx < 0) return fail(NEST_ERR_INVALID_ARG, "negative extent");
    const int64_t lines = (nz > 2 && ny > 2) ? (nz - 2) * (ny - 2) : 0;
    Plan p;
    nest_status s = make_plan(desc, lines, 1, laplace_payload, &p);
    if (s != NEST_OK) return s;
    if (lines == 0 || nx <= 2) return NEST_OK;
    if (!u || !out) return fail(NEST_ERR_INVALID_ARG, "u/out is NULL");
    if (u == out) return fail(NEST_ERR_INVALID_ARG, "u and out must not alias (Jacobi step)");
    if ((p.flags & NEST_F_VEC128) &&
        ((nx & 1) || (reinterpret_cast<uintptr_t>(u) & 15) || (reinterpret_cast<uintptr_t>(out) & 15)))
        return fail(NEST_ERR_UNSUPPORTED, "NEST_F_VEC128 (laplace3d) needs an even nx and 16-byte aligned u and out");
    unsigned char* fb = nullptr;
    if ((s = prepare_fallback(p, &fb, stream)) != NEST_OK) return s;
    return launch_laplace(p, nz, ny, nx, alpha, u, out, fb, as_stream(stream));
}

NEST_API nest_status nest_probe_mapping(const nest_desc* desc, int32_t* out_map, int64_t trip,
                                        int32_t* hits, int32_t* owner, double* totals,
                                        void* stream) {
    if (!desc || desc->num_teams <= 0) return fail(NEST_ERR_INVALID_ARG, "probe needs num_teams > 0");
    if (trip < 0) return fail(NEST_ERR_INVALID_ARG, "trip < 0");
    if (!valid_simdlen(desc->simdlen)) return fail(NEST_ERR_INVALID_ARG, "simdlen %d", desc->simdlen);
    const int32_t T = desc->threads_per_team ? desc->threads_per_team : kDefaultThreads;
    const int64_t outer = (int64_t)desc->num_teams * (T / desc->simdlen);
    Plan p;
    nest_status s = make_plan(desc, outer, 1, probe_payload, &p);
    if (s != NEST_OK) return s;
    unsigned char* fb = nullptr;
    if ((s = prepare_fallback(p, &fb, stream)) != NEST_OK) return s;
    return launch_probe(p, out_map, trip, hits, owner, totals, fb, as_stream(stream));
}

NEST_API nest_status nest_csr_validate(int64_t nrows, int64_t ncols, int64_t nnz,
                                       const int64_t* rowptr, const int32_t* colind, int32_t* d_bad,
                                       void* stream) {
    if (nrows < 0 || ncols < 0 || nnz < 0 || !rowptr || !d_bad || (nnz > 0 && !colind))
        return fail(NEST_ERR_INVALID_ARG, "bad arguments");
    csr_validate_kernel<<<1184, 256, 0, as_stream(stream)>>>(nrows, ncols, nnz, rowptr, colind, d_bad);
    const cudaError_t e = cudaGetLastError();
    return e == cudaSuccess ? NEST_OK : cuda_fail(e, "csr_validate launch");
}

NEST_API nest_status nest_util_l2_flush(void* buf, size_t bytes, void* stream) {
    if (!buf && bytes) return fail(NEST_ERR_INVALID_ARG, "buf is NULL");
    static uint32_t salt = 1;
    const size_t n16 = bytes / 16;
    if (n16 == 0) return NEST_OK;
    if (g_persist_used) {
        // persisting lines survive a plain flush: return them to normal first,
        // after the work queued on `stream` (a persisting launch) has finished
        cudaError_t e = cudaStreamSynchronize(as_stream(stream));
        if (e == cudaSuccess) e = cudaCtxResetPersistingL2Cache();
        if (e != cudaSuccess) return cuda_fail(e, "reset persisting L2 lines");
    }
    l2_flush_kernel<<<1184, 512, 0, as_stream(stream)>>>(static_cast<uint4*>(buf), n16, salt++);
    l2_clean_kernel<<<1184, 512, 0, as_stream(stream)>>>(static_cast<const uint4*>(buf), n16 / 2, nullptr);
    const cudaError_t e = cudaGetLastError();
    return e == cudaSuccess ? NEST_OK : cuda_fail(e, "l2_flush launch");
}

NEST_API nest_status nest_shutdown(void) {
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return cuda_fail(e, "cudaGetDevice");
    std::lock_guard<std::mutex> lk(g_scratch_mu);
    cudaError_t first = cudaSuccess;
    for (auto it = g_scratch.begin(); it != g_scratch.end();) {
        if (it->first.first == dev) {
            if (it->second.ptr && (e = cudaFree(it->second.ptr)) != cudaSuccess && first == cudaSuccess) first = e;
            it = g_scratch.erase(it);
        } else {
            ++it;
        }
    }
    if (first != cudaSuccess) return cuda_fail(first, "cudaFree(fallback)");
    std::lock_guard<std::mutex> lk2(g_hostio_mu);
    auto h = g_hostio.find(dev);
    if (h != g_hostio.end()) {
        hostio_destroy(h->second);
        g_hostio.erase(h);
    }
    // NEST_F_X_L2_PERSIST: persisting lines back to normal, the set-aside back to what it was
    std::lock_guard<std::mutex> lk3(g_persist_mu);
    auto q = g_persist_orig.find(dev);
    if (q != g_persist_orig.end()) {
        if ((e = cudaCtxResetPersistingL2Cache()) != cudaSuccess ||
            (e = cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, q->second)) != cudaSuccess)
            return cuda_fail(e, "restore the persisting-L2 limit");
        g_persist_orig.erase(q);
    }
    return NEST_OK;
}
