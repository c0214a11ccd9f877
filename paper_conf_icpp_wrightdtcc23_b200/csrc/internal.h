// internal.h -- host-side declarations shared by the translation units of
// libnest.so (never exported; the ABI is include/nest.h).
#pragma once

#include <cuda_runtime.h>

#include <cstdint>

#include "nest.h"

#define NEST_API extern "C" __attribute__((visibility("default")))

namespace nest {

// a1: the resolved launch plan.
struct Plan {
    int32_t grid = 0;
    int32_t block = 0;
    int32_t simdlen = 0;
    int32_t mode = 0;      // effective mode (S == 1 runs SPMD: PAPER.md:691-693)
    int32_t reduce = 0;
    int32_t groups = 0;    // G
    int32_t slot_bytes = 0;
    int32_t payload_bytes = 0;
    int32_t fallback = 0;
    int32_t unroll = 1;    // U
    int32_t smem_bytes = 0;
    uint32_t flags = 0;
    int64_t outer = 0;
    int64_t chunk = 0;     // NEST_F_BLOCKED: outer iterations per team chunk (a multiple of G)
    int32_t x_halo = 0;    // SpMV x ring: window half-width H (0 = no ring)
    // x ring (device/spmv_ring.cuh), planned by plan_spmv_ring
    int32_t ring_nseg = 0;       // x segment slots
    int32_t ring_nrp = 0;        // row-bound stages per consumer warp (prefetch depth)
    int32_t ring_rp_stride = 0;  // int64 entries per row-bound stage
    int32_t ring_kb = 1;         // rows per group per round (= outer_unroll)
    int32_t ring_tps = 0;        // teams per SM the ring is sized for
    int64_t per_team = 0;        // rows per team
    // NEST_F_X_L2_PERSIST: per-launch access-policy window over x (launch_one)
    const void* l2_win = nullptr;    // base (x); nullptr = plain launch
    int64_t l2_win_bytes = 0;        // bytes under the window
    int64_t l2_setaside = 0;         // persisting-L2 set-aside the hit ratio is computed from
};

// 32-bit row / nonzero indices (and 32-bit outer-loop cursors, engine.cuh
// outer_index) when every index and every schedule position fits with room to
// spare: fewer instructions and registers per row.
inline bool spmv_index32(const Plan& p, int64_t nnz) {
    const int64_t lim = (int64_t)1 << 30;
    // every cursor position: outer iterations, team chunk starts (grid * chunk), and
    // the cyclic schedule's group ids and strides (grid * groups) -- ADVICE r1
    return nnz < ((int64_t)1 << 31) - 8 && p.outer < lim && (int64_t)p.grid * p.chunk < lim &&
           (int64_t)p.grid * p.groups < lim;
}

// NEST_F_X_L2_PERSIST sizing for an x of ncols doubles on the current device:
// window = min(x bytes, max window), set-aside = max(current limit, min(max
// persisting, 3/8 of L2)).  apply: also raise the device's persisting-L2 limit
// to the set-aside (once per device) and point the window at x.
nest_status x_persist_window(Plan* p, const double* x, int64_t ncols, bool apply);

// Launch `kern` with the plan's geometry arguments; when the plan carries an x window
// (NEST_F_X_L2_PERSIST) the launch goes through cudaLaunchKernelEx with a per-launch
// access-policy window (hits persisting, misses normal), so the caller's stream
// attributes stay untouched.  Returns the launch error.
template <class Kern, class... Args>
cudaError_t launch_with_plan(const Plan& p, Kern kern, dim3 grid, dim3 block, size_t smem, cudaStream_t st,
                             Args... args) {
    if (!p.l2_win) {
        kern<<<grid, block, smem, st>>>(args...);
        return cudaGetLastError();
    }
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeAccessPolicyWindow;
    attr[0].val.accessPolicyWindow.base_ptr = const_cast<void*>(p.l2_win);
    attr[0].val.accessPolicyWindow.num_bytes = (size_t)p.l2_win_bytes;
    attr[0].val.accessPolicyWindow.hitRatio =
        p.l2_setaside >= p.l2_win_bytes ? 1.0f : (float)((double)p.l2_setaside / (double)p.l2_win_bytes);
    attr[0].val.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
    attr[0].val.accessPolicyWindow.missProp = cudaAccessPropertyNormal;
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = grid;
    cfg.blockDim = block;
    cfg.dynamicSmemBytes = smem;
    cfg.stream = st;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    return cudaLaunchKernelEx(&cfg, kern, args...);
}

// Record a thread-local error message and return `s`.
nest_status fail(nest_status s, const char* fmt, ...) __attribute__((format(printf, 2, 3)));
nest_status cuda_fail(cudaError_t e, const char* what);

// Validate `d` and compute the plan for `outer` outer iterations of a body
// with `steps_per_outer` simd loops each; payload_of(U) is the generic payload
// one group posts per simd batch at unroll U.
using PayloadFn = int32_t (*)(int32_t unroll);
nest_status make_plan(const nest_desc* d, int64_t outer, int32_t steps_per_outer,
                      PayloadFn payload_of, Plan* p, bool spmv_window = false);
// as make_plan with a fixed payload (the nest_plan ABI entry)
nest_status make_plan_fixed(const nest_desc* d, int64_t outer, int32_t steps_per_outer,
                            int32_t payload_bytes, Plan* p, bool spmv_window = false);

// Library-owned global fallback for the sharing space:
// grown lazily, never shrunk, released by nest_shutdown().
nest_status fallback_scratch(size_t bytes, unsigned char** out, void* stream);
// the fallback a plan needs (nullptr when it needs none)
nest_status prepare_fallback(const Plan& p, unsigned char** fb, void* stream);

// Payload bytes a body posts per simd batch for a given unroll.
int32_t spmv_payload(int32_t U);
int32_t batched_payload(int32_t U);
int32_t stencil_payload(int32_t U);
int32_t probe_payload(int32_t U);
int32_t laplace_payload(int32_t U);

// Kernel launchers (one translation unit per body).
nest_status launch_spmv(const Plan& p, bool hints, int64_t nrows, const int64_t* rowptr,
                        const int32_t* col, const double* val, const double* x, double* y,
                        unsigned char* fb, cudaStream_t st, int64_t nnz);
// x ring (x_halo > 0): finish the plan (ring sizes, teams, payload of the launched
// body) from the matrix shape, and launch.
nest_status plan_spmv_ring(Plan* p, int64_t nrows, int64_t nnz, int32_t num_teams, int32_t teams_per_sm);
nest_status launch_spmv_ring(const Plan& p, int64_t nrows, int64_t ncols, int64_t nnz, const int64_t* rowptr,
                             const int32_t* col, const double* val, const double* x, double* y,
                             unsigned char* fb, cudaStream_t st);
// payload (bytes of one generic slot) of the body launch_spmv runs for plan p
int32_t spmv_body_payload(const Plan& p, int64_t nnz);
nest_status resident_blocks(int32_t T, int32_t smem, int64_t* out);
nest_status launch_batched(const Plan& p, int64_t batch, int32_t m, int32_t n, const float* A,
                           const float* x, float* y, unsigned char* fb, cudaStream_t st);
nest_status launch_stencil(const Plan& p, int64_t nouter, int32_t L, const double* in,
                           const double* coef, const double* w, double* out,
                           unsigned long long* visits, unsigned char* fb, cudaStream_t st);
nest_status launch_spmv_teams_generic(const Plan& p, int64_t nrows, const int64_t* rowptr, const int32_t* col,
                                      const double* val, const double* x, double* y, cudaStream_t st);
nest_status launch_laplace(const Plan& p, int64_t nz, int64_t ny, int64_t nx, double alpha, const double* u,
                           double* out, unsigned char* fb, cudaStream_t st);
nest_status launch_probe(const Plan& p, int32_t* out_map, int64_t trip, int32_t* hits,
                         int32_t* owner, double* totals, unsigned char* fb, cudaStream_t st);

}  // namespace nest
