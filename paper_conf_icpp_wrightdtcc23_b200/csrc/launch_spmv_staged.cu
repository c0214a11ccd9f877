// launch_spmv_staged.cu -- a8 CSR SpMV, warp-specialised bulk-copy pipeline
// (NEST_F_STAGED): planning of the stage sizes and the template dispatch.
#include <cstdio>
#include <cstdlib>

#include "device/spmv_staged.cuh"
#include "internal.h"

namespace nest {

static constexpr int32_t kStagedMaxSmem = 227 * 1024;

// Stage sizes: chunks of R rows (a multiple of the G*U rows of a batch, even)
// whose nonzeros are staged up to NB per stage (rows beyond take the global
// path); the x ring needs NS*R + 2H doubles (spmv_staged.cuh).  NB is sized
// for 1.25x the chunk's expected nonzeros; among the (NS, R) that fit shared
// memory take the most bytes in flight while a stage is consumed, (NS-1)*R.
nest_status plan_spmv_staged(Plan* p, int64_t nrows, int64_t nnz, int32_t sharing_bytes) {
    const int32_t T = p->block;
    const int32_t S = p->simdlen;
    const int32_t G = (T - 32 * (1 + kGatherWarps)) / S;
    if (G <= 0)
        return fail(NEST_ERR_INVALID_ARG, "NEST_F_STAGED: threads_per_team %d leaves no consumer warps (need >= %d)",
                    T, 32 * (2 + kGatherWarps));
    const int32_t B = G * p->unroll;
    const bool smem_mode = p->mode == NEST_MODE_GENERIC_SMEM;
    p->groups = G;
    p->slot_bytes = (sharing_bytes / G) & ~7;   // even split, 8-byte aligned slots (R8)
    p->fallback = smem_mode && p->payload_bytes > p->slot_bytes;
    const int32_t sh = smem_mode ? p->slot_bytes * G : 0;
    const double avg = nrows > 0 && nnz > 0 ? (double)nnz / (double)nrows : 1.0;
    const int64_t halo = ((int64_t)p->x_halo + 1) & ~(int64_t)1;
    double best_score = -1;
    int32_t best_ns = 0, best_nb = 0, best_xw = 0, best_r = 0;
    // developer overrides for tuning sweeps (NEST_STAGED_NS / NEST_STAGED_R)
    const char* env_ns = std::getenv("NEST_STAGED_NS");
    const char* env_r = std::getenv("NEST_STAGED_R");
    const int32_t ns_lo = env_ns ? std::atoi(env_ns) : 2, ns_hi = env_ns ? std::atoi(env_ns) : 4;
    for (int32_t ns = ns_lo; ns <= ns_hi; ++ns) {
        // candidate chunk sizes, largest first: 64B, 63B, ..., B, B/2, B/4, ... (even)
        for (int64_t m = 64 + 6; m >= 1; --m) {
            int64_t R = m > 6 ? (int64_t)B * (m - 6) : ((int64_t)B >> (7 - m));
            if (env_r) {
                if (m != 1) continue;
                R = std::atoi(env_r);
            }
            if (R < 2) continue;
            R = (R + 1) & ~(int64_t)1;
            if (R > 16384) continue;
            int64_t xw = halo > 0 ? (int64_t)ns * R + 2 * halo : 0;
            xw = (xw + 1) & ~(int64_t)1;
            if (xw > (1 << 24)) continue;
            const int64_t want = (((int64_t)(1.25 * avg * R) + 8) + 3) & ~(int64_t)3;
            // the largest NB <= want that fits shared memory
            const StagedLayout l0 = staged_layout((int32_t)xw, 0, ns, (int32_t)R, sh);
            if (l0.total >= (uint32_t)kStagedMaxSmem) continue;
            int64_t nb = ((int64_t)kStagedMaxSmem - l0.total) / ns / 20;
            nb &= ~(int64_t)3;
            if (nb > want) nb = want;
            while (nb >= 64 && staged_layout((int32_t)xw, (int32_t)nb, ns, (int32_t)R, sh).total >
                                   (uint32_t)kStagedMaxSmem)
                nb -= 4;
            if (nb < 64) continue;
            // bytes in flight while a stage is consumed, discounted when rows spill past NB
            const double score = (double)(ns - 1) * (double)R * ((double)nb / (double)want);
            if (score > best_score + 1e-9) {
                best_score = score;
                best_ns = ns;
                best_nb = (int32_t)nb;
                best_xw = (int32_t)xw;
                best_r = (int32_t)R;
            }
            if (nb == want) break;   // the largest chunk whose nonzeros fit at this NS
        }
    }
    if (best_ns == 0)
        return fail(NEST_ERR_UNSUPPORTED,
                    "NEST_F_STAGED: x_halo %d with %d rows per batch does not fit shared memory", p->x_halo, B);
    p->x_halo = (int32_t)halo;
    p->ns = best_ns;
    p->nb = best_nb;
    p->xw = best_xw;
    p->rmax = best_r;
    p->smem_bytes = (int32_t)staged_layout(best_xw, best_nb, best_ns, best_r, sh).total;
    if (std::getenv("NEST_DEBUG_PLAN"))
        std::fprintf(stderr, "[nest] staged plan: T=%d S=%d U=%d G=%d B=%d R=%d NB=%d NS=%d XW=%d smem=%d\n", T, S,
                     p->unroll, G, B, best_r, best_nb, best_ns, best_xw, p->smem_bytes);
    if (p->grid <= 0) {
        int64_t resident = 0;
        nest_status s = resident_blocks(T, p->smem_bytes, &resident);
        if (s != NEST_OK) return s;
        const int64_t needed = (nrows + best_r - 1) / best_r;
        p->grid = (int32_t)(needed < resident ? (needed > 0 ? needed : 1) : resident);
    }
    return NEST_OK;
}

template <int S, int MODE, int OP, int U>
static nest_status staged_one(const Plan& p, const StagedArgs& a, cudaStream_t st) {
    auto* k = spmv_staged_kernel<S, MODE, OP, U>;
    cudaError_t e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, p.smem_bytes);
    if (e != cudaSuccess) return cuda_fail(e, "cudaFuncSetAttribute(max dynamic smem)");
    k<<<p.grid, p.block, p.smem_bytes, st>>>(a);
    e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_fail(e, "spmv_staged launch");
    return NEST_OK;
}

template <int S, int MODE, int U>
static nest_status staged_op(const Plan& p, const StagedArgs& a, cudaStream_t st) {
    switch (p.reduce) {
        case RED_SUM: return staged_one<S, MODE, RED_SUM, U>(p, a, st);
        case RED_MAX: return staged_one<S, MODE, RED_MAX, U>(p, a, st);
        case RED_MIN: return staged_one<S, MODE, RED_MIN, U>(p, a, st);
    }
    return fail(NEST_ERR_INVALID_ARG, "reduce %d", p.reduce);
}

template <int S, int U>
static nest_status staged_mode(const Plan& p, const StagedArgs& a, cudaStream_t st) {
    if constexpr (S == 1) {
        return staged_op<1, MODE_SPMD, U>(p, a, st);
    } else {
        switch (p.mode) {
            case MODE_SPMD: return staged_op<S, MODE_SPMD, U>(p, a, st);
            case MODE_GENERIC_SMEM: return staged_op<S, MODE_GENERIC_SMEM, U>(p, a, st);
            case MODE_GENERIC_SHFL: return staged_op<S, MODE_GENERIC_SHFL, U>(p, a, st);
        }
    }
    return fail(NEST_ERR_INVALID_ARG, "mode %d", p.mode);
}

template <int U>
static nest_status staged_simdlen(const Plan& p, const StagedArgs& a, cudaStream_t st) {
    switch (p.simdlen) {
        case 1: return staged_mode<1, U>(p, a, st);
        case 2: return staged_mode<2, U>(p, a, st);
        case 4: return staged_mode<4, U>(p, a, st);
        case 8: return staged_mode<8, U>(p, a, st);
        case 16: return staged_mode<16, U>(p, a, st);
        case 32: return staged_mode<32, U>(p, a, st);
    }
    return fail(NEST_ERR_INVALID_ARG, "simdlen %d", p.simdlen);
}

nest_status launch_spmv_staged(const Plan& p, int64_t nrows, int64_t ncols, int64_t nnz,
                               const int64_t* rowptr, const int32_t* col, const double* val,
                               const double* x, double* y, unsigned char* fb, cudaStream_t st) {
    static unsigned long long* trace = nullptr;
    if (!trace && std::getenv("NEST_TRACE")) {
        if (cudaMallocManaged(&trace, 256 * sizeof(unsigned long long)) != cudaSuccess) trace = nullptr;
        std::atexit([] {
            cudaDeviceSynchronize();
            const char* tag = "PFGC";
            for (int k = 0; k < 64; ++k) {
                std::fprintf(stderr, "[nest trace] %d", k);
                for (int e = 0; e < 4; ++e)
                    std::fprintf(stderr, " %c=%.3f", tag[e], trace[e * 64 + k] ? (trace[e * 64 + k] - trace[0]) / 1e3 : -1.0);
                std::fprintf(stderr, "\n");
            }
        });
    }
    const StagedArgs a{rowptr, col, val, x, y, nrows, ncols, nnz, p.x_halo, p.xw, p.nb, p.ns,
                       p.rmax, p.slot_bytes, trace, fb};
    switch (p.unroll) {
        case 1: return staged_simdlen<1>(p, a, st);
        case 2: return staged_simdlen<2>(p, a, st);
        case 4: return staged_simdlen<4>(p, a, st);
    }
    return fail(NEST_ERR_INVALID_ARG, "outer_unroll %d", p.unroll);
}

}  // namespace nest
