// launch_spmv_ring.cu -- a8 CSR SpMV with the x ring (x_halo > 0): the planner
// (a1 for this kernel) and the launcher.  Kernel: device/spmv_ring.cuh.
#include <algorithm>

#include "ring_dispatch.cuh"

namespace nest {

namespace {

constexpr int32_t kSmemPerSm = 228 * 1024;
constexpr int32_t kSmemReservedPerBlock = 1024;
constexpr int32_t kMaxDynSmem = 227 * 1024;

enum RingBody { kScalar32, kScalar64, kPair32, kQuad32, kNone };

RingBody ring_body(const Plan& p, int64_t nrows, int64_t nnz) {
    (void)nrows;
    const bool i32 = nnz < ((int64_t)1 << 31) - 8;
    if (p.flags & NEST_F_VEC128) return i32 ? ((p.flags & NEST_F_VEC_QUAD) ? kQuad32 : kPair32) : kNone;
    return i32 ? kScalar32 : kScalar64;
}

int32_t ring_payload(RingBody b) {
    switch (b) {
        case kScalar32: return payload_bytes<RingScalar32, 1>();
        case kScalar64: return payload_bytes<RingScalar64, 1>();
        case kPair32: return payload_bytes<RingPair32, 1>();
        case kQuad32: return payload_bytes<RingQuad32, 1>();
        default: return 0;
    }
}

}  // namespace

// Ring geometry: the copy warp plus nc = T/32 - 1 consumer warps,
// G = nc*32/S consumer groups, rounds of R = G * KB rows (KB = outer_unroll), per
// consumer warp kRingDepth row-bound stages of KB*(32/S + 1) entries, and an x
// ring of NS segments of kRingSeg doubles.  One round's window spans at most
// ceil((R + 2H) / SEG) + 1 segments; the ring must hold that plus slack for the
// warps to drift apart.  Preference: the requested / fitting teams per SM with
// >= max(4, 2R/SEG) slack segments (two teams first: latency hiding), then any
// ring with slack >= 1.
nest_status plan_spmv_ring(Plan* q, int64_t nrows, int64_t nnz, int32_t num_teams, int32_t teams_per_sm) {
    const int32_t T = q->block, S = q->simdlen;
    const int32_t nc = T / 32 - 1;
    if (nc < 1) return fail(NEST_ERR_INVALID_ARG, "x_halo needs threads_per_team >= 64 (a copy warp + consumers)");
    if (nrows >= ((int64_t)1 << 31) - 8) return fail(NEST_ERR_UNSUPPORTED, "x_halo needs nrows < 2^31");
    const RingBody body = ring_body(*q, nrows, nnz);
    if (body == kNone) return fail(NEST_ERR_UNSUPPORTED, "x_halo with NEST_F_VEC128 needs nnz, nrows < 2^31");
    const int64_t G = (int64_t)nc * 32 / S;
    const int64_t KB = q->unroll;
    const int64_t R = G * KB;
    const int64_t H = q->x_halo;
    const int64_t span = (R + 2 * H + kRingSeg - 1) / kRingSeg + 1;
    const int64_t want = std::max<int64_t>(4, 2 * ((R + kRingSeg - 1) / kRingSeg));
    const int32_t stage = (int32_t)((KB * (32 / S + 1) + 1) & ~(int64_t)1);
    const int32_t sharing = q->smem_bytes;   // generic-SMEM sharing space (0 otherwise)
    int32_t best_tps = 0, best_ns = 0, best_total = 0;
    for (int pass = 0; pass < 2 && !best_tps; ++pass) {
        for (int32_t tps = 2; tps >= 1 && !best_tps; --tps) {
            if ((tps == 2 && T > 768) || (teams_per_sm && tps != teams_per_sm)) continue;   // registers
            const int32_t budget = std::min(kSmemPerSm / tps - kSmemReservedPerBlock, kMaxDynSmem);
            int64_t ns = (budget - RingLayout::of(0, nc, kRingDepth, stage, sharing).total) / (kRingSeg * 8 + 16);
            while (ns > 0 && RingLayout::of((int32_t)ns, nc, kRingDepth, stage, sharing).total > budget) --ns;
            if (ns >= span + (pass == 0 ? want : 1)) {
                // no more ring than the window plus its slack: the rest of the SM's
                // unified L1/shared array stays L1 for the CSR stream and far gathers
                if (pass == 0) ns = std::min<int64_t>(ns, span + 2 * want);
                best_tps = tps, best_ns = (int32_t)ns;
                best_total = RingLayout::of((int32_t)ns, nc, kRingDepth, stage, sharing).total;
            }
        }
    }
    if (!best_tps)
        return fail(NEST_ERR_UNSUPPORTED,
                    "x_halo %d with rounds of %lld rows needs more than %d B of shared memory per team",
                    q->x_halo, (long long)R, kMaxDynSmem);
    q->groups = (int32_t)G;
    q->slot_bytes = (sharing / q->groups) & ~7;   // the sharing space split among the consumer groups
    q->payload_bytes = ring_payload(body);
    q->fallback = sharing > 0 && q->payload_bytes > q->slot_bytes;
    q->ring_kb = (int32_t)KB;
    q->ring_nrp = kRingDepth;
    q->ring_nseg = best_ns;
    q->ring_rp_stride = stage;
    q->ring_tps = best_tps;
    q->smem_bytes = best_total;
    const int64_t rounds = (nrows + R - 1) / R;
    if (num_teams > 0) {
        q->grid = num_teams;
    } else {
        // one league of resident teams: best_tps per SM (the kernel's register budget
        // is sized for exactly that many, __launch_bounds__)
        int64_t resident = 0;
        nest_status s = resident_blocks(T, best_total, &resident);
        if (s != NEST_OK) return s;
        int64_t per_sm_1 = 0;
        if ((s = resident_blocks(2048, 0, &per_sm_1)) != NEST_OK) return s;   // = the SM count
        resident = std::min<int64_t>(resident, per_sm_1 * best_tps);
        q->grid = (int32_t)std::max<int64_t>(1, std::min(resident, rounds));
    }
    q->per_team = std::max<int64_t>(1, (nrows + q->grid - 1) / q->grid);
    q->chunk = q->per_team;
    return NEST_OK;
}

nest_status launch_spmv_ring(const Plan& p, int64_t nrows, int64_t ncols, int64_t nnz, const int64_t* rowptr,
                             const int32_t* col, const double* val, const double* x, double* y,
                             unsigned char* fb, cudaStream_t st) {
    const RingArgs a{rowptr, col, val, x, y, nrows, ncols, nnz, p.per_team, p.x_halo,
                     p.ring_nseg, p.ring_nrp, p.ring_rp_stride, p.ring_kb, p.slot_bytes, fb,
                     FastDivU32::make((uint32_t)p.ring_nseg)};
    static_assert(kRingDepth == 4, "RingArgs.depth mirrors the kernel's constant");
    switch (ring_body(p, nrows, nnz)) {
        case kScalar32: return ring_scalar32(p, a, st);
        case kScalar64: return ring_scalar64(p, a, st);
        case kPair32: return ring_pair32(p, a, st);
        case kQuad32: return ring_quad32(p, a, st);
        default: return fail(NEST_ERR_UNSUPPORTED, "x_halo with NEST_F_VEC128 needs nnz, nrows < 2^31");
    }
}

}  // namespace nest
