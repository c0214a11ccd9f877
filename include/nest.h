/*
 * nest.h -- C ABI of the B200 three-level (teams -> parallel -> simd) loop-nest
 * library.  ABI v2 (v2: NEST_F_X_L2_PERSIST and the nest_plan_info l2_* fields).
 *
 * What it executes (PAPER.md = /root/reference/PAPER.md, Wright et al.,
 * "Implementing OpenMP's SIMD Directive in LLVM's GPU Runtime", ICPP'23):
 *   - teams    -> thread blocks ("league of teams")
 *   - parallel -> SIMD groups of `simdlen` adjacent lanes inside one warp
 *                 (getSimdGroup/Id/Size, isSimdGroupLeader,
 *                 simdmask: PAPER.md:507-529)
 *   - simd     -> the lanes of a group, cyclic worksharing iv = id, id+S, ...
 *                 (Fig 8)
 * in one of the two execution models of the parallel region:
 *   - SPMD (GPU-centric): every lane runs the sequential
 *     code redundantly, side effects guarded to the SIMD main;
 *   - generic (CPU-centric, Figs 3/4/6): only the SIMD
 *     main runs the sequential code; before each simd loop it posts
 *     {fn, trip count, loop state} to its group and releases the workers with
 *     a warp-level barrier; a null fn terminates.  The state travels through
 *     the group's slot of a shared-memory "variable sharing space"
 *     (2048 B per team by default, split evenly, global
 *     fallback when it does not fit) -- NEST_MODE_GENERIC_SMEM -- or through
 *     warp shuffles from the main -- NEST_MODE_GENERIC_SHFL (north_star).
 * Each simd loop ends with a reduction across the group's lanes by a
 * __shfl_xor_sync butterfly (north_star addition: the paper has no reduction,
 * PAPER.md:868-873, 880-884).  simdlen = 1 is the flat two-level mapping
 * (simd folded into threads).
 *
 * Conventions for every entry point:
 *   - Array arguments are DEVICE pointers owned by the caller (except the
 *     *_hostio call, whose data arguments are HOST pointers).  `stream` is a
 *     cudaStream_t passed as void* (NULL = legacy default stream).
 *   - Calls are asynchronous and stream-ordered; they never synchronise the
 *     device except where stated.  Device faults surface at the caller's
 *     next synchronisation.
 *   - All validation happens BEFORE any launch; a non-OK status means nothing
 *     was enqueued.  Zero-size problems return NEST_OK without a launch.
 *   - nest_last_error() returns a thread-local description of the last
 *     non-OK status.  Nothing throws across the ABI.
 *   - Preconditions that are documented but not checked in the hot path:
 *     rowptr monotone with rowptr[0] == 0 and rowptr[nrows] == nnz,
 *     0 <= colind < ncols; pointers suitably aligned for their type.
 *     nest_csr_validate() checks the CSR ones on the device.
 *   - The library allocates nothing per call in steady state.  Library-owned
 *     lazily-grown device scratch (the sharing-space global fallback,
 *     PAPER.md:680-684), one buffer per (device, stream) so that concurrent
 *     launches on different streams never share slots, is released by
 *     nest_shutdown() (all of the current device's buffers).
 */
#ifndef NEST_H
#define NEST_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define NEST_ABI_VERSION 2u

typedef enum {
    NEST_OK = 0,
    NEST_ERR_INVALID_ARG = 1,   /* bad extent, simdlen, team size, null pointer ... */
    NEST_ERR_UNSUPPORTED = 2,   /* valid but not built (e.g. T above the kernel's limit) */
    NEST_ERR_CUDA = 3,          /* a CUDA runtime call failed (no device, launch error) */
    NEST_ERR_NCCL = 4,
    NEST_ERR_NO_MEMORY = 5
} nest_status;

/* Execution model of the parallel region. */
typedef enum {
    NEST_MODE_SPMD = 0,          /* all lanes run everything; no communication */
    NEST_MODE_GENERIC_SMEM = 1,  /* main posts loop state in the shared sharing space */
    NEST_MODE_GENERIC_SHFL = 2,  /* main broadcasts loop state with warp shuffles */
    /* NEXT-1, SpMV only: the paper's TWO-level baseline --
     * teams in generic mode with an extra team-main warp and a block-level
     * state machine, `parallel for` over a row's nonzeros on the team's
     * threads_per_team workers; no simd level (simdlen must be 1). */
    NEST_MODE_TEAMS_GENERIC = 3
} nest_mode;

/* Reduction of the simd loop (identity +0.0 / -inf / +inf). */
typedef enum { NEST_REDUCE_SUM = 0, NEST_REDUCE_MAX = 1, NEST_REDUCE_MIN = 2 } nest_reduce;

/* flags */
enum {
    /* grid = min(needed, resident blocks) and teams stride over the outer
     * loop ("teams distribute" with a persistent league).  Implied when the
     * sharing space falls back to global memory. */
    NEST_F_PERSISTENT_GRID = 1u << 0,
    /* SpMV cache hints (results unchanged): scalar path -- stream the CSR arrays
     * with L1 no-allocate / L2 evict-first loads; 128-bit path -- the CSR
     * tuples with L1 no-allocate loads (L1 kept for the x gathers). */
    NEST_F_STREAM_HINTS = 1u << 1,
    /* bit 2 is reserved (an earlier staged-pipeline variant; rejected as an unknown flag). */
    /* "teams distribute" with a static block schedule: team b owns the
     * contiguous outer range [b*C, (b+1)*C) (C = ceil(outer / grid) rounded up
     * to a multiple of G, or team_chunk: then chunks b, b + grid, ...) and its
     * SIMD groups take it cyclically, so the rows in flight on an SM are
     * neighbours (x stays in L1/L2 for banded matrices).  Implies a persistent
     * grid.  Results are identical (the schedule never changes a row's
     * arithmetic). */
    NEST_F_BLOCKED = 1u << 3,
    /* 128-bit loads (SpMV; nested stencil: pairs of inner iterations, see
     * nest_nested_stencil_f64; batched matvec: float4 tuples of a row, needs
     * n % 4 == 0 and 16-byte aligned A and x).  SpMV: the simd loop runs over pairs of nonzeros
     * (one 128-bit val load, one 64-bit colind load per pair), lane l taking
     * pairs l, l+S, ... of the row ("blocked-cyclic" order: real results
     * differ from the scalar order by rounding only).  Needs 16-byte aligned
     * val and 8-byte aligned colind. */
    NEST_F_VEC128 = 1u << 4,
    /* with NEST_F_VEC128: quads instead of pairs (one 128-bit colind load and
     * one 256-bit val load per lane iteration); needs 16-byte aligned colind and
     * 32-byte aligned val. */
    NEST_F_VEC_QUAD = 1u << 5,
    /* SpMV (nest_kernel variants: cyclic / blocked, scalar / pair / quad loads;
     * the x ring; also the dist and hostio entry points): x is marked L2-persisting for
     * this launch.  Why: the far columns of a short-row matrix gather x at
     * random, and with x (80-100 MB) competing against the streamed CSR arrays
     * for the 126 MB L2 most of those gathers miss and cost a DRAM access each
     * (DESIGN.md §6).  How: the library makes sure the device's persisting-L2
     * set-aside (cudaLimitPersistingL2CacheSize, a DEVICE-WIDE limit; normal
     * accesses still use it while no persisting line occupies it) is at least
     * min(cudaDevAttrMaxPersistingL2CacheSize, 1/2 of L2), and launches the
     * kernel with a per-launch access-policy window over x (cudaLaunchKernelEx:
     * hitRatio = set-aside / window bytes, hits persisting, misses normal), so
     * the caller's stream attributes are untouched.  Results are identical (a
     * cache policy only).  The persisting lines outlive the call (a following
     * SpMV on the same x finds them); nest_util_l2_flush returns them to
     * normal, and nest_shutdown also restores the limit.  With
     * NEST_MODE_TEAMS_GENERIC or the peer-gather SpMV: NEST_ERR_UNSUPPORTED;
     * other entry points: NEST_ERR_INVALID_ARG. */
    NEST_F_X_L2_PERSIST = 1u << 6
};

/* The nest descriptor: team, thread and simd extents, mode and reduction.
 * Zero-initialise, set abi_version = NEST_ABI_VERSION, then override. */
typedef struct {
    uint32_t abi_version;       /* == NEST_ABI_VERSION */
    int32_t num_teams;          /* grid size; 0 = auto (see nest_plan) */
    int32_t threads_per_team;   /* T: multiple of 32 in [32, 1024]; 0 = 256 */
    int32_t simdlen;            /* S: SIMD group size 1, 2, 4, 8, 16 or 32 */
    int32_t mode;               /* nest_mode */
    int32_t reduce;             /* nest_reduce */
    int32_t sharing_bytes;      /* generic sharing space per team; 0 = 2048 */
    uint32_t flags;             /* NEST_F_* */
    int32_t outer_unroll;       /* U: outer iterations a group keeps in flight (1, 2, 4); 0 = 1 */
    int32_t x_halo;             /* SpMV only.  H > 0: the x ring.  Each team owns a
                                 * contiguous range of rows and walks it in rounds of R = G*U rows
                                 * (G = (T - 32)/S consumer groups; here outer_unroll U is the rows a
                                 * group runs per round, one after another); its last warp bulk-copies
                                 * (TMA engine) each round's row bounds and the x window
                                 * [row0 - H, row0 + R + H) into shared-memory rings ahead of use, with
                                 * mbarriers instead of team barriers.  Columns inside the window read
                                 * the ring, others read x in global memory: results are identical for
                                 * every H (bit-identical to nest_kernel at the same S, mode and loads).
                                 * Needs T >= 64 and 16-byte aligned x; scalar, pair or quad loads
                                 * (tuples need nnz < 2^31); nrows < 2^31.  0 = no ring. */
    int32_t team_chunk;         /* with NEST_F_BLOCKED: outer iterations per team chunk, rounded up to
                                 * a multiple of G; team b takes chunks b, b + grid, b + 2 grid, ...
                                 * (its groups cyclically inside a chunk), so all teams sweep the
                                 * outer range together.  0 = one contiguous range per team. */
    int32_t teams_per_sm;       /* x ring only: teams sharing an SM that the rings are sized for
                                 * (1 or 2; 0 = the planner's choice).  Two teams of
                                 * 1024 get 32 registers per thread and ~94 KB of ring each; one team
                                 * gets 64 registers and ~190 KB.  Must be 0 without x_halo. */
} nest_desc;

/* Which kernel an SpMV plan launches (nest_plan_info.kernel). */
enum {
    NEST_KERNEL_NEST = 0,           /* nest_kernel: the loop-nest engine (engine.cuh) */
    NEST_KERNEL_XRING = 1,          /* spmv_ring_kernel: x_halo > 0 (device/spmv_ring.cuh) */
    NEST_KERNEL_TEAMS_GENERIC = 2   /* NEXT-1 two-level baseline (device/teams_generic.cuh) */
};

/* Resolved launch geometry (a1). */
typedef struct {
    int32_t grid;                 /* teams (blocks) */
    int32_t block;                /* threads per team T */
    int32_t groups_per_team;      /* G = T / S (x ring: (T - 32) / S consumer groups) */
    int32_t slot_bytes;           /* sharing_bytes / G rounded down to 8 (generic-SMEM slot per group) */
    int32_t payload_bytes;        /* bytes one group posts per simd batch (nest_spmv_plan: of the body
                                   * that actually runs) */
    int32_t uses_global_fallback; /* payload_bytes > slot_bytes (GENERIC_SMEM only); the kernel
                                   * follows this decision */
    int32_t outer_unroll;         /* U */
    int32_t smem_bytes;           /* dynamic shared memory per team */
    int32_t kernel;               /* NEST_KERNEL_* */
    int32_t index_bits;           /* 32 or 64: row / nonzero index width of the launched body */
    int32_t ring_segments;        /* x ring: segment slots of 256 doubles (else 0) */
    int32_t ring_row_slots;       /* x ring: row-bound slots (else 0) */
    int64_t chunk;                /* blocked schedule / x ring: outer iterations per team chunk (else 0) */
    int64_t l2_window_bytes;      /* NEST_F_X_L2_PERSIST: bytes of x under the access-policy window (else 0) */
    int64_t l2_setaside_bytes;    /* NEST_F_X_L2_PERSIST: the persisting-L2 set-aside the launch uses (hit
                                   * ratio = min(1, setaside / window)); else 0 */
} nest_plan_info;

uint32_t nest_abi_version(void);
const char *nest_status_str(nest_status s);
const char *nest_last_error(void);

/* a1: validate `desc` and resolve the geometry for `outer_iters` outer
 * iterations whose generic payload is `payload_bytes` per group.  Host-only
 * unless the grid must be sized from device occupancy (num_teams == 0 with
 * NEST_F_PERSISTENT_GRID or a global fallback), which queries the current
 * device (NEST_ERR_CUDA without one).  Errors: NEST_ERR_INVALID_ARG. */
nest_status nest_plan(const nest_desc *desc, int64_t outer_iters, int32_t payload_bytes,
                      nest_plan_info *out);

/* a1 for a8: the plan nest_spmv_csr_f64 launches for this descriptor and
 * matrix shape -- kernel, geometry, index width, x-ring sizing, and the payload
 * of the body that runs, so uses_global_fallback is exactly the kernel's
 * choice.  Queries the current device when the grid is sized from occupancy
 * (num_teams == 0 with a persistent/blocked grid, a fallback, or the x ring).
 * Errors: as nest_spmv_csr_f64's validation. */
nest_status nest_spmv_plan(const nest_desc *desc, int64_t nrows, int64_t ncols, int64_t nnz,
                           nest_plan_info *out);

/* a8: CSR SpMV, y[i] = (+)_{k in [rowptr[i], rowptr[i+1])} val[k] * x[colind[k]]
 * (sparse_matvec).  Outer (parallel) unit = a row; simd
 * unit = a nonzero of the row.  rowptr int64[nrows+1], colind int32[nnz],
 * val f64[nnz], x f64[ncols], y f64[nrows] (written).  nrows, ncols, nnz >= 0. */
nest_status nest_spmv_csr_f64(const nest_desc *desc, int64_t nrows, int64_t ncols, int64_t nnz,
                              const int64_t *rowptr, const int32_t *colind, const double *val,
                              const double *x, double *y, void *stream);

/* a8 end to end from HOST buffers (pinned for asynchronous copies): copies
 * rowptr/colind/val/x into `d_workspace` (device, >= nest_spmv_hostio_workspace_bytes),
 * runs nest_spmv_csr_f64 and copies y back into h_y.  Above 8 Mi nonzeros the
 * rows are split into chunks of ~8 Mi nonzeros (at most 32; NEST_HOSTIO_CHUNKS
 * overrides): x, then each chunk's rowptr/colind/val cross on a library-owned
 * H2D stream, chunk c's SpMV runs on `stream` once the entries it can read
 * have landed, and its y rows return on a library-owned D2H stream, so the
 * copies overlap the kernels and the two PCIe directions overlap each other.
 * Ordering is still that of `stream`: the copies start after the work queued
 * on it before the call, and work queued on it after the call starts after
 * the last y row is on the host.  Results equal nest_spmv_csr_f64's bit for
 * bit.  rowptr must start at 0 and end at nnz.  The host buffers must stay
 * valid, and h_y unread, until `stream` reaches that point.  d_workspace must
 * be 256-byte aligned.  The H2D/D2H streams and events are library-owned, one
 * set per device, guarded by a lock: concurrent callers on one device
 * serialise their enqueueing (not their kernels).  Pageable host buffers work
 * but make the copies synchronous. */
size_t nest_spmv_hostio_workspace_bytes(int64_t nrows, int64_t ncols, int64_t nnz);
nest_status nest_spmv_csr_f64_hostio(const nest_desc *desc, int64_t nrows, int64_t ncols,
                                     int64_t nnz, const int64_t *h_rowptr,
                                     const int32_t *h_colind, const double *h_val,
                                     const double *h_x, double *h_y, void *d_workspace,
                                     size_t workspace_bytes, void *stream);

/* a9: batched small dense matvec (SU3_bench stand-in):
 * y[b][r] = (+)_{k<n} A[b][r][k] * x[b][k], fp32.  Outer unit = a batch b;
 * the parallel region runs r = 0..m-1 sequentially, one simd loop over k each.
 * A f32[batch][m][n] row-major, x f32[batch][n], y f32[batch][m]. */
nest_status nest_batched_matvec_f32(const nest_desc *desc, int64_t batch, int32_t m, int32_t n,
                                    const float *A, const float *x, float *y, void *stream);

/* a10: nested loop with a sequential prologue ("benchmark kernel" stand-in,
 * PAPER.md:900-907; generic-vs-SPMD study PAPER.md:944-972).  For each outer i:
 *   scale = w[i]; base = 1 + i*L; visits += 1 (guarded: once per i in every mode);
 *   trip = scale == 0 ? 0 : L;
 *   s = (+)_{j<trip} coef[j] * ((in[base+j-1] + 2*in[base+j]) + in[base+j+1]);
 *   out[i] = trip == 0 ? +0.0 : scale * s.
 * in f64[nouter*L+2], coef f64[L], w f64[nouter], out f64[nouter];
 * visits: one u64 accumulated into (may be NULL).  NEST_F_VEC128: the simd
 * unit is a pair of inner iterations (two 128-bit loads of in, one of coef per
 * pair); needs an even L and 16-byte aligned in and coef (else
 * NEST_ERR_UNSUPPORTED); real results differ from the scalar lane order by
 * rounding only. */
nest_status nest_nested_stencil_f64(const nest_desc *desc, int64_t nouter, int32_t L,
                                    const double *in, const double *coef, const double *w,
                                    double *out, unsigned long long *visits, void *stream);

/* NEXT-2: laplace3d heat-diffusion step (Fig 10 cost study),
 * a simd loop WITHOUT a reduction.  u, out f64[nz][ny][nx] row-major (x fastest).
 * For every interior point (1 <= i < nz-1, 1 <= j < ny-1, 1 <= k < nx-1):
 *   lap = (((((u[i-1][j][k] + u[i+1][j][k]) + u[i][j-1][k]) + u[i][j+1][k])
 *            + u[i][j][k-1]) + u[i][j][k+1]) - 6*u[i][j][k]
 *   out[i][j][k] = u[i][j][k] + alpha*lap      (no FMA contraction)
 * Boundary points of out are not written.  Outer (parallel) unit = a line
 * (i, j), simd unit = k.  u and out must not alias.  NEST_F_VEC128: the simd
 * unit is the aligned pair k = 2t, 2t+1 (t < nx/2; boundary points computed
 * but not stored); needs an even nx and 16-byte aligned u and out (else
 * NEST_ERR_UNSUPPORTED); results are bit-identical to the scalar unit. */
nest_status nest_laplace3d_f64(const nest_desc *desc, int64_t nz, int64_t ny, int64_t nx,
                               double alpha, const double *u, double *out, void *stream);

/* a2/a5/a6 probe.  out_map int32[grid*block*5] (may be NULL): per thread
 * {getSimdGroup, getSimdGroupId, getSimdGroupSize, isSimdGroupLeader, simdmask}
 * (PAPER.md:507-529).  Then one outer iteration per group (outer = grid*G)
 * runs one simd loop of `trip` iterations through the selected mode engine:
 * hits int32[trip] (zeroed by the caller, may be NULL) receives one atomic
 * increment per group per iteration; owner int32[trip] (may be NULL) receives
 * the lane id that ran iteration j in global group 0 (Fig 8); totals
 * f64[grid*G] (may be NULL) receives each group's reduced count of executed
 * iterations (== trip under SUM).  num_teams must be > 0. */
nest_status nest_probe_mapping(const nest_desc *desc, int32_t *out_map, int64_t trip,
                               int32_t *hits, int32_t *owner, double *totals, void *stream);

/* Debug: check CSR preconditions on the device.  *d_bad (device int32, zeroed
 * by the caller) receives a nonzero value if rowptr is not monotone, does not
 * start at 0 / end at nnz, or a column index is out of range. */
nest_status nest_csr_validate(int64_t nrows, int64_t ncols, int64_t nnz, const int64_t *rowptr,
                              const int32_t *colind, int32_t *d_bad, void *stream);

/* Bench utility: flush L2.  Synchronises `stream`, returns every persisting L2
 * line of the context to normal (cudaCtxResetPersistingL2Cache: nothing a
 * NEST_F_X_L2_PERSIST launch left behind survives), then overwrites `bytes` of
 * device memory at `buf` and reads back its first half, so that L2 ends up
 * holding only clean lines unrelated to any later kernel (no dirty write-backs
 * inside the next, timed, kernel).  `bytes` should exceed twice the L2 size
 * (bench: 512 MiB). */
nest_status nest_util_l2_flush(void *buf, size_t bytes, void *stream);

/* ---- a12: row-partitioned multi-GPU SpMV (north_star; the paper is single-GPU) ----
 * One process per GPU.  Rank r owns rows [r*chunk, min((r+1)*chunk, n)) and the
 * same slice of x, chunk = ceil(n / nranks).  Each call all-gathers x over NCCL
 * (NVLink) into x_full (nranks*chunk doubles, so global column j is x_full[j])
 * and runs the local SpMV on the same stream. */
typedef struct nest_comm nest_comm;

/* 128-byte NCCL unique id, created on one rank and broadcast by the caller. */
nest_status nest_comm_unique_id(uint8_t out[128]);
/* Collective: every rank calls with the same id; binds the current device. */
nest_status nest_comm_init(const uint8_t id[128], int32_t nranks, int32_t rank, nest_comm **out);
nest_status nest_comm_destroy(nest_comm *comm);
/* Rows: chunk = ceil(nrows_global / nranks), this rank's nrows_local rows start at
 * rank*chunk; rowptr_local is 0-based for them and colind holds GLOBAL column
 * indices.  x: xchunk = ceil(ncols_global / nranks); x_local holds xchunk doubles
 * (entries past ncols_global on the tail rank are ignored); x_full receives
 * nranks*xchunk doubles, so global column j is x_full[j]. */
nest_status nest_spmv_csr_f64_dist(const nest_desc *desc, nest_comm *comm, int64_t nrows_global,
                                   int64_t ncols_global, int64_t nrows_local, int64_t nnz_local,
                                   const int64_t *rowptr_local, const int32_t *colind,
                                   const double *val, const double *x_local, double *x_full,
                                   double *y_local, void *stream);

/* a12's exchange step on its own: ncclAllGather of every rank's x_local
 * (xchunk doubles) into x_full (nranks*xchunk doubles) on `stream`. */
nest_status nest_comm_allgather_x(nest_comm *comm, const double *x_local, double *x_full, int64_t xchunk,
                                  void *stream);

/* a12 end to end from HOST buffers (pinned for asynchronous copies): the rank's
 * CSR shard (0-based rowptr_local, global colind), its x slice (xchunk doubles)
 * are copied into `d_workspace` (device, >= nest_spmv_dist_hostio_workspace_bytes,
 * 256-byte aligned), then nest_spmv_csr_f64_dist runs on the copies and y_local
 * returns to h_y_local.  All validation before the first copy. */
size_t nest_spmv_dist_hostio_workspace_bytes(int64_t nrows_local, int64_t nnz_local, int64_t xchunk,
                                             int32_t nranks);
nest_status nest_spmv_csr_f64_dist_hostio(const nest_desc *desc, nest_comm *comm, int64_t nrows_global,
                                          int64_t ncols_global, int64_t nrows_local, int64_t nnz_local,
                                          const int64_t *h_rowptr_local, const int32_t *h_colind,
                                          const double *h_val, const double *h_x_local, double *h_y_local,
                                          void *d_workspace, size_t workspace_bytes, void *stream);

/* ---- NEXT-3: several parallel regions with their own simdlen in ONE kernel ----
 * PAPER.md:511-513 ("the size could differ between parallel regions") and
 * PAPER.md:686-698.  Every team runs regions[0..nregions) in order; region k
 * partitions the team into SIMD groups of regions[k].simdlen lanes, re-divides
 * the sharing space among its T / simdlen groups (global fallback when the
 * region's payload does not fit) and ends with the team
 * barrier of the end of a parallel region.  Teams are independent, so a region
 * must not read what another team writes in an earlier region.  `desc` gives
 * the team geometry (num_teams: 0 = one resident league; threads_per_team;
 * sharing_bytes); its simdlen and mode are validated but unused; reduce must be
 * SUM, outer_unroll 1, flags and team_chunk 0.  Each region's output is
 * bit-identical to the stand-alone entry point at the same simdlen and mode. */
#define NEST_MAX_REGIONS 4
typedef enum {
    NEST_REGION_SPMV_CSR_F64 = 0,       /* n = {nrows, ncols, nnz}; in = {rowptr, colind, val, x}; out = {y} */
    NEST_REGION_BATCHED_MATVEC_F32 = 1, /* n = {batch, m, n}; in = {A, x}; out = {y} */
    NEST_REGION_NESTED_STENCIL_F64 = 2  /* n = {nouter, L, 0}; in = {in, coef, w}; out = {out, visits or NULL} */
} nest_region_kind;
typedef struct {
    int32_t kind;        /* nest_region_kind */
    int32_t simdlen;     /* this region's SIMD group size: 1, 2, 4, 8, 16, 32 */
    int32_t mode;        /* NEST_MODE_SPMD / GENERIC_SMEM / GENERIC_SHFL */
    int32_t blocked;     /* 1: blocked team schedule (as NEST_F_BLOCKED), 0: cyclic */
    int64_t n[3];        /* extents (per kind, above) */
    const void *in[4];   /* device input arrays (per kind) */
    void *out[2];        /* device output arrays (per kind) */
} nest_region;
nest_status nest_region_program(const nest_desc *desc, const nest_region *regions, int32_t nregions,
                                void *stream);

/* ---- NEXT-4: comm-free row-partitioned SpMV over peer memory ----
 * Same row and x partition as nest_spmv_csr_f64_dist, but x is never gathered:
 * every rank keeps its x slice (xchunk = ceil(ncols_global / nranks) doubles) in
 * a library-owned buffer that all peers map (CUDA IPC; NVLink/NVSwitch loads),
 * and the simd lanes of the SpMV read x[c] straight from the owner's slice
 * (owner = c / xchunk).  Ordering between ranks uses a flag barrier in peer
 * memory (system-scope release/acquire), no NCCL.  Results are bit-identical to
 * the single-GPU kernel at the same (simdlen, mode, variant) (R16).
 *
 * Set-up (collective over the ranks, in this order):
 *   nest_xpeer_create(nranks, rank, ncols_global, &xp, handle)  -> this rank's
 *       handle blob (nest_xpeer_handle_bytes() bytes: IPC handles of its x slice
 *       and barrier flags);
 *   the caller all-gathers the blobs (e.g. torch.distributed), rank order;
 *   nest_xpeer_open(xp, all_blobs)  -> maps every peer's slice and flags.
 * The current device must be the rank's GPU; peers on other GPUs need P2P
 * access (NVLink), which nest_xpeer_open enables. */
typedef struct nest_xpeer nest_xpeer;
size_t nest_xpeer_handle_bytes(void);
nest_status nest_xpeer_create(int32_t nranks, int32_t rank, int64_t ncols_global, nest_xpeer **out,
                              uint8_t *handle /* [nest_xpeer_handle_bytes()] */);
nest_status nest_xpeer_open(nest_xpeer *xp, const uint8_t *all_handles /* [nranks][handle_bytes] */);
/* Single-process form (tests, or one process driving several slices): `slices`
 * is a HOST array of nranks device pointers to the ranks' x slices (xchunk
 * doubles each, caller-owned, readable from the current device).  No barrier:
 * the caller orders writes to the slices against the SpMV. */
nest_status nest_xpeer_create_local(int32_t nranks, int32_t rank, int64_t ncols_global,
                                    const double *const *slices, nest_xpeer **out);
/* Device pointer of this rank's x slice (xchunk doubles; the caller writes its
 * part of x here, entries past ncols_global on the tail rank are never read). */
double *nest_xpeer_local_x(nest_xpeer *xp);
int64_t nest_xpeer_xchunk(const nest_xpeer *xp);
/* Stream-ordered device-to-device copy of min(n, slice length) doubles from
 * x_local (device) into this rank's slice; slice length = min(xchunk,
 * ncols_global - rank*xchunk).  IPC form only. */
nest_status nest_xpeer_set_x(nest_xpeer *xp, const double *x_local, int64_t n, void *stream);
/* Stream-ordered barrier over the ranks (all prior work of every rank on its
 * stream, including writes to its x slice, is visible to all peers after it). */
nest_status nest_xpeer_barrier(nest_xpeer *xp, void *stream);
/* barrier; y_local = A[local rows] x with peer gathers of x; barrier (so the
 * caller may overwrite its slice on return).  Arguments as
 * nest_spmv_csr_f64_dist (GLOBAL column indices, 0-based local rowptr).
 * Variants: the cyclic / blocked schedules, scalar or 128-bit pair loads
 * (NEST_F_VEC128 without NEST_F_VEC_QUAD); x_halo and NEST_MODE_TEAMS_GENERIC
 * return NEST_ERR_UNSUPPORTED. */
nest_status nest_spmv_csr_f64_xpeer(const nest_desc *desc, nest_xpeer *xp, int64_t nrows_global,
                                    int64_t nrows_local, int64_t nnz_local, const int64_t *rowptr_local,
                                    const int32_t *colind, const double *val, double *y_local,
                                    void *stream);
nest_status nest_xpeer_destroy(nest_xpeer *xp);

/* ---- NEXT-4b: symmetric x -- every rank's slice of x mapped into ONE virtual range ----
 * The peer-gather SpMV above looks up the owner of each far column and loads that
 * rank's slice pointer (a division and a dependent load per gather: +21-79% on one
 * GPU, profiles/r02s3_x_l2_persist.md §12).  Here each rank's x slice is a CUDA
 * virtual-memory allocation (cuMemCreate) exported as a POSIX file descriptor;
 * every rank imports the others' descriptors and maps all slices back to back, so
 * global column j is at nest_xsym_x(xs)[j] on every rank and the row-partitioned
 * SpMV is the ordinary nest_spmv_csr_f64 on that pointer (rows = the rank's shard,
 * 0-based rowptr, GLOBAL column indices; any variant), its remote columns read
 * from the owners' memory over NVLink / NVSwitch.  Slices hold xchunk columns each,
 * xchunk = ceil(ncols / nranks) rounded up to the allocation granularity (so the
 * slices tile x exactly); rank r owns columns [r*xchunk, (r+1)*xchunk) and writes
 * them through nest_xsym_local_x.  Ordering is the caller's: the writes of every
 * rank's slice must complete (stream sync + a process barrier) before any rank's
 * SpMV, and the SpMVs before a slice is rewritten.  Driver entry points are resolved
 * at run time (NEST_ERR_UNSUPPORTED without them).
 *   nest_xsym_create(nranks, rank, ncols, &xs, &fd): this rank's slice, its FD;
 *   the caller passes every FD to every other rank (e.g. SCM_RIGHTS on a unix socket);
 *   nest_xsym_open(xs, fds[nranks]): import and map (fds[rank] ignored; the caller
 *   may close the received descriptors afterwards).
 * nest_xsym_create_local: single process, nranks slices on the current device
 * mapped the same way (tests, or one process driving several slices). */
typedef struct nest_xsym nest_xsym;
nest_status nest_xsym_create(int32_t nranks, int32_t rank, int64_t ncols_global, nest_xsym **out,
                             int32_t *fd_out);
nest_status nest_xsym_open(nest_xsym *xs, const int32_t *fds /* [nranks] */);
nest_status nest_xsym_create_local(int32_t nranks, int64_t ncols_global, nest_xsym **out);
/* The contiguous x (device pointer; NULL before open) and this rank's slice of it. */
double *nest_xsym_x(nest_xsym *xs);
double *nest_xsym_local_x(nest_xsym *xs);
int64_t nest_xsym_xchunk(const nest_xsym *xs);
/* Stream-ordered device-to-device copy of min(n, xchunk) doubles from src into rank
 * `rank`'s slice (columns [rank*xchunk, ...)); multi-process form: the own rank only. */
nest_status nest_xsym_set_x(nest_xsym *xs, int32_t rank, const double *src, int64_t n, void *stream);
/* Synchronises the device, unmaps and releases. */
nest_status nest_xsym_destroy(nest_xsym *xs);

/* Release library-owned device scratch of the current device; if a
 * NEST_F_X_L2_PERSIST call raised the device's persisting-L2 limit, return the
 * persisting lines to normal and restore the limit it found. */
nest_status nest_shutdown(void);

#ifdef __cplusplus
}
#endif

#endif /* NEST_H */
