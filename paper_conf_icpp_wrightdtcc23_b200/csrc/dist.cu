// dist.cu -- a12: row-partitioned multi-GPU SpMV (north_star; the paper is
// single-GPU).  One process per GPU; a library-owned NCCL
// communicator bootstrapped from a unique id the caller broadcasts (e.g. with
// torch.distributed).  Each call all-gathers x over NVLink into x_full, then
// runs the local rows through the same three-level SpMV on the same stream.
#include <nccl.h>

#include <cstring>
#include <new>

#include "internal.h"

struct nest_comm {
    ncclComm_t comm = nullptr;
    int32_t nranks = 0;
    int32_t rank = 0;
};

using namespace nest;

static nest_status nccl_fail(ncclResult_t r, const char* what) {
    return fail(NEST_ERR_NCCL, "%s: %s", what, ncclGetErrorString(r));
}

NEST_API nest_status nest_comm_unique_id(uint8_t out[128]) {
    if (!out) return fail(NEST_ERR_INVALID_ARG, "out is NULL");
    static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId is 128 bytes");
    ncclUniqueId id;
    const ncclResult_t r = ncclGetUniqueId(&id);
    if (r != ncclSuccess) return nccl_fail(r, "ncclGetUniqueId");
    std::memcpy(out, &id, sizeof(id));
    return NEST_OK;
}

NEST_API nest_status nest_comm_init(const uint8_t id[128], int32_t nranks, int32_t rank,
                                    nest_comm** out) {
    if (!id || !out || nranks <= 0 || rank < 0 || rank >= nranks)
        return fail(NEST_ERR_INVALID_ARG, "bad comm arguments (nranks %d, rank %d)", nranks, rank);
    ncclUniqueId uid;
    std::memcpy(&uid, id, sizeof(uid));
    nest_comm* c = new (std::nothrow) nest_comm;
    if (!c) return fail(NEST_ERR_NO_MEMORY, "nest_comm");
    const ncclResult_t r = ncclCommInitRank(&c->comm, nranks, uid, rank);
    if (r != ncclSuccess) {
        delete c;
        return nccl_fail(r, "ncclCommInitRank");
    }
    c->nranks = nranks;
    c->rank = rank;
    *out = c;
    return NEST_OK;
}

NEST_API nest_status nest_comm_destroy(nest_comm* c) {
    if (!c) return NEST_OK;
    const ncclResult_t r = ncclCommDestroy(c->comm);
    delete c;
    return r == ncclSuccess ? NEST_OK : nccl_fail(r, "ncclCommDestroy");
}

NEST_API nest_status nest_spmv_csr_f64_dist(const nest_desc* desc, nest_comm* c,
                                            int64_t nrows_global, int64_t ncols_global,
                                            int64_t nrows_local, int64_t nnz_local,
                                            const int64_t* rowptr_local, const int32_t* colind,
                                            const double* val, const double* x_local,
                                            double* x_full, double* y_local, void* stream) {
    if (!c) return fail(NEST_ERR_INVALID_ARG, "comm is NULL");
    if (nrows_global < 0 || ncols_global < 0 || nrows_local < 0 || nnz_local < 0)
        return fail(NEST_ERR_INVALID_ARG, "negative extent");
    const int64_t chunk = (nrows_global + c->nranks - 1) / c->nranks;
    int64_t b = (int64_t)c->rank * chunk;
    if (b > nrows_global) b = nrows_global;
    const int64_t e = b + chunk < nrows_global ? b + chunk : nrows_global;
    if (nrows_local != e - b)
        return fail(NEST_ERR_INVALID_ARG, "rank %d owns %lld rows, got nrows_local %lld", c->rank,
                    (long long)(e - b), (long long)nrows_local);
    const int64_t xchunk = (ncols_global + c->nranks - 1) / c->nranks;
    if (xchunk > 0 && (!x_local || !x_full)) return fail(NEST_ERR_INVALID_ARG, "x_local/x_full is NULL");
    // validate the local launch before enqueuing the collective (no side effects on error)
    nest_plan_info info;
    nest_status s = nest_spmv_plan(desc, nrows_local, ncols_global, nnz_local, &info);
    if (s != NEST_OK) return s;
    if (nrows_local > 0 && (!rowptr_local || !y_local)) return fail(NEST_ERR_INVALID_ARG, "rowptr/y is NULL");
    if (nnz_local > 0 && (!colind || !val)) return fail(NEST_ERR_INVALID_ARG, "colind/val is NULL");
    cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
    if (xchunk > 0) {
        const ncclResult_t r =
            ncclAllGather(x_local, x_full, (size_t)xchunk, ncclDouble, c->comm, st);
        if (r != ncclSuccess) return nccl_fail(r, "ncclAllGather(x)");
    }
    return nest_spmv_csr_f64(desc, nrows_local, ncols_global, nnz_local, rowptr_local, colind, val,
                             x_full, y_local, stream);
}
