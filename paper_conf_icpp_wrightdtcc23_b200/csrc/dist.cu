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

// a12's exchange step on its own (timed separately by bench.py): x_full[r*xchunk ..]
// = rank r's x_local, over NCCL (NVLink / NVSwitch).
NEST_API nest_status nest_comm_allgather_x(nest_comm* c, const double* x_local, double* x_full, int64_t xchunk,
                                           void* stream) {
    if (!c) return fail(NEST_ERR_INVALID_ARG, "comm is NULL");
    if (xchunk < 0 || (xchunk > 0 && (!x_local || !x_full))) return fail(NEST_ERR_INVALID_ARG, "bad x buffers");
    if (xchunk == 0) return NEST_OK;
    const ncclResult_t r = ncclAllGather(x_local, x_full, (size_t)xchunk, ncclDouble, c->comm,
                                         reinterpret_cast<cudaStream_t>(stream));
    return r == ncclSuccess ? NEST_OK : nccl_fail(r, "ncclAllGather(x)");
}

static size_t a256(size_t b) { return (b + 255) & ~(size_t)255; }

NEST_API size_t nest_spmv_dist_hostio_workspace_bytes(int64_t nrows_local, int64_t nnz_local, int64_t xchunk,
                                                      int32_t nranks) {
    if (nrows_local < 0 || nnz_local < 0 || xchunk < 0 || nranks <= 0) return 0;
    return a256((size_t)(nrows_local + 1) * 8) + a256((size_t)nnz_local * 4) + a256((size_t)nnz_local * 8) +
           a256((size_t)xchunk * 8) + a256((size_t)xchunk * nranks * 8) + a256((size_t)nrows_local * 8);
}

// a12 end to end from HOST buffers: the rank's CSR shard and x slice cross PCIe
// into the workspace, x is all-gathered, the local SpMV runs, y_local returns.
NEST_API nest_status nest_spmv_csr_f64_dist_hostio(const nest_desc* desc, nest_comm* c, int64_t nrows_global,
                                                   int64_t ncols_global, int64_t nrows_local, int64_t nnz_local,
                                                   const int64_t* h_rowptr, const int32_t* h_colind,
                                                   const double* h_val, const double* h_x_local, double* h_y,
                                                   void* d_workspace, size_t workspace_bytes, void* stream) {
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
    nest_plan_info info;
    nest_status s = nest_spmv_plan(desc, nrows_local, ncols_global, nnz_local, &info);
    if (s != NEST_OK) return s;
    const int64_t xchunk = (ncols_global + c->nranks - 1) / c->nranks;
    const size_t need = nest_spmv_dist_hostio_workspace_bytes(nrows_local, nnz_local, xchunk, c->nranks);
    if (!d_workspace || workspace_bytes < need || (reinterpret_cast<uintptr_t>(d_workspace) & 255))
        return fail(NEST_ERR_INVALID_ARG, "workspace: need %zu bytes, 256-byte aligned", need);
    if (!h_rowptr || (nrows_local > 0 && !h_y) || (nnz_local > 0 && (!h_colind || !h_val)) ||
        (xchunk > 0 && !h_x_local))
        return fail(NEST_ERR_INVALID_ARG, "host buffer is NULL");
    if (h_rowptr[0] != 0 || h_rowptr[nrows_local] != nnz_local)
        return fail(NEST_ERR_INVALID_ARG, "rowptr_local must run from 0 to nnz_local");
    unsigned char* w = static_cast<unsigned char*>(d_workspace);
    int64_t* d_rp = reinterpret_cast<int64_t*>(w);
    w += a256((size_t)(nrows_local + 1) * 8);
    int32_t* d_col = reinterpret_cast<int32_t*>(w);
    w += a256((size_t)nnz_local * 4);
    double* d_val = reinterpret_cast<double*>(w);
    w += a256((size_t)nnz_local * 8);
    double* d_xl = reinterpret_cast<double*>(w);
    w += a256((size_t)xchunk * 8);
    double* d_xf = reinterpret_cast<double*>(w);
    w += a256((size_t)xchunk * c->nranks * 8);
    double* d_y = reinterpret_cast<double*>(w);
    cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
    cudaError_t ce;
    if ((ce = cudaMemcpyAsync(d_rp, h_rowptr, (size_t)(nrows_local + 1) * 8, cudaMemcpyHostToDevice, st)) ||
        (nnz_local && (ce = cudaMemcpyAsync(d_col, h_colind, (size_t)nnz_local * 4, cudaMemcpyHostToDevice, st))) ||
        (nnz_local && (ce = cudaMemcpyAsync(d_val, h_val, (size_t)nnz_local * 8, cudaMemcpyHostToDevice, st))) ||
        (xchunk && (ce = cudaMemcpyAsync(d_xl, h_x_local, (size_t)xchunk * 8, cudaMemcpyHostToDevice, st))))
        return cuda_fail(ce, "host->device copy");
    if ((s = nest_spmv_csr_f64_dist(desc, c, nrows_global, ncols_global, nrows_local, nnz_local, d_rp, d_col, d_val,
                                    d_xl, d_xf, d_y, stream)) != NEST_OK)
        return s;
    if (nrows_local && (ce = cudaMemcpyAsync(h_y, d_y, (size_t)nrows_local * 8, cudaMemcpyDeviceToHost, st)))
        return cuda_fail(ce, "device->host copy");
    return NEST_OK;
}
