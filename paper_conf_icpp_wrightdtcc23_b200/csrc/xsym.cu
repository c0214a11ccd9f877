// xsym.cu -- NEXT-4b: the distributed x as ONE virtual range (symmetric x).
//
// The peer-gather SpMV (xpeer.cu) finds the owner of a column and loads that
// rank's slice pointer for every far gather; on one GPU that lookup alone costs
// 21-79% (profiles/r02s3_x_l2_persist.md §12).  Here every rank's x slice is a
// CUDA virtual-memory allocation (cuMemCreate) exported as a POSIX file
// descriptor; each rank imports the others' and maps all of them back to back
// into one reserved range, so global column j is at x[j] on every rank and the
// SpMV is the ordinary kernel (any variant: quads, the persisting window...),
// its remote columns loads from the owners' memory over NVLink/NVSwitch.
// Driver entry points are resolved at run time (cudaGetDriverEntryPointByVersion):
// libnest.so keeps no link-time dependency on libcuda.
#include <cuda.h>
#include <cuda_runtime.h>
#include <unistd.h>

#include <cstdint>
#include <vector>

#include "internal.h"

namespace nest {
namespace {

struct Drv {
    decltype(&cuMemCreate) create = nullptr;
    decltype(&cuMemRelease) release = nullptr;
    decltype(&cuMemMap) map = nullptr;
    decltype(&cuMemUnmap) unmap = nullptr;
    decltype(&cuMemSetAccess) set_access = nullptr;
    decltype(&cuMemAddressReserve) reserve = nullptr;
    decltype(&cuMemAddressFree) addr_free = nullptr;
    decltype(&cuMemExportToShareableHandle) export_handle = nullptr;
    decltype(&cuMemImportFromShareableHandle) import_handle = nullptr;
    decltype(&cuMemGetAllocationGranularity) granularity = nullptr;
    bool ok = false;
};

template <class F>
bool resolve(const char* name, F& f) {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPointByVersion(name, &p, 12000, cudaEnableDefault, &q) != cudaSuccess ||
        q != cudaDriverEntryPointSuccess || !p) {
        cudaGetLastError();
        return false;
    }
    f = reinterpret_cast<F>(p);
    return true;
}

const Drv& drv() {
    static const Drv d = [] {
        Drv r;
        r.ok = resolve("cuMemCreate", r.create) && resolve("cuMemRelease", r.release) &&
               resolve("cuMemMap", r.map) && resolve("cuMemUnmap", r.unmap) &&
               resolve("cuMemSetAccess", r.set_access) && resolve("cuMemAddressReserve", r.reserve) &&
               resolve("cuMemAddressFree", r.addr_free) &&
               resolve("cuMemExportToShareableHandle", r.export_handle) &&
               resolve("cuMemImportFromShareableHandle", r.import_handle) &&
               resolve("cuMemGetAllocationGranularity", r.granularity);
        return r;
    }();
    return d;
}

nest_status cu_fail(CUresult r, const char* what) {
    return fail(NEST_ERR_CUDA, "%s: CUresult %d", what, (int)r);
}

CUmemAllocationProp alloc_prop(int dev, bool exportable) {
    CUmemAllocationProp p = {};
    p.type = CU_MEM_ALLOCATION_TYPE_PINNED;
    p.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
    p.location.id = dev;
    p.requestedHandleTypes = exportable ? CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR : CU_MEM_HANDLE_TYPE_NONE;
    return p;
}

}  // namespace
}  // namespace nest

using namespace nest;

struct nest_xsym {
    int32_t nranks = 0, rank = 0;
    int64_t ncols = 0, xchunk = 0;   // columns per rank (slice bytes / 8)
    size_t slice_bytes = 0;
    size_t gran = 0;   // allocation granularity (the reservation's alignment)
    int dev = 0;
    std::vector<CUmemGenericAllocationHandle> handles;   // [nranks]; 0 = not yet imported
    CUdeviceptr base = 0;
    bool mapped = false, local = false;
};

static nest_status xsym_plan(int32_t nranks, int32_t rank, int64_t ncols, bool exportable, nest_xsym* xs) {
    if (nranks < 1 || rank < 0 || rank >= nranks || ncols < 0)
        return fail(NEST_ERR_INVALID_ARG, "nranks %d, rank %d, ncols %lld", nranks, rank, (long long)ncols);
    if (!drv().ok) return fail(NEST_ERR_UNSUPPORTED, "CUDA virtual-memory driver entry points unavailable");
    cudaError_t e = cudaGetDevice(&xs->dev);
    if (e != cudaSuccess) return cuda_fail(e, "cudaGetDevice");
    const CUmemAllocationProp prop = alloc_prop(xs->dev, exportable);
    size_t gran = 0;
    CUresult r = drv().granularity(&gran, &prop, CU_MEM_ALLOC_GRANULARITY_RECOMMENDED);
    if (r != CUDA_SUCCESS) return cu_fail(r, "cuMemGetAllocationGranularity");
    // every rank owns a whole number of granules of columns, so the slices tile x exactly
    const int64_t per = (ncols + nranks - 1) / nranks;
    const size_t cols_per_gran = gran / 8;
    xs->xchunk = (int64_t)(((size_t)(per > 0 ? per : 1) + cols_per_gran - 1) / cols_per_gran * cols_per_gran);
    xs->slice_bytes = (size_t)xs->xchunk * 8;
    xs->gran = gran;
    xs->nranks = nranks;
    xs->rank = rank;
    xs->ncols = ncols;
    xs->handles.assign(nranks, 0);
    return NEST_OK;
}

static nest_status xsym_map(nest_xsym* xs) {
    const size_t total = xs->slice_bytes * (size_t)xs->nranks;
    CUresult r = drv().reserve(&xs->base, total, xs->gran, 0, 0);   // alignment: a power of two
    if (r != CUDA_SUCCESS) {
        xs->base = 0;
        return cu_fail(r, "cuMemAddressReserve");
    }
    int32_t done = 0;
    const char* what = nullptr;
    for (; done < xs->nranks; ++done) {
        r = drv().map(xs->base + (CUdeviceptr)(xs->slice_bytes * (size_t)done), xs->slice_bytes, 0,
                      xs->handles[done], 0);
        if (r != CUDA_SUCCESS) {
            what = "cuMemMap";
            break;
        }
    }
    if (!what) {
        CUmemAccessDesc acc = {};
        acc.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
        acc.location.id = xs->dev;
        acc.flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
        r = drv().set_access(xs->base, total, &acc, 1);
        if (r == CUDA_SUCCESS) {
            xs->mapped = true;
            return NEST_OK;
        }
        what = "cuMemSetAccess";
    }
    // undo: the slices mapped so far, then the reservation (destroy then only releases handles)
    for (int32_t q = 0; q < done; ++q) drv().unmap(xs->base + (CUdeviceptr)(xs->slice_bytes * (size_t)q), xs->slice_bytes);
    drv().addr_free(xs->base, total);
    xs->base = 0;
    return cu_fail(r, what);
}

NEST_API nest_status nest_xsym_destroy(nest_xsym* xs) {
    if (!xs) return NEST_OK;
    nest_status s = NEST_OK;
    if (xs->base) {
        cudaDeviceSynchronize();   // no kernel may still read the range
        const size_t total = xs->slice_bytes * (size_t)xs->nranks;
        if (xs->mapped) drv().unmap(xs->base, total);
        if (drv().addr_free(xs->base, total) != CUDA_SUCCESS) s = fail(NEST_ERR_CUDA, "cuMemAddressFree");
    }
    for (CUmemGenericAllocationHandle h : xs->handles)
        if (h) drv().release(h);
    delete xs;
    return s;
}

NEST_API nest_status nest_xsym_create(int32_t nranks, int32_t rank, int64_t ncols_global, nest_xsym** out,
                                      int32_t* fd_out) {
    if (!out || !fd_out) return fail(NEST_ERR_INVALID_ARG, "out/fd_out is NULL");
    *out = nullptr;
    nest_xsym* xs = new nest_xsym;
    nest_status s = xsym_plan(nranks, rank, ncols_global, true, xs);
    if (s != NEST_OK) {
        delete xs;
        return s;
    }
    const CUmemAllocationProp prop = alloc_prop(xs->dev, true);
    CUresult r = drv().create(&xs->handles[rank], xs->slice_bytes, &prop, 0);
    if (r != CUDA_SUCCESS) {
        nest_xsym_destroy(xs);
        return cu_fail(r, "cuMemCreate");
    }
    int fd = -1;
    r = drv().export_handle(&fd, xs->handles[rank], CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR, 0);
    if (r != CUDA_SUCCESS) {
        nest_xsym_destroy(xs);
        return cu_fail(r, "cuMemExportToShareableHandle");
    }
    *fd_out = fd;
    *out = xs;
    return NEST_OK;
}

NEST_API nest_status nest_xsym_open(nest_xsym* xs, const int32_t* fds) {
    if (!xs || !fds || xs->local || xs->mapped) return fail(NEST_ERR_INVALID_ARG, "xsym is NULL, local or open");
    for (int32_t q = 0; q < xs->nranks; ++q) {
        if (q == xs->rank) continue;
        CUresult r = drv().import_handle(&xs->handles[q], reinterpret_cast<void*>((uintptr_t)fds[q]),
                                         CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR);
        if (r != CUDA_SUCCESS) return cu_fail(r, "cuMemImportFromShareableHandle");
    }
    return xsym_map(xs);
}

NEST_API nest_status nest_xsym_create_local(int32_t nranks, int64_t ncols_global, nest_xsym** out) {
    if (!out) return fail(NEST_ERR_INVALID_ARG, "out is NULL");
    *out = nullptr;
    nest_xsym* xs = new nest_xsym;
    nest_status s = xsym_plan(nranks, 0, ncols_global, false, xs);
    if (s != NEST_OK) {
        delete xs;
        return s;
    }
    xs->local = true;
    const CUmemAllocationProp prop = alloc_prop(xs->dev, false);
    for (int32_t q = 0; q < nranks; ++q) {
        CUresult r = drv().create(&xs->handles[q], xs->slice_bytes, &prop, 0);
        if (r != CUDA_SUCCESS) {
            nest_xsym_destroy(xs);
            return cu_fail(r, "cuMemCreate");
        }
    }
    if ((s = xsym_map(xs)) != NEST_OK) {
        nest_xsym_destroy(xs);
        return s;
    }
    *out = xs;
    return NEST_OK;
}

NEST_API double* nest_xsym_x(nest_xsym* xs) {
    return xs && xs->mapped ? reinterpret_cast<double*>(xs->base) : nullptr;
}

NEST_API double* nest_xsym_local_x(nest_xsym* xs) {
    return xs && xs->mapped ? reinterpret_cast<double*>(xs->base + (CUdeviceptr)(xs->slice_bytes * (size_t)xs->rank))
                            : nullptr;
}

NEST_API int64_t nest_xsym_xchunk(const nest_xsym* xs) { return xs ? xs->xchunk : 0; }

NEST_API nest_status nest_xsym_set_x(nest_xsym* xs, int32_t rank, const double* src, int64_t n, void* stream) {
    if (!xs || !xs->mapped) return fail(NEST_ERR_INVALID_ARG, "xsym is NULL or not open");
    if (rank < 0 || rank >= xs->nranks || n < 0 || (n > 0 && !src))
        return fail(NEST_ERR_INVALID_ARG, "rank %d, n %lld", rank, (long long)n);
    if (!xs->local && rank != xs->rank) return fail(NEST_ERR_INVALID_ARG, "only the own slice is written");
    const int64_t m = n < xs->xchunk ? n : xs->xchunk;
    if (m == 0) return NEST_OK;
    const cudaError_t e = cudaMemcpyAsync(reinterpret_cast<void*>(xs->base + (CUdeviceptr)(xs->slice_bytes * (size_t)rank)),
                                          src, (size_t)m * 8, cudaMemcpyDeviceToDevice,
                                          reinterpret_cast<cudaStream_t>(stream));
    return e == cudaSuccess ? NEST_OK : cuda_fail(e, "cudaMemcpyAsync (xsym slice)");
}
