// launch_spmv_teams.cu -- NEXT-1: the paper's two-level teams-generic SpMV baseline.
#include "device/teams_generic.cuh"
#include "internal.h"

namespace nest {

nest_status launch_spmv_teams_generic(const Plan& p, int64_t nrows, const int64_t* rowptr, const int32_t* col,
                                      const double* val, const double* x, double* y, cudaStream_t st) {
    const int threads = p.block + 32;   // the extra team-main warp
    switch (p.reduce) {
        case RED_SUM: spmv_teams_generic_kernel<RED_SUM><<<p.grid, threads, 0, st>>>(rowptr, col, val, x, y, nrows); break;
        case RED_MAX: spmv_teams_generic_kernel<RED_MAX><<<p.grid, threads, 0, st>>>(rowptr, col, val, x, y, nrows); break;
        case RED_MIN: spmv_teams_generic_kernel<RED_MIN><<<p.grid, threads, 0, st>>>(rowptr, col, val, x, y, nrows); break;
        default: return fail(NEST_ERR_INVALID_ARG, "reduce %d", p.reduce);
    }
    const cudaError_t e = cudaGetLastError();
    return e == cudaSuccess ? NEST_OK : cuda_fail(e, "spmv_teams_generic launch");
}

}  // namespace nest
