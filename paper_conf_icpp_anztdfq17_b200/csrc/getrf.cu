// getrf.cu -- host driver of hot-path row a3 (kernels: getrf_kernels.cuh,
// instantiated per (dtype, size class) in getrf_inst.cu so they compile in
// parallel).
#include "common.cuh"
#include "internal.h"

namespace bj {

template <typename R, int MLO, int MHI>
bj_status launch_getrf_class(R *A, const int64_t *val_off, const int64_t *vec_off, int32_t *piv, int32_t *info,
                             const PlanView &p, cudaStream_t s);

// info for blocks of order 0 (nothing to factor) and of invalid order (-1).
__global__ void k_info_trivial(int32_t *__restrict__ info, const int32_t *__restrict__ order,
                               const int64_t *__restrict__ bin_start) {
    const int64_t z0 = bin_start[0], z1 = bin_start[1];
    const int64_t b0 = bin_start[kInvalidBin], b1 = bin_start[kInvalidBin + 1];
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < (z1 - z0) + (b1 - b0); i += stride) {
        if (i < z1 - z0) info[order[z0 + i]] = 0;
        else info[order[b0 + i - (z1 - z0)]] = -1;
    }
}

template <typename R>
bj_status getrf_run(R *A, const int64_t *val_off, const int64_t *vec_off, int32_t *piv, int32_t *info,
                    const PlanView &p, cudaStream_t s) {
    if (p.nblocks == 0) return BJ_OK;
    bj_status st;
    if ((st = launch_getrf_class<R, 17, 32>(A, val_off, vec_off, piv, info, p, s)) != BJ_OK) return st;
    if ((st = launch_getrf_class<R, 9, 16>(A, val_off, vec_off, piv, info, p, s)) != BJ_OK) return st;
    if ((st = launch_getrf_class<R, 5, 8>(A, val_off, vec_off, piv, info, p, s)) != BJ_OK) return st;
    if ((st = launch_getrf_class<R, 1, 4>(A, val_off, vec_off, piv, info, p, s)) != BJ_OK) return st;
    k_info_trivial<<<sm_count(), 256, 0, s>>>(info, p.order, p.bin_start);
    BJ_LAUNCH_CHECK();
    return BJ_OK;
}

template bj_status getrf_run<double>(double *, const int64_t *, const int64_t *, int32_t *, int32_t *,
                                     const PlanView &, cudaStream_t);
template bj_status getrf_run<float>(float *, const int64_t *, const int64_t *, int32_t *, int32_t *,
                                    const PlanView &, cudaStream_t);

}  // namespace bj
