// getrf.cu -- host driver of hot-path row a3 (kernels: getrf_fast.cuh,
// instantiated per (dtype, size class) in getrf_inst.cu so they compile in
// parallel).
#include "getrf_fast.cuh"

namespace bj {

template <typename R, int MLO, int MHI>
bj_status launch_getrf_fast(R *A, const int64_t *val_off, const int64_t *vec_off, int32_t *piv, int32_t *info,
                            const PlanView &p, int32_t *safe_list, unsigned *safe_count, cudaStream_t s);

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
                    const PlanView &p, const int32_t *sizes, cudaStream_t s) {
    if (p.nblocks == 0) return BJ_OK;
    char *scratch = nullptr;
    BJ_CUDA_TRY(cudaMallocAsync((void **)&scratch, 16 + sizeof(int32_t) * (size_t)p.nblocks, s));
    // the scratch is released (stream-ordered) on every return path
    struct Free {
        char *p;
        cudaStream_t s;
        ~Free() { cudaFreeAsync(p, s); }
    } guard{scratch, s};
    unsigned *safe_count = reinterpret_cast<unsigned *>(scratch);
    int32_t *safe_list = reinterpret_cast<int32_t *>(scratch + 16);
    BJ_CUDA_TRY(cudaMemsetAsync(safe_count, 0, sizeof(unsigned), s));
    bj_status st;
    // orders 32..17: one kernel per order (each gets the register allocation of
    // its own order; chained by programmatic dependent launch), then the
    // sub-warp classes.
#define BJ_GETRF_M(M) \
    if ((st = launch_getrf_fast<R, M, M>(A, val_off, vec_off, piv, info, p, safe_list, safe_count, s)) != BJ_OK) return st;
    BJ_GETRF_M(32) BJ_GETRF_M(31) BJ_GETRF_M(30) BJ_GETRF_M(29) BJ_GETRF_M(28) BJ_GETRF_M(27) BJ_GETRF_M(26)
    BJ_GETRF_M(25) BJ_GETRF_M(24) BJ_GETRF_M(23) BJ_GETRF_M(22) BJ_GETRF_M(21) BJ_GETRF_M(20) BJ_GETRF_M(19)
    BJ_GETRF_M(18) BJ_GETRF_M(17)
#undef BJ_GETRF_M
    if ((st = launch_getrf_fast<R, 9, 16>(A, val_off, vec_off, piv, info, p, safe_list, safe_count, s)) != BJ_OK) return st;
    if ((st = launch_getrf_fast<R, 5, 8>(A, val_off, vec_off, piv, info, p, safe_list, safe_count, s)) != BJ_OK) return st;
    if ((st = launch_getrf_fast<R, 1, 4>(A, val_off, vec_off, piv, info, p, safe_list, safe_count, s)) != BJ_OK) return st;
    k_getrf_safe<R><<<sm_count() * 2, 128, 0, s>>>(A, sizes, val_off, vec_off, piv, info, safe_list, safe_count);
    BJ_LAUNCH_CHECK();
    k_info_trivial<<<sm_count(), 256, 0, s>>>(info, p.order, p.bin_start);
    BJ_LAUNCH_CHECK();
    return BJ_OK;
}

template bj_status getrf_run<double>(double *, const int64_t *, const int64_t *, int32_t *, int32_t *,
                                     const PlanView &, const int32_t *, cudaStream_t);
template bj_status getrf_run<float>(float *, const int64_t *, const int64_t *, int32_t *, int32_t *,
                                    const PlanView &, const int32_t *, cudaStream_t);

}  // namespace bj
