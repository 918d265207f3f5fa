// getrf.cu -- host driver of hot-path row a3 (kernels: getrf_fast.cuh,
// instantiated per (dtype, order range) in getrf_inst.cu so they compile in
// parallel), and of the fused factor + solve (bj_gesv_vbatched).
#include "getrf_fast.cuh"

namespace bj {

template <typename R, int MLO, int MHI, bool SOLVE>
bj_status launch_getrf_fast(R *A, const int64_t *val_off, const int64_t *vec_off, int32_t *piv, int32_t *info,
                            const PlanView &p, int32_t *safe_list, unsigned *safe_count, const R *b, R *x,
                            cudaStream_t s);

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

// GETRF over a plan; with b != nullptr also the fused solve x = A^{-1} b
// (bit-identical to getrf_run followed by getrs_run).
template <typename R, bool SOLVE>
static bj_status getrf_solve_run(R *A, const int64_t *val_off, const int64_t *vec_off, int32_t *piv, int32_t *info,
                                 const PlanView &p, const int32_t *sizes, const R *b, R *x, cudaStream_t s) {
    if (p.nblocks == 0) return BJ_OK;
    AsyncScratch scratch(s);                 // released (stream-ordered) on every return path
    BJ_CUDA_TRY(cudaMallocAsync((void **)&scratch.p, 16 + sizeof(int32_t) * (size_t)p.nblocks, s));
    unsigned *safe_count = reinterpret_cast<unsigned *>(scratch.p);
    int32_t *safe_list = reinterpret_cast<int32_t *>(scratch.p + 16);
    BJ_CUDA_TRY(cudaMemsetAsync(safe_count, 0, sizeof(unsigned), s));
    bj_status st;
    // orders 32..17: one kernel per order (each gets the register allocation of
    // its own order; chained by programmatic dependent launch), then the
    // sub-warp classes.
#define BJ_GETRF_C(LO, HI)                                                                                  \
    if ((st = launch_getrf_fast<R, LO, HI, SOLVE>(A, val_off, vec_off, piv, info, p, safe_list, safe_count, b, \
                                                  x, s)) != BJ_OK)                                           \
        return st;
    BJ_GETRF_C(32, 32) BJ_GETRF_C(31, 31) BJ_GETRF_C(30, 30) BJ_GETRF_C(29, 29) BJ_GETRF_C(28, 28)
    BJ_GETRF_C(27, 27) BJ_GETRF_C(26, 26) BJ_GETRF_C(25, 25) BJ_GETRF_C(24, 24) BJ_GETRF_C(23, 23)
    BJ_GETRF_C(22, 22) BJ_GETRF_C(21, 21) BJ_GETRF_C(20, 20) BJ_GETRF_C(19, 19) BJ_GETRF_C(18, 18)
    BJ_GETRF_C(17, 17) BJ_GETRF_C(9, 16) BJ_GETRF_C(5, 8) BJ_GETRF_C(1, 4)
#undef BJ_GETRF_C
    k_getrf_safe<R><<<persistent_grid(k_getrf_safe<R>, 128), 128, 0, s>>>(A, sizes, val_off, vec_off, piv, info,
                                                                           safe_list, safe_count, b, x);
    BJ_LAUNCH_CHECK();
    k_info_trivial<<<sm_count(), 256, 0, s>>>(info, p.order, p.bin_start);
    BJ_LAUNCH_CHECK();
    return BJ_OK;
}

bj_status info_trivial_run(int32_t *info, const PlanView &p, cudaStream_t s) {
    k_info_trivial<<<sm_count(), 256, 0, s>>>(info, p.order, p.bin_start);
    BJ_LAUNCH_CHECK();
    return BJ_OK;
}

template <typename R, int M>
bj_status launch_setup_fused(const bj_csr &Acsr, const int32_t *block_ptr, R *A, const int64_t *val_off,
                             const int64_t *vec_off, int32_t *piv, int32_t *info, const PlanView &p,
                             int32_t *safe_list, unsigned *safe_count, cudaStream_t s);

// NEXT(1): setup = extraction of the blocks of order <= 16 (and of blocks
// with more than kHeavy entries) into `out`, then the fused extract + GETRF
// kernels for orders 32..17 (no dense round trip through HBM), then the
// GETRF classes 1-16 and the safe path -- outputs bit-identical to
// extract_run + getrf_run.
template <typename R>
bj_status setup_run(const bj_csr &Acsr, const int32_t *block_ptr, R *A, const int64_t *val_off,
                    const int64_t *vec_off, int32_t *piv, int32_t *info, const PlanView &p, const int32_t *sizes,
                    cudaStream_t s) {
    if (p.nblocks == 0) return BJ_OK;
    bj_status st;
    if ((st = extract_run<R>(Acsr, block_ptr, p.nblocks, val_off, A, s, 17)) != BJ_OK) return st;
    AsyncScratch scratch(s);
    BJ_CUDA_TRY(cudaMallocAsync((void **)&scratch.p, 16 + sizeof(int32_t) * (size_t)p.nblocks, s));
    unsigned *safe_count = reinterpret_cast<unsigned *>(scratch.p);
    int32_t *safe_list = reinterpret_cast<int32_t *>(scratch.p + 16);
    BJ_CUDA_TRY(cudaMemsetAsync(safe_count, 0, sizeof(unsigned), s));
#define BJ_FUSED_M(M)                                                                                      \
    if ((st = launch_setup_fused<R, M>(Acsr, block_ptr, A, val_off, vec_off, piv, info, p, safe_list,       \
                                       safe_count, s)) != BJ_OK)                                           \
        return st;
    BJ_FUSED_M(32) BJ_FUSED_M(31) BJ_FUSED_M(30) BJ_FUSED_M(29) BJ_FUSED_M(28) BJ_FUSED_M(27) BJ_FUSED_M(26)
    BJ_FUSED_M(25) BJ_FUSED_M(24) BJ_FUSED_M(23) BJ_FUSED_M(22) BJ_FUSED_M(21) BJ_FUSED_M(20) BJ_FUSED_M(19)
    BJ_FUSED_M(18) BJ_FUSED_M(17)
#undef BJ_FUSED_M
#define BJ_GETRF_C(LO, HI)                                                                                  \
    if ((st = launch_getrf_fast<R, LO, HI, false>(A, val_off, vec_off, piv, info, p, safe_list, safe_count,  \
                                                  nullptr, nullptr, s)) != BJ_OK)                            \
        return st;
    BJ_GETRF_C(9, 16) BJ_GETRF_C(5, 8) BJ_GETRF_C(1, 4)
#undef BJ_GETRF_C
    k_getrf_safe<R><<<persistent_grid(k_getrf_safe<R>, 128), 128, 0, s>>>(A, sizes, val_off, vec_off, piv, info,
                                                                           safe_list, safe_count);
    BJ_LAUNCH_CHECK();
    k_info_trivial<<<sm_count(), 256, 0, s>>>(info, p.order, p.bin_start);
    BJ_LAUNCH_CHECK();
    return BJ_OK;
}

template bj_status setup_run<double>(const bj_csr &, const int32_t *, double *, const int64_t *, const int64_t *,
                                     int32_t *, int32_t *, const PlanView &, const int32_t *, cudaStream_t);
template bj_status setup_run<float>(const bj_csr &, const int32_t *, float *, const int64_t *, const int64_t *,
                                    int32_t *, int32_t *, const PlanView &, const int32_t *, cudaStream_t);

template <typename R>
bj_status getrf_run(R *A, const int64_t *val_off, const int64_t *vec_off, int32_t *piv, int32_t *info,
                    const PlanView &p, const int32_t *sizes, cudaStream_t s) {
    return getrf_solve_run<R, false>(A, val_off, vec_off, piv, info, p, sizes, nullptr, nullptr, s);
}

template <typename R>
bj_status gesv_run(R *A, const int64_t *val_off, const int64_t *vec_off, int32_t *piv, int32_t *info,
                   const PlanView &p, const int32_t *sizes, const R *b, R *x, cudaStream_t s) {
    return getrf_solve_run<R, true>(A, val_off, vec_off, piv, info, p, sizes, b, x, s);
}

template bj_status gesv_run<double>(double *, const int64_t *, const int64_t *, int32_t *, int32_t *,
                                    const PlanView &, const int32_t *, const double *, double *, cudaStream_t);
template bj_status gesv_run<float>(float *, const int64_t *, const int64_t *, int32_t *, int32_t *,
                                   const PlanView &, const int32_t *, const float *, float *, cudaStream_t);
template bj_status getrf_run<double>(double *, const int64_t *, const int64_t *, int32_t *, int32_t *,
                                     const PlanView &, const int32_t *, cudaStream_t);
template bj_status getrf_run<float>(float *, const int64_t *, const int64_t *, int32_t *, int32_t *,
                                    const PlanView &, const int32_t *, cudaStream_t);

}  // namespace bj
