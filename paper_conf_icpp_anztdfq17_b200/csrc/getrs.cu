// getrs.cu -- host driver of hot-path rows a4/a5 (kernels: getrs_kernels.cuh,
// instantiated per (dtype, size class) in getrs_inst.cu).
#include "common.cuh"
#include "internal.h"

namespace bj {

template <typename R, int MLO, int MHI>
bj_status launch_getrs_class(const R *LU, const int64_t *val_off, const int64_t *vec_off, const int32_t *piv,
                             const R *b, R *x, const PlanView &p, cudaStream_t s);

template <typename R>
bj_status getrs_run(const R *LU, const int64_t *val_off, const int64_t *vec_off, const int32_t *piv,
                    const R *b, R *x, const PlanView &p, cudaStream_t s) {
    if (p.nblocks == 0) return BJ_OK;
    bj_status st;
    if ((st = launch_getrs_class<R, 17, 32>(LU, val_off, vec_off, piv, b, x, p, s)) != BJ_OK) return st;
    if ((st = launch_getrs_class<R, 9, 16>(LU, val_off, vec_off, piv, b, x, p, s)) != BJ_OK) return st;
    if ((st = launch_getrs_class<R, 5, 8>(LU, val_off, vec_off, piv, b, x, p, s)) != BJ_OK) return st;
    if ((st = launch_getrs_class<R, 1, 4>(LU, val_off, vec_off, piv, b, x, p, s)) != BJ_OK) return st;
    return BJ_OK;
}

template bj_status getrs_run<double>(const double *, const int64_t *, const int64_t *, const int32_t *,
                                     const double *, double *, const PlanView &, cudaStream_t);
template bj_status getrs_run<float>(const float *, const int64_t *, const int64_t *, const int32_t *,
                                    const float *, float *, const PlanView &, cudaStream_t);

}  // namespace bj
