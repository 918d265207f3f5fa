// internal.h -- host-side interfaces between the C-ABI layer (api.cu) and the
// kernel translation units.  Not installed; not part of the C ABI.
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include "bj.h"

namespace bj {

struct PlanView;

// a1
bj_status layout_sizes(int64_t nb, const int32_t *sizes, int elem, int64_t *vec, int64_t *val,
                       cudaStream_t s);
bj_status layout_block_ptr(int64_t nb, const int32_t *bp, int elem, int32_t *sizes, int64_t *vec,
                           int64_t *val, cudaStream_t s);
bj_status build_plan(int64_t nb, const int32_t *sizes, int32_t *order, int64_t *bin_start,
                     cudaStream_t s);

// a3 / a4: launch the size-class kernels over a plan.
template <typename R>
bj_status getrf_run(R *values, const int64_t *val_off, const int64_t *vec_off, int32_t *piv,
                    int32_t *info, const PlanView &plan, const int32_t *sizes, cudaStream_t s);
template <typename R>
bj_status gesv_run(R *values, const int64_t *val_off, const int64_t *vec_off, int32_t *piv, int32_t *info,
                   const PlanView &plan, const int32_t *sizes, const R *b, R *x, cudaStream_t s);
bj_status info_trivial_run(int32_t *info, const PlanView &plan, cudaStream_t s);
// NEXT(3): inversion-based variant (getri.cu)
template <typename R>
bj_status getri_run(R *values, const int64_t *val_off, const int64_t *vec_off, int32_t *piv, int32_t *info,
                    const PlanView &plan, const int32_t *sizes, cudaStream_t s);
template <typename R>
bj_status gemv_run(const R *dinv, const int64_t *val_off, const int64_t *vec_off, const R *x, R *y,
                   const PlanView &plan, cudaStream_t s);
template <typename R>
bj_status getrs_run(const R *lu, const int64_t *val_off, const int64_t *vec_off, const int32_t *piv,
                    const R *b, R *x, const PlanView &plan, cudaStream_t s);

// a2
// mlo_skip > 0: blocks of order >= mlo_skip with at most kHeavy entries are
// left to the fused setup (setup_run)
template <typename R>
bj_status extract_run(const bj_csr &A, const int32_t *block_ptr, int64_t nb, const int64_t *val_off,
                      R *out, cudaStream_t s, int mlo_skip = 0);
// NEXT(1): block-Jacobi setup with the extraction fused into GETRF for orders
// 17..32 (setup_fused.cuh); the values of out must be laid out per block_ptr
template <typename R>
bj_status setup_run(const bj_csr &A, const int32_t *block_ptr, R *out, const int64_t *val_off,
                    const int64_t *vec_off, int32_t *piv, int32_t *info, const PlanView &plan,
                    const int32_t *sizes, cudaStream_t s);

// NEXT(2)
bj_status supervariable_run(const bj_csr &A, int32_t bound, int32_t *block_ptr, int64_t *nblocks_h,
                            cudaStream_t s);

}  // namespace bj
