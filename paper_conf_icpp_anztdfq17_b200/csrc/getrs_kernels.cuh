#pragma once
// getrs_kernels.cuh -- hot-path rows a4/a5: batched GETRS, P:218-238 steps 2-4,
// section III.B, Fig. 2 bottom (eager, column-oriented).
//
// Same size-class / tile structure as getrf.cu.  Lane r of a tile holds row r
// of L\U (read column by column: coalesced) and one element of the
// right-hand side, loaded through the permutation (b := P b while
// distributing b over the lanes).  The eager lower solve
// broadcasts y_k and every lane below applies one fused AXPY term; the upper
// solve (mirrored, R8) divides y_k by U(k,k) in lane k first.  Every y_i
// receives the same sequence of correctly rounded operations as the oracle.
#include "common.cuh"
#include "internal.h"
#include "getrs_tile.cuh"

namespace bj {

constexpr int kGetrsThreads = 128;

template <typename R, int M, int MHI>
__device__ __forceinline__ void getrs_dispatch(int m, const R *LU, const int64_t *val_off, const int64_t *vec_off,
                                               const int32_t *piv, const R *b, R *x, const int32_t *order,
                                               int64_t first, int64_t last) {
    if (m == M) {
        const int lane = threadIdx.x & 31;
        constexpr int T = tile_width(M);
        const int64_t idx = first + lane / T;
        const bool tile_ok = idx < last;
        const int blk = tile_ok ? __ldg(order + idx) : 0;
        const int64_t vo = tile_ok ? __ldg(vec_off + blk) : 0;
        const int64_t lo = tile_ok ? __ldg(val_off + blk) : 0;
        getrs_tile<R, M>(LU + lo, piv + vo, b + vo, x + vo, tile_ok);
    } else {
        if constexpr (M < MHI) getrs_dispatch<R, M + 1, MHI>(m, LU, val_off, vec_off, piv, b, x, order, first, last);
    }
}

template <typename R, int MLO, int MHI>
__global__ void __launch_bounds__(kGetrsThreads)
k_getrs_class(const R *__restrict__ LU, const int64_t *__restrict__ val_off, const int64_t *__restrict__ vec_off,
              const int32_t *__restrict__ piv, const R *b, R *x, const int32_t *__restrict__ order,
              const int64_t *__restrict__ bin_start) {
    constexpr int NM = MHI - MLO + 1;
    __shared__ int64_t s_pref[NM + 1], s_first[NM], s_last[NM];
    if (threadIdx.x == 0) {
        int64_t acc = 0;
        for (int i = 0; i < NM; ++i) {
            const int m = MLO + i;
            const int64_t b0 = bin_start[m], b1 = bin_start[m + 1];
            const int g = tiles_per_warp(m);
            s_first[i] = b0;
            s_last[i] = b1;
            s_pref[i] = acc;
            acc += (b1 - b0 + g - 1) / g;
        }
        s_pref[NM] = acc;
    }
    __syncthreads();
    const int64_t ntask = s_pref[NM];
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t task = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; task < ntask; task += nwarps) {
        int i = 0;
        while (i + 1 < NM && s_pref[i + 1] <= task) ++i;
        const int m = MLO + i;
        const int64_t first = s_first[i] + (task - s_pref[i]) * tiles_per_warp(m);
        getrs_dispatch<R, MLO, MHI>(m, LU, val_off, vec_off, piv, b, x, order, first, s_last[i]);
    }
}

template <typename R, int MLO, int MHI>
bj_status launch_getrs_class(const R *LU, const int64_t *val_off, const int64_t *vec_off, const int32_t *piv,
                              const R *b, R *x, const PlanView &p, cudaStream_t s) {
    static int grid = 0;
    if (grid == 0) {
        int per_sm = 0;
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_getrs_class<R, MLO, MHI>, kGetrsThreads, 0);
        grid = (per_sm < 1 ? 1 : per_sm) * sm_count();
    }
    k_getrs_class<R, MLO, MHI><<<grid, kGetrsThreads, 0, s>>>(LU, val_off, vec_off, piv, b, x, p.order,
                                                                p.bin_start);
    BJ_LAUNCH_CHECK();
    return BJ_OK;
}

}  // namespace bj
