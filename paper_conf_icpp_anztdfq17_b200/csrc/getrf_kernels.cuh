#pragma once
// getrf_kernels.cuh -- hot-path row a3: variable-size batched LU with implicit
// (swap-free) partial pivoting, Fig. 1 bottom, section III.A
// (P:400-464).
//
// B200 design:
//  * blocks are grouped by exact order m (plan, layout.cu); one kernel per size
//    class {1-4, 5-8, 9-16, 17-32}, persistent grid (SMs x resident CTAs),
//    warps take "tasks" = groups of 32/T same-order blocks;
//  * a block occupies a tile of T = pow2ceil(m) lanes, lane r holds row r in
//    registers (m values), so the matrix is read from HBM once and
//    no lane computes on padding (the reference pads to 32);
//  * the code is fully specialised on m (unrolled k and j loops), so the
//    register indices are static;
//  * pivot search: unsigned max over the |a| bit patterns (+1 for candidates,
//    0 for pivoted rows) within the tile, lowest lane among the maxima via a
//    ballot -> exactly the oracle's tie rule (R1, R2);
//  * implicit pivoting: a per-lane tag (step at which the row was pivoted);
//    the pivot row is broadcast, never swapped;
//  * combined row swap at write-back: lane r stores its row at position
//    tag-1 of every column (a permutation inside each column -> coalesced),
//    and the permutation vector perm[tag-1] = r.
#include "common.cuh"
#include "internal.h"

namespace bj {

constexpr int kGetrfThreads = 128;

template <typename R, int M>
__device__ __forceinline__ void getrf_tile(R *__restrict__ A, const int64_t *__restrict__ val_off,
                                           const int64_t *__restrict__ vec_off, int32_t *__restrict__ piv,
                                           int32_t *__restrict__ info, const int32_t *__restrict__ order,
                                           int64_t first, int64_t last) {
    using Key = typename Num<R>::Key;
    constexpr int T = tile_width(M);
    constexpr unsigned TMASK = (T == 32) ? kFull : ((1u << (T & 31)) - 1u);
    const int lane = threadIdx.x & 31;
    const int t = lane / T;
    const int r = lane % T;
    const int tbase = t * T;
    const int64_t idx = first + t;
    const bool tile_ok = idx < last;
    const int blk = tile_ok ? __ldg(order + idx) : 0;
    const bool row_ok = tile_ok && (r < M);
    R *Ab = A + (tile_ok ? __ldg(val_off + blk) : 0);

    // Load row r (column-major: lanes of a tile read consecutive addresses).
    R a[M];
    static_for<0, M>([&](auto jc) {
        constexpr int j = decltype(jc)::value;
        a[j] = row_ok ? Ab[r + j * M] : R(0);
    });

    int tag = row_ok ? 0 : -1;   // 0: candidate; k+1: pivot of step k; -1: padding lane
    int inf = 0;
    static_for<0, M>([&](auto kc) {
        constexpr int k = decltype(kc)::value;
        // lines 5-7 of Fig. 1 bottom: max |a_ik| over the unpivoted rows.
        const Key key = (tag == 0) ? Key(Num<R>::absbits(a[k]) + 1) : Key(0);
        Key kmax = key;
#pragma unroll
        for (int off = T / 2; off >= 1; off >>= 1) {
            const Key o = __shfl_xor_sync(kFull, kmax, off);
            kmax = o > kmax ? o : kmax;
        }
        const unsigned ball = __ballot_sync(kFull, key == kmax);
        const unsigned tb = (T == 32) ? ball : ((ball >> tbase) & TMASK);
        const int ipiv = __ffs(tb) - 1;                 // lowest row among the maxima
        const bool sing = (kmax == Key(1));             // all candidates are +-0 (R4)
        if (r == ipiv) tag = k + 1;                     // line 9: p(ipiv) = k
        const R d = __shfl_sync(kFull, a[k], tbase + ipiv);   // line 12
        const bool upd = (tag == 0) && !sing;
        if (upd) a[k] = Num<R>::div(a[k], d);           // line 13: SCAL
        static_for<k + 1, M>([&](auto jc) {             // lines 14-15: GER
            constexpr int j = decltype(jc)::value;
            const R u = __shfl_sync(kFull, a[j], tbase + ipiv);
            if (upd) a[j] = Num<R>::fma(-a[k], u, a[j]);
        });
        if (sing && inf == 0) inf = k + 1;
    });
    // lines 18-19: combined row swap while off-loading L\U.
    if (row_ok) {
        const int pos = tag - 1;
        static_for<0, M>([&](auto jc) {
            constexpr int j = decltype(jc)::value;
            Ab[pos + j * M] = a[j];
        });
        piv[__ldg(vec_off + blk) + pos] = r;
    }
    if (tile_ok && r == 0) info[blk] = inf;
}

template <typename R, int M, int MHI>
__device__ __forceinline__ void getrf_dispatch(int m, R *A, const int64_t *val_off, const int64_t *vec_off,
                                               int32_t *piv, int32_t *info, const int32_t *order,
                                               int64_t first, int64_t last) {
    if (m == M) {
        getrf_tile<R, M>(A, val_off, vec_off, piv, info, order, first, last);
    } else {
        if constexpr (M < MHI) getrf_dispatch<R, M + 1, MHI>(m, A, val_off, vec_off, piv, info, order, first, last);
    }
}

// One size class [MLO, MHI].  Tasks are enumerated bin by bin (all tasks of
// order MLO first); warp w takes tasks w, w + nwarps, ...
template <typename R, int MLO, int MHI>
__global__ void __launch_bounds__(kGetrfThreads)
k_getrf_class(R *A, const int64_t *__restrict__ val_off, const int64_t *__restrict__ vec_off,
              int32_t *__restrict__ piv, int32_t *__restrict__ info, const int32_t *__restrict__ order,
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
        getrf_dispatch<R, MLO, MHI>(m, A, val_off, vec_off, piv, info, order, first, s_last[i]);
    }
}

template <typename K>
static inline int persistent_grid(K kernel, int threads) {
    int per_sm = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kernel, threads, 0);
    if (per_sm < 1) per_sm = 1;
    return per_sm * sm_count();
}

template <typename R, int MLO, int MHI>
bj_status launch_getrf_class(R *A, const int64_t *val_off, const int64_t *vec_off, int32_t *piv,
                              int32_t *info, const PlanView &p, cudaStream_t s) {
    static int grid = 0;
    if (grid == 0) grid = persistent_grid(k_getrf_class<R, MLO, MHI>, kGetrfThreads);
    k_getrf_class<R, MLO, MHI><<<grid, kGetrfThreads, 0, s>>>(A, val_off, vec_off, piv, info, p.order,
                                                                p.bin_start);
    BJ_LAUNCH_CHECK();
    return BJ_OK;
}

}  // namespace bj
