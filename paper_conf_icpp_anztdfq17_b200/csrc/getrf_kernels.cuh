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
//  * pivot search: unsigned max (REDUX for a full warp) over the high word of
//    |a| (bit 31 set for candidates, 0 for pivoted rows) within the tile, lowest
//    lane among the maxima via a ballot; high-word ties are resolved on the low
//    word -> exactly the oracle's order and tie rule (R1, R2);
//  * implicit pivoting: a per-lane tag (step at which the row was pivoted);
//    the pivot row is never swapped: its lane publishes its trailing part to a
//    per-warp smem buffer (16-B stores) and the unpivoted lanes read it back
//    as 16-B broadcasts inside a divergent branch, so pivoted rows need no
//    selects;
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
                                           int64_t first, int64_t last, R *__restrict__ wbuf) {
    constexpr int T = tile_width(M);
    const int lane = threadIdx.x & 31;
    const int t = lane / T;
    const int r = lane % T;
    const int tbase = t * T;
    const int64_t idx = first + t;
    const bool tile_ok = idx < last;
    const int blk = tile_ok ? __ldg(order + idx) : 0;
    const bool row_ok = tile_ok && (r < M);
    R *Ab = A + (tile_ok ? __ldg(val_off + blk) : 0);
    R *buf = wbuf + tbase;                 // this tile's pivot-row buffer (T elements, smem)

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
        // Fig. 1 bottom lines 5-7: max |a_ik| over the unpivoted rows.  Key =
        // high word of |a| with bit 31 set for candidates (0 for pivoted rows);
        // exact ties of the high word (or |a| < 2^-1022) are resolved on the low
        // word in a rare second pass, so the order is exactly the oracle's.
        const unsigned key = (tag == 0) ? (Num<R>::key_hi(a[k]) | 0x80000000u) : 0u;
        const unsigned kmax = tile_max<T>(key);
        unsigned tb = tile_bits<T>(__ballot_sync(kFull, key == kmax), tbase);
        bool sing;
        if constexpr (sizeof(R) == 8) {
            const bool amb = (__popc(tb) > 1) || (kmax == 0x80000000u);
            sing = false;
            if (__any_sync(kFull, amb)) {
                const bool cand = (key == kmax);
                const unsigned lo = cand ? Num<R>::key_lo(a[k]) : 0u;
                const unsigned lmax = tile_max<T>(lo);
                tb = tile_bits<T>(__ballot_sync(kFull, cand && lo == lmax), tbase);
                sing = (kmax == 0x80000000u) && (lmax == 0u);
            }
        } else {
            sing = (kmax == 0x80000000u);
        }
        const int ipiv = __ffs(tb) - 1;                 // lowest row among the maxima (R1)
        if (r == ipiv) {                                // line 9: p(ipiv) = k; publish the pivot row
            tag = k + 1;
            if constexpr (sizeof(R) == 8 && T > 1) {
                constexpr int j0 = k & ~1;
                static_for<0, (M - j0 + 1) / 2>([&](auto pc) {
                    constexpr int j = j0 + 2 * decltype(pc)::value;
                    if constexpr (j + 1 < M) *reinterpret_cast<double2 *>(buf + j) = make_double2(a[j], a[j + 1]);
                    else buf[j] = a[j];
                });
            } else {
                static_for<k, M>([&](auto jc) {
                    constexpr int j = decltype(jc)::value;
                    buf[j] = a[j];
                });
            }
        }
        __syncwarp();
        const R d = buf[k];                             // line 12
        if (tag == 0 && !sing) {                        // lines 13-15 on the unpivoted rows
            const R l = Num<R>::div(a[k], d);           // SCAL (IEEE division)
            a[k] = l;
            if constexpr (sizeof(R) == 8) {             // GER, pivot row read as 16-B pairs
                if constexpr ((k + 1) & 1) {
                    a[k + 1] = Num<R>::fma(-l, buf[k + 1], a[k + 1]);
                }
                constexpr int j0 = (k + 2) & ~1;
                static_for<0, (M - j0 + 1) / 2>([&](auto pc) {
                    constexpr int j = j0 + 2 * decltype(pc)::value;
                    if constexpr (j + 1 < M) {
                        const double2 u = *reinterpret_cast<const double2 *>(buf + j);
                        a[j] = Num<R>::fma(-l, u.x, a[j]);
                        a[j + 1] = Num<R>::fma(-l, u.y, a[j + 1]);
                    } else {
                        a[j] = Num<R>::fma(-l, buf[j], a[j]);
                    }
                });
            } else {
                static_for<k + 1, M>([&](auto jc) {
                    constexpr int j = decltype(jc)::value;
                    a[j] = Num<R>::fma(-l, buf[j], a[j]);
                });
            }
        }
        if (sing && inf == 0) inf = k + 1;
        __syncwarp();
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
                                               int64_t first, int64_t last, R *wbuf) {
    if (m == M) {
        getrf_tile<R, M>(A, val_off, vec_off, piv, info, order, first, last, wbuf);
    } else {
        if constexpr (M < MHI)
            getrf_dispatch<R, M + 1, MHI>(m, A, val_off, vec_off, piv, info, order, first, last, wbuf);
    }
}

// One size class [MLO, MHI].  Tasks are enumerated bin by bin (all tasks of
// order MLO first); warp w takes tasks w, w + nwarps, ...
template <typename R, int MLO, int MHI>
__global__ void __launch_bounds__(kGetrfThreads, 4)
k_getrf_class(R *A, const int64_t *__restrict__ val_off, const int64_t *__restrict__ vec_off,
              int32_t *__restrict__ piv, int32_t *__restrict__ info, const int32_t *__restrict__ order,
              const int64_t *__restrict__ bin_start) {
    constexpr int NM = MHI - MLO + 1;
    __shared__ int64_t s_pref[NM + 1], s_first[NM], s_last[NM];
    __shared__ __align__(16) R s_buf[kGetrfThreads];          // 32 elements per warp
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
        getrf_dispatch<R, MLO, MHI>(m, A, val_off, vec_off, piv, info, order, first, s_last[i],
                                    s_buf + (threadIdx.x & ~31));
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
