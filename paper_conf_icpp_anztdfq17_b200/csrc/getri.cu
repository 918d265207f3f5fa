// getri.cu -- NEXT(3) of SURVEY 8(f): the inversion-based block-Jacobi
// variant: explicit block inverses by
// Gauss-Jordan elimination in the setup, the apply as a matrix-vector product.
// Readings R23-R26 fix every operation; the kernels
// reproduce oracle/bj_oracle.c bjo_getri_* / bjo_gemv_* bit for bit.
//
// GETRI (k_getri): like GETRF, a block occupies T = pow2ceil(m) lanes, lane r
// holds row r in registers (fully unrolled per order m), 32/T blocks per warp.
// Step k: pivot search by one REDUX per tile on the packed key (R1/R2; a
// truncated-key ambiguity sends the block to k_getri_safe), the WHOLE pivot
// row is broadcast (SHFL from the warp-uniform pivot lane for full-warp
// tiles, a shared-memory row buffer for sub-warp tiles), every other row of
// the tile -- pivoted or not -- applies f = a_k / d and one FMA per column
// j != k, then stores -f in column k; the pivot row keeps its values (its
// multiplier is +0 and fma(+0, u, u) == u for every u, -0 included), with 1
// in column k.  The pivot lane remembers its pivot d for the final row
// division X(i,:) = W(i,:) / d_i, then Dinv(pos_r, perm[c]) = X(r, c) is
// written column by column (R25).  Singular steps (d == +-0) are skipped by a
// tile-uniform branch.
//
// GEMV apply (k_gemv): lane r of a tile computes y(r) = fma-chain over the
// columns b = 0..m-1 from +0 (R26); the loads of a column are one coalesced
// segment, x(b) is broadcast from the lane that loaded it.
#include "common.cuh"
#include "internal.h"

namespace bj {

constexpr int kGetriThreads = 128;
constexpr int kGemvThreads = 256;

template <typename R>
struct GetriSmem {
    R row[32];        // pivot-row buffer (sub-warp tiles), T elements per tile
    int pv[32];       // pivot lane of each step, per tile (tbase + k)
};

template <typename R, int M>
__device__ __forceinline__ void getri_tile(R *__restrict__ A, int64_t lo, int64_t vo, int blk, bool tile_ok,
                                           int32_t *__restrict__ piv, int32_t *__restrict__ info,
                                           int32_t *__restrict__ safe_list, unsigned *__restrict__ safe_count,
                                           GetriSmem<R> &sm) {
    constexpr int T = tile_width(M);
    constexpr bool W32 = (T == 32);
    const int lane = threadIdx.x & 31;
    const int t = lane / T;
    const int r = lane % T;
    const int tbase = t * T;
    const bool row_ok = tile_ok && r < M;
    R *Ab = A + lo;
    R a[M];
    bool redo = false;          // non-finite input or W, ambiguous key, slow-path quotient, singular block
    static_for<0, M>([&](auto jc) {
        constexpr int j = decltype(jc)::value;
        a[j] = row_ok ? Ab[r + j * M] : R(0);
        redo = redo || !(fabs(a[j]) <= Num<R>::big());
    });
    int tag = row_ok ? 0 : -1;
    int inf = 0;
    R mydiag = R(0);
    const unsigned lanebits = 0x80000000u | (unsigned)(31 - r);
    static_for<0, M>([&](auto kc) {
        constexpr int k = decltype(kc)::value;
        const bool cand = (tag == 0);
        const unsigned key = cand ? ((Num<R>::key_hi(a[k]) & 0x7fffffe0u) | lanebits) : 0u;
        const unsigned kmax = tile_max_key<T>(key, t);
        const int ipiv = (31 - (int)(kmax & 31u)) & (T - 1);
        const bool isp = (r == ipiv) && row_ok;
        if (isp) tag = k + 1;
        if (r == 0) sm.pv[tbase + k] = ipiv;
        R d;
        R *buf = sm.row + tbase;
        if constexpr (W32) {
            d = __shfl_sync(kFull, a[k], ipiv);
        } else {
            static_for<0, M>([&](auto jc) {
                constexpr int j = decltype(jc)::value;
                st_shared_pred(isp, buf + j, a[j]);
            });
            __syncwarp();
            d = buf[k];
        }
        redo = redo || (cand && !isp && (fabs(a[k]) > fabs(d)));   // ambiguous truncated key
        const bool sing = (d == R(0));                                 // R4: skip the step
        if (isp) mydiag = d;
        if (sing && inf == 0) inf = k + 1;
        bool bad = false;
        const R f = Num<R>::div_pre_flag(a[k], d, Num<R>::rcp_refine(d), bad);
        redo = redo || (row_ok && !isp && !sing && bad);
        const R nf = isp ? R(0) : -f;                                   // pivot row: multiplier +0
        if (!sing) {                                                    // tile-uniform

            static_for<0, M>([&](auto jc) {
                constexpr int j = decltype(jc)::value;
                if constexpr (j != k) {
                    R u;
                    if constexpr (W32) u = __shfl_sync(kFull, a[j], ipiv);
                    else u = buf[j];
                    a[j] = Num<R>::fma(nf, u, a[j]);
                }
            });
            a[k] = isp ? R(1) : -f;
        }
        if constexpr (!W32) __syncwarp();
    });
    // final row division X(i,:) = W(i,:) / d_i and output Dinv(pos, perm[c]) = X(r, c);
    // singular blocks (info != 0) and non-finite W go to the safe kernel
    redo = redo || (inf != 0);
    static_for<0, M>([&](auto jc) { redo = redo || !(fabs(a[decltype(jc)::value]) <= Num<R>::big()); });
    const R y = Num<R>::rcp_refine(mydiag);
    static_for<0, M>([&](auto jc) {
        constexpr int j = decltype(jc)::value;
        bool bad = false;
        a[j] = Num<R>::div_pre_flag(a[j], mydiag, y, bad);
        redo = redo || (row_ok && bad);
    });
    __syncwarp();
    const bool again = tile_bits<T>(__ballot_sync(kFull, redo && tile_ok), tbase) != 0u;
    if (again && tile_ok && r == 0) safe_list[atomicAdd(safe_count, 1u)] = blk;
    if (tile_ok && !again) {
        if (row_ok) {
            const int pos = tag - 1;
            static_for<0, M>([&](auto jc) {
                constexpr int j = decltype(jc)::value;
                Ab[pos + sm.pv[tbase + j] * M] = a[j];
            });
            piv[vo + pos] = r;
        }
        if (r == 0) info[blk] = inf;
    }
    __syncwarp();
}

template <typename R, int M, int MHI>
__device__ __forceinline__ void getri_dispatch(int m, R *A, int64_t lo, int64_t vo, int blk, bool ok, int32_t *piv,
                                               int32_t *info, int32_t *safe_list, unsigned *safe_count,
                                               GetriSmem<R> &sm) {
    if (m == M) getri_tile<R, M>(A, lo, vo, blk, ok, piv, info, safe_list, safe_count, sm);
    else if constexpr (M < MHI)
        getri_dispatch<R, M + 1, MHI>(m, A, lo, vo, blk, ok, piv, info, safe_list, safe_count, sm);
}

// One order class [MLO, MHI], persistent over tasks of 32/T same-order blocks.
template <typename R, int MLO, int MHI>
__global__ void __launch_bounds__(kGetriThreads)
k_getri(R *A, const int64_t *__restrict__ val_off, const int64_t *__restrict__ vec_off, int32_t *__restrict__ piv,
        int32_t *__restrict__ info, const int32_t *__restrict__ order, const int64_t *__restrict__ bin_start,
        int32_t *__restrict__ safe_list, unsigned *__restrict__ safe_count) {
    constexpr int NM = MHI - MLO + 1;
    __shared__ int64_t s_pref[NM + 1], s_first[NM], s_last[NM];
    __shared__ __align__(16) GetriSmem<R> s_sm[kGetriThreads / 32];
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
    const int64_t warp = __reduce_max_sync(kFull, (unsigned)(((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5));
    GetriSmem<R> &sm = s_sm[threadIdx.x >> 5];
    for (int64_t task = warp; task < ntask; task += nwarps) {
        int i = 0;
        while (i + 1 < NM && s_pref[i + 1] <= task) ++i;
        const int m = MLO + i;
        const int64_t idx = s_first[i] + (task - s_pref[i]) * tiles_per_warp(m) + (threadIdx.x & 31) / tile_width(m);
        const bool ok = idx < s_last[i];
        const int blk = ok ? __ldg(order + idx) : 0;
        const int64_t lo = ok ? __ldg(val_off + blk) : 0;
        const int64_t vo = ok ? __ldg(vec_off + blk) : 0;
        getri_dispatch<R, MLO, MHI>(m, A, lo, vo, blk, ok, piv, info, safe_list, safe_count, sm);
    }
}

// Safe path: the oracle's algorithm literally, block in shared memory (row
// stride 33), lane r = row r, runtime m, exact 64-bit pivot keys, IEEE
// division (Num::div); rarely used.
template <typename R>
__global__ void __launch_bounds__(128)
k_getri_safe(R *A, const int32_t *__restrict__ sizes, const int64_t *__restrict__ val_off,
             const int64_t *__restrict__ vec_off, int32_t *__restrict__ piv, int32_t *__restrict__ info,
             const int32_t *__restrict__ list, const unsigned *__restrict__ count) {
    __shared__ R S[4][32 * 33];
    __shared__ int P[4][32];
    const int r = threadIdx.x & 31, w = threadIdx.x >> 5;
    R *s = S[w];
    const unsigned n = *count;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t it = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; it < n; it += nwarps) {
        const int blk = list[it];
        const int m = sizes[blk];
        R *Ab = A + val_off[blk];
        for (int j = 0; j < m; ++j)
            if (r < m) s[r + j * 33] = Ab[r + j * m];
        __syncwarp();
        int tag = r < m ? 0 : -1;
        int inf = 0;
        R mydiag = R(0);
        for (int k = 0; k < m; ++k) {
            const R v = r < m ? s[r + k * 33] : R(0);
            unsigned long long key = 0ull;
            if (tag == 0) {
                key = (sizeof(R) == 8) ? ((unsigned long long)__double_as_longlong((double)v) & 0x7fffffffffffffffULL)
                                       : (unsigned long long)(__float_as_uint((float)v) & 0x7fffffffu);
                key += 1ull;
            }
            unsigned long long best = key;
            int bl = r;
#pragma unroll
            for (int off = 16; off >= 1; off >>= 1) {
                const unsigned long long ok = __shfl_xor_sync(kFull, best, off);
                const int ol = __shfl_xor_sync(kFull, bl, off);
                if (ok > best || (ok == best && ol < bl)) { best = ok; bl = ol; }
            }
            const int ipiv = bl;
            const bool sing = (best == 1ull);
            if (r == ipiv) { tag = k + 1; mydiag = s[r + k * 33]; }
            if (r == 0) P[w][k] = ipiv;
            __syncwarp();
            if (sing) {
                if (inf == 0) inf = k + 1;
                continue;
            }
            const R d = s[ipiv + k * 33];
            if (r < m && r != ipiv) {
                const R f = Num<R>::div(v, d);
                for (int j = 0; j < m; ++j)
                    if (j != k) s[r + j * 33] = Num<R>::fma(-f, s[ipiv + j * 33], s[r + j * 33]);
                s[r + k * 33] = -f;
            }
            __syncwarp();
            if (r == ipiv) s[r + k * 33] = R(1);
            __syncwarp();
        }
        if (r < m) {
            const int pos = tag - 1;
            for (int j = 0; j < m; ++j) Ab[pos + P[w][j] * m] = Num<R>::div(s[r + j * 33], mydiag);
            piv[vec_off[blk] + pos] = r;
        }
        if (r == 0) info[blk] = inf;
        __syncwarp();
    }
}

// ------------------------------------------------------------------ GEMV apply
// Lanes per block: tile_width(m) (a warp serves 32/T blocks); lane r owns
// row r.  y(r) = +0, then fma(Dinv(r,b), x(b), y) for b = 0..m-1 (R26).
template <typename R, int M>
__device__ __forceinline__ void gemv_tile(const R *__restrict__ D, const R *__restrict__ x, R *__restrict__ y,
                                          bool ok) {
    constexpr int T = tile_width(M);
    const int lane = threadIdx.x & 31;
    const int r = lane % T;
    const int tbase = lane - r;
    const bool row_ok = ok && r < M;
    // every load of the block issued up front (unpredicated, clamped to a valid
    // element for idle lanes) so the whole row is in flight at once
    const int rr = row_ok ? r : 0;
    const R *Dr = ok ? D + rr : D;
    R dv[M];
    static_for<0, M>([&](auto bc) {
        constexpr int b = decltype(bc)::value;
        dv[b] = __ldg(Dr + b * M);
    });
    const R xr = x[rr];                                   // x may alias y: plain (coherent) load
    R acc = R(0);
    static_for<0, M>([&](auto bc) {
        constexpr int b = decltype(bc)::value;
        const R xb = __shfl_sync(kFull, xr, tbase + b);
        acc = Num<R>::fma(dv[b], xb, acc);
    });
    __syncwarp();                                        // x may alias y: every x read first
    if (row_ok) y[r] = acc;
}

template <typename R, int M, int MHI>
__device__ __forceinline__ void gemv_dispatch(int m, const R *D, const R *x, R *y, bool ok) {
    if (m == M) gemv_tile<R, M>(D, x, y, ok);
    else if constexpr (M < MHI) gemv_dispatch<R, M + 1, MHI>(m, D, x, y, ok);
}

template <typename R, int MLO, int MHI>
__global__ void __launch_bounds__(kGemvThreads)
k_gemv(const R *__restrict__ Dinv, const int64_t *__restrict__ val_off, const int64_t *__restrict__ vec_off,
       const R *x, R *y, const int32_t *__restrict__ order, const int64_t *__restrict__ bin_start) {
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
    const int64_t warp = __reduce_max_sync(kFull, (unsigned)(((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5));
    for (int64_t task = warp; task < ntask; task += nwarps) {
        int i = 0;
        while (i + 1 < NM && s_pref[i + 1] <= task) ++i;
        const int m = MLO + i;
        const int64_t idx = s_first[i] + (task - s_pref[i]) * tiles_per_warp(m) + (threadIdx.x & 31) / tile_width(m);
        const bool ok = idx < s_last[i];
        const int blk = ok ? __ldg(order + idx) : 0;
        const int64_t lo = ok ? __ldg(val_off + blk) : 0;
        const int64_t vo = ok ? __ldg(vec_off + blk) : 0;
        gemv_dispatch<R, MLO, MHI>(m, Dinv + lo, x + vo, y + vo, ok);
    }
}

template <typename R>
bj_status getri_run(R *A, const int64_t *val_off, const int64_t *vec_off, int32_t *piv, int32_t *info,
                    const PlanView &p, const int32_t *sizes, cudaStream_t s) {
    if (p.nblocks == 0) return BJ_OK;
    AsyncScratch scratch(s);
    BJ_CUDA_TRY(cudaMallocAsync((void **)&scratch.p, 16 + sizeof(int32_t) * (size_t)p.nblocks, s));
    unsigned *safe_count = reinterpret_cast<unsigned *>(scratch.p);
    int32_t *safe_list = reinterpret_cast<int32_t *>(scratch.p + 16);
    BJ_CUDA_TRY(cudaMemsetAsync(safe_count, 0, sizeof(unsigned), s));
#define BJ_GETRI_C(LO, HI)                                                                               \
    k_getri<R, LO, HI><<<persistent_grid(k_getri<R, LO, HI>, kGetriThreads), kGetriThreads, 0, s>>>(     \
        A, val_off, vec_off, piv, info, p.order, p.bin_start, safe_list, safe_count);                    \
    BJ_LAUNCH_CHECK();
    BJ_GETRI_C(25, 32) BJ_GETRI_C(17, 24) BJ_GETRI_C(9, 16) BJ_GETRI_C(5, 8) BJ_GETRI_C(1, 4)
#undef BJ_GETRI_C
    k_getri_safe<R><<<sm_count() * 2, 128, 0, s>>>(A, sizes, val_off, vec_off, piv, info, safe_list, safe_count);
    BJ_LAUNCH_CHECK();
    return info_trivial_run(info, p, s);
}

template <typename R>
bj_status gemv_run(const R *Dinv, const int64_t *val_off, const int64_t *vec_off, const R *x, R *y,
                   const PlanView &p, cudaStream_t s) {
    if (p.nblocks == 0) return BJ_OK;
#define BJ_GEMV_C(LO, HI)                                                                              \
    k_gemv<R, LO, HI><<<persistent_grid(k_gemv<R, LO, HI>, kGemvThreads), kGemvThreads, 0, s>>>(       \
        Dinv, val_off, vec_off, x, y, p.order, p.bin_start);                                           \
    BJ_LAUNCH_CHECK();
    BJ_GEMV_C(17, 32) BJ_GEMV_C(9, 16) BJ_GEMV_C(5, 8) BJ_GEMV_C(1, 4)
#undef BJ_GEMV_C
    return BJ_OK;
}

template bj_status getri_run<double>(double *, const int64_t *, const int64_t *, int32_t *, int32_t *,
                                     const PlanView &, const int32_t *, cudaStream_t);
template bj_status getri_run<float>(float *, const int64_t *, const int64_t *, int32_t *, int32_t *,
                                    const PlanView &, const int32_t *, cudaStream_t);
template bj_status gemv_run<double>(const double *, const int64_t *, const int64_t *, const double *, double *,
                                    const PlanView &, cudaStream_t);
template bj_status gemv_run<float>(const float *, const int64_t *, const int64_t *, const float *, float *,
                                   const PlanView &, cudaStream_t);

}  // namespace bj
