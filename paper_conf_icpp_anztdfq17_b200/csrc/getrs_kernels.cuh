#pragma once
// getrs_kernels.cuh -- hot-path rows a4/a5: batched GETRS, P:218-238 steps 2-4,
// section III.B, Fig. 2 bottom (eager, column-oriented).
//
// Same size classes as getrf.cu; the tile (getrs_tile.cuh) gives each lane
// up to 4 rows and each warp 32 / rs_lanes(m) blocks.  The eager lower solve
// broadcasts y_k and every row below applies one fused AXPY term; the upper
// solve (mirrored, R8) divides y_k by U(k,k) first.  Every y_i receives the
// same sequence of correctly rounded operations as the oracle.
#include "common.cuh"
#include "internal.h"
#include "getrs_tile.cuh"

namespace bj {

constexpr int kGetrsThreads = 128;
#ifndef BJ_RS_DEPTH
#define BJ_RS_DEPTH 12   // scripts/micro/getrs_bench.cu sweep (B200, 3-stage index pipeline): 12 > 4
#endif
#ifndef BJ_RS_MINB
#define BJ_RS_MINB 4
#endif

// Per-lane metadata of one task (G blocks).  The dependent index chain
// order -> offsets -> perm is pipelined across iterations: rs_fetch_idx runs
// three tasks ahead, rs_fetch_off two, rs_fetch_piv one, so no load waits on
// another inside an iteration.
struct RsTask {
    int m;                 // block order (warp-uniform), 0 = no task
    bool ok;               // this lane's tile has a block
    int blk;
    int64_t vo, lo;        // vec_off / val_off of the tile's block
    int pv[4];             // perm of the lane's rows (q + s T)
};

template <int NM>
__device__ __forceinline__ RsTask rs_fetch_idx(int64_t task, int64_t ntask, int mlo, const int64_t *s_pref,
                                               const int64_t *s_first, const int64_t *s_last,
                                               const int32_t *order) {
    RsTask t;
    t.m = 0;
    t.ok = false;
    t.blk = 0;
    t.vo = t.lo = 0;
    t.pv[0] = t.pv[1] = t.pv[2] = t.pv[3] = 0;
    if (task >= ntask) return t;
    int i = 0;
    while (i + 1 < NM && s_pref[i + 1] <= task) ++i;
    const int m = mlo + i;
    const int T = rs_lanes(m);
    const int lane = threadIdx.x & 31;
    const int64_t last = s_last[i];
    const int64_t idx = s_first[i] + (task - s_pref[i]) * rs_tiles(m) + lane / T;
    t.m = m;
    t.ok = idx < last;
    t.blk = __ldg(order + (t.ok ? idx : last - 1));   // clamped: see getrs_rows
    return t;
}
__device__ __forceinline__ void rs_fetch_off(RsTask &t, const int64_t *val_off, const int64_t *vec_off) {
    if (t.m == 0) return;
    t.vo = __ldg(vec_off + t.blk);
    t.lo = __ldg(val_off + t.blk);
}
__device__ __forceinline__ void rs_fetch_piv(RsTask &t, const int32_t *piv) {
    if (t.m == 0) return;
    const int T = rs_lanes(t.m);
    const int q = (threadIdx.x & 31) % T;
#pragma unroll
    for (int s = 0; s < 4; ++s) {
        const int r = q + s * T;
        t.pv[s] = r < t.m ? __ldg(piv + t.vo + r) : 0;
    }
}

template <typename R, int M, int MHI>
__device__ __forceinline__ void getrs_dispatch(const RsTask &t, const R *LU, const int32_t *piv, const R *b, R *x) {
    if (t.m == M) {
        constexpr int T = rs_lanes(M);
        getrs_rows<R, M, BJ_RS_DEPTH>(LU + t.lo, piv + t.vo, b + t.vo, x + t.vo, t.ok, (threadIdx.x & 31) % T, t.pv);
    } else {
        if constexpr (M < MHI) getrs_dispatch<R, M + 1, MHI>(t, LU, piv, b, x);
    }
}

template <typename R, int MLO, int MHI>
__global__ void __launch_bounds__(kGetrsThreads, BJ_RS_MINB)
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
            const int g = rs_tiles(m);
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
    // The warp index goes through a warp reduction so the compiler sees it
    // (and everything derived from it: task, order m) as warp-uniform; the
    // shuffles inside the size-specialised code are then plain SHFLs rather
    // than collective-emulation sequences.
    const int64_t warp = __reduce_max_sync(kFull, (unsigned)(((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5));
    RsTask cur = rs_fetch_idx<NM>(warp, ntask, MLO, s_pref, s_first, s_last, order);
    RsTask nxt = rs_fetch_idx<NM>(warp + nwarps, ntask, MLO, s_pref, s_first, s_last, order);
    RsTask nn = rs_fetch_idx<NM>(warp + 2 * nwarps, ntask, MLO, s_pref, s_first, s_last, order);
    rs_fetch_off(cur, val_off, vec_off);
    rs_fetch_off(nxt, val_off, vec_off);
    rs_fetch_piv(cur, piv);
    for (int64_t task = warp; task < ntask; task += nwarps) {
        const RsTask n3 = rs_fetch_idx<NM>(task + 3 * nwarps, ntask, MLO, s_pref, s_first, s_last, order);
        rs_fetch_off(nn, val_off, vec_off);
        rs_fetch_piv(nxt, piv);
        getrs_dispatch<R, MLO, MHI>(cur, LU, piv, b, x);
        cur = nxt;
        nxt = nn;
        nn = n3;
    }
}

template <typename R, int MLO, int MHI>
bj_status launch_getrs_class(const R *LU, const int64_t *val_off, const int64_t *vec_off, const int32_t *piv,
                              const R *b, R *x, const PlanView &p, cudaStream_t s) {
    const int grid = persistent_grid(k_getrs_class<R, MLO, MHI>, kGetrsThreads);
    k_getrs_class<R, MLO, MHI><<<grid, kGetrsThreads, 0, s>>>(LU, val_off, vec_off, piv, b, x, p.order,
                                                                p.bin_start);
    BJ_LAUNCH_CHECK();
    return BJ_OK;
}

}  // namespace bj
