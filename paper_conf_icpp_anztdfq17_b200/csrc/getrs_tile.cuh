// getrs_tile.cuh -- one warp-tile of GETRS (used by getrs.cu and by the
// block-Jacobi apply, which is the same solve over global-vector segments).
#pragma once

#include "common.cuh"

namespace bj {

// LU: this tile's block (column-major, rows in pivot order), piv/b/x: this
// block's vector segments.  Each lane of the tile handles one row.
template <typename R, int M>
__device__ __forceinline__ void getrs_tile(const R *__restrict__ LU, const int32_t *__restrict__ piv,
                                           const R *b, R *x, bool tile_ok) {
    constexpr int T = tile_width(M);
    const int lane = threadIdx.x & 31;
    const int r = lane % T;
    const int tbase = lane - r;
    const bool row_ok = tile_ok && (r < M);

    R a[M];                                     // row r of L\U
    static_for<0, M>([&](auto jc) {
        constexpr int j = decltype(jc)::value;
        a[j] = row_ok ? __ldg(LU + r + j * M) : R(0);
    });
    // U(r,r) again (same cache lines) so lane r can refine 1/U(r,r) off the
    // critical path; the quotient itself is still the IEEE one (Num::div_pre).
    const R dg = row_ok ? __ldg(LU + r + r * M) : R(1);
    const R yrcp = Num<R>::rcp_refine(dg);
    // b := P b: lane r receives b[perm[r]].
    R y = row_ok ? b[__ldg(piv + r)] : R(0);

    // L y = P b, eager (Fig. 2 bottom): y_i -= L(i,k) y_k for i > k.
    // (T == 32: the source lane is a compile-time constant -> the cheap
    // warp-uniform SHFL; sub-warp tiles need per-tile sources.)
    static_for<0, M - 1>([&](auto kc) {
        constexpr int k = decltype(kc)::value;
        const R yk = (T == 32) ? __shfl_sync(kFull, y, k) : __shfl_sync(kFull, y, tbase + k);
        Num<R>::pfma(r > k, y, -a[k], yk);
    });
    // U x = y, eager and mirrored (R8): y_k /= U(k,k); y_i -= U(i,k) y_k, i < k.
    static_for<0, M>([&](auto kk) {
        constexpr int k = M - 1 - decltype(kk)::value;
        if (r == k) y = Num<R>::div_pre(y, dg, yrcp);
        const R yk = (T == 32) ? __shfl_sync(kFull, y, k) : __shfl_sync(kFull, y, tbase + k);
        Num<R>::pfma(r < k, y, -a[k], yk);
    });
    __syncwarp();                               // every lane has read b before x is written (x may alias b)
    if (row_ok) x[r] = y;
}

}  // namespace bj
