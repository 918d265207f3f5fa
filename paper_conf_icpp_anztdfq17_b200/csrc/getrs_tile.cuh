// getrs_tile.cuh -- one tile of GETRS (hot-path rows a4/a5): b := P b, eager
// unit-lower solve, eager upper solve (P:218-238 steps 2-4, Fig. 2 bottom
// P:498-506, mirrored upper solve P:480-483, R8).
//
// B200 design.  GETRS reads every factor element exactly
// once and does one FMA with it ("only a limited amount of data
// reuse"), so the kernel must spend few instructions per element.  A tile of
// T = rs_lanes(M) lanes (T = 8 for M = 17..32, 4 for 9..16, 2 for 5..8, 1 for
// M <= 4) solves one block; a warp solves G = 32 / T blocks of the same order
// in lockstep.  Lane q of a tile holds the RR = ceil(M / T) <= 4 right-hand-side
// entries of rows i = q + s T (cyclic rows), so every broadcast y_k (one
// segment SHFL from a compile-time source lane) and every per-step
// instruction is shared by G blocks and feeds RR FMAs.  The factor is streamed
// column by column (T consecutive rows = one contiguous segment per tile, the
// coalesced column access of P:520-524) through a register ring D columns
// deep; the lower pass reads the strictly lower part of each column, the
// upper pass the upper part, so each element is loaded once.
#pragma once

#include "common.cuh"

namespace bj {

// Lanes per GETRS tile and blocks per warp.
__host__ __device__ constexpr int rs_lanes(int m) { return m <= 4 ? 1 : m <= 8 ? 2 : m <= 16 ? 4 : 8; }
__host__ __device__ constexpr int rs_tiles(int m) { return 32 / rs_lanes(m); }

// Slow path of getrs_rows: one lane recomputes a whole block in plain scalar
// code with the full IEEE division (same operations, same order -- the fast
// path's quotients are bit-identical wherever they apply) and writes x.  All
// of b is read before x is written (x may alias b).
template <typename R>
__device__ __noinline__ void getrs_slow_block(const R *LU, const int32_t *piv, const R *b, R *x, int m) {
    R v[kMaxM];
    for (int i = 0; i < m; ++i) v[i] = b[piv[i]];
    for (int k = 0; k + 1 < m; ++k)
        for (int i = k + 1; i < m; ++i) v[i] = Num<R>::fma(-LU[i + k * m], v[k], v[i]);
    for (int k = m - 1; k >= 0; --k) {
        v[k] = Num<R>::div(v[k], LU[k + k * m]);
        for (int i = 0; i < k; ++i) v[i] = Num<R>::fma(-LU[i + k * m], v[k], v[i]);
    }
    for (int i = 0; i < m; ++i) x[i] = v[i];
}

// LU: this tile's block (column-major, rows in pivot order); piv/b/x: this
// block's vector segments (x may alias b exactly).  q = lane within the tile.
// Tiles past the end of the batch are given a valid block (the caller clamps
// the index) and only skip the final store, so no load needs a tile predicate.
// pv[s] = perm[q + s T] (prefetched by the caller, one task ahead).
// Factor loads: read-only path (__ldg) when the factors come from an earlier
// kernel; L2-coherent (__ldcg) when this kernel just wrote them (the deferred
// solve of bj_gesv_vbatched, getrf_fast.cuh).
template <bool COH, typename R>
__device__ __forceinline__ R ld_factor(const R *p) {
    if constexpr (COH) return __ldcg(p);
    else return __ldg(p);
}

template <typename R, int M, int DR = 8, bool COH = false>
__device__ __forceinline__ void getrs_rows(const R *__restrict__ LU, const int32_t *__restrict__ piv, const R *b,
                                           R *x, bool tile_ok, int q, const int (&pv)[4]) {
    constexpr int T = rs_lanes(M);
    constexpr int RR = (M + T - 1) / T;
    static_assert(RR <= 4, "at most 4 rows per lane");
    constexpr int NP = 2 * M - 1;                 // phases: lower columns 0..M-2, upper columns M-1..0
    constexpr int D = (NP < DR) ? NP : DR;        // ring depth (columns in flight per lane)
    // Only the last slot can hold rows >= M (when T does not divide M).
    auto in_block = [&](int s, int i) { return (s * T + T - 1 < M) || i < M; };
    const R *col = LU + q;                        // row q of column 0

    R y[RR], dg[RR], yr[RR];
    // b := P b: row i receives b[perm[i]]; lane q also fetches
    // U(i,i) of its rows and refines 1/U(i,i) off the critical path.
    static_for<0, RR>([&](auto sc) {
        constexpr int s = decltype(sc)::value;
        const int i = q + s * T;
        const bool ok = in_block(s, i);
        y[s] = ok ? b[pv[s]] : R(0);
        dg[s] = ok ? ld_factor<COH>(col + s * T + (int64_t)i * M) : R(1);
        yr[s] = Num<R>::rcp_refine(dg[s]);
    });

    bool bad = false;
    R ring[D][RR];
    // Phase p: the column it streams and the rows it uses -- i > k (lower) or
    // i < k (upper; the diagonal was fetched above).  Statically empty slots
    // load nothing.
    auto load = [&](auto pc) {
        constexpr int p = decltype(pc)::value;
        constexpr bool lower = p < M - 1;
        constexpr int k = lower ? p : 2 * M - 2 - p;
        static_for<0, RR>([&](auto sc) {
            constexpr int s = decltype(sc)::value;
            constexpr bool none = lower ? (s * T + T - 1 <= k) : (s * T >= k);
            if constexpr (!none) {
                const int i = q + s * T;
                ring[p % D][s] = in_block(s, i) ? ld_factor<COH>(col + s * T + k * M) : R(0);
            }
        });
    };
    static_for<0, D>([&](auto pc) { load(pc); });

    static_for<0, NP>([&](auto pc) {
        constexpr int p = decltype(pc)::value;
        constexpr bool lower = p < M - 1;
        constexpr int k = lower ? p : 2 * M - 2 - p;
        constexpr int ks = k / T, kl = k % T;   // slot and lane of row k
        if constexpr (!lower) {
            // U x = y (R8): y_k <- y_k / U(k,k) in the lane that holds row k
            // (every lane divides its own slot-ks row).  Fast-path quotient
            // only: a quotient that needs the IEEE slow path sets `bad` and
            // the tile is redone below -- no branch inside the solve.
            bool bq = false;
            const R qv = Num<R>::div_pre_flag(y[ks], dg[ks], yr[ks], bq);
            if (q == kl) { y[ks] = qv; bad = bad || bq; }
        }
        R yk;
        if constexpr (T == 1) yk = y[ks];
        else yk = __shfl_sync(kFull, y[ks], kl, T);
        static_for<0, RR>([&](auto sc) {
            constexpr int s = decltype(sc)::value;
            constexpr bool none = lower ? (s * T + T - 1 <= k) : (s * T >= k);
            constexpr bool all = lower ? (s * T > k) : (s * T + T - 1 < k);
            if constexpr (all) {
                y[s] = Num<R>::fma(-ring[p % D][s], yk, y[s]);
            } else if constexpr (!none) {
                const int i = q + s * T;
                Num<R>::pfma(lower ? (i > k) : (i < k), y[s], -ring[p % D][s], yk);
            }
        });
        if constexpr (p + D < NP) load(std::integral_constant<int, p + D>{});
    });
    // Rare (denormal / extreme-range / special diagonal): the tile is redone
    // by getrs_slow_block instead of storing the fast-path result.
    const unsigned flagged = __ballot_sync(kFull, bad);
    const int lane = threadIdx.x & 31;
    const bool redo = ((flagged >> (lane - q)) & ((T == 32) ? kFull : ((1u << T) - 1u))) != 0u;
    __syncwarp();   // every lane has read b before x is written (x may alias b)
    static_for<0, RR>([&](auto sc) {
        constexpr int s = decltype(sc)::value;
        const int i = q + s * T;
        if (tile_ok && !redo && in_block(s, i)) x[i] = y[s];
    });
    if (flagged != 0u && redo && tile_ok && q == 0) getrs_slow_block<R>(LU, piv, b, x, M);
}

}  // namespace bj
