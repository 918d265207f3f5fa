#pragma once
// getrf_fast.cuh -- hot-path row a3: variable-size batched LU with implicit
// (swap-free) partial pivoting, Fig. 1 bottom, section III.A
// (P:400-464).  Production kernels (the earlier variants in getrf_kernels.cuh
// are kept for the micro benchmarks).
//
// Design, driven by B200 measurements
// (scripts/micro/*.cu, profiles/):
//  * blocks grouped by exact order m (plan, layout.cu); one persistent kernel
//    per size class {1-4, 5-8, 9-16, 17-32}; a warp takes a "task" of
//    G = 32/T same-order blocks, a block occupies a tile of T = pow2ceil(m)
//    lanes and lane r holds row r in registers (static indices: the code is
//    fully unrolled per m).  A is read from HBM once and no lane
//    computes on the reference's 32 x 32 padding.
//  * The per-step critical path is the dependent chain pivot search ->
//    pivot broadcast -> division -> update of column k+1 -> next search.
//    Measured on B200 (one warp alone) it was ~400 cycles per step with
//    REDUX + 2 VOTEs + a shared-memory round trip + the full division; here:
//      - one REDUX.MAX per tile on a key that packs the candidate flag, the
//        top 26 bits of |a| and the inverted lane, so the max also names the
//        pivot lane; an ambiguity VOTE (another candidate with the same
//        truncated key) runs off the critical path and triggers an exact
//        pass only in that rare case -> exactly the oracle's order and tie
//        rule (R1, R2);
//      - every lane refines 1/a_kk of its own candidate while the search
//        runs; the pivot's reciprocal is broadcast with the pivot, leaving a
//        3-operation IEEE quotient (Num::div_pre_u, bit-identical to
//        __ddiv_rn) on the chain;
//      - full-warp tiles broadcast by SHFL from the warp-uniform pivot lane
//        (cheap path of the shuffle unit, ~0.5 SM cycle per 32-bit word);
//        sub-warp tiles publish through a per-warp smem slot / row buffer.
//  * The GER is branch-free: rows that must not change (pivoted rows, padding
//    lanes, singular steps R4) get the multiplier +0 and fma(-0, u, a) == a
//    bit for bit whenever u is finite and a != -0.  That holds at every step
//    if the block's entries are finite, not -0 and below 2^990 (no new -0 can
//    arise and partial pivoting grows entries by at most 2^31 in 32 steps).
//    Blocks failing that check at load time are deferred to a list and
//    factored by k_getrf_safe (plain predicated algorithm in smem).
//  * Combined row swap at write-back: lane r stores its row at
//    position tag-1 of every column and perm[tag-1] = r.
#include "common.cuh"
#include "internal.h"

namespace bj {

constexpr int kFastThreads = 128;
#ifdef BJ_TRACE
__device__ long long g_ftrace[64];
#endif

// "Safe for the zero-multiplier GER" (see header comment).
template <typename R> __device__ __forceinline__ bool zero_mult_safe(R x);
template <> __device__ __forceinline__ bool zero_mult_safe<double>(double x) {
    const unsigned hi = (unsigned)__double2hiint(x), lo = (unsigned)__double2loint(x);
    return ((hi & 0x7fffffffu) < 0x7DD00000u) && !(hi == 0x80000000u && lo == 0u);
}
template <> __device__ __forceinline__ bool zero_mult_safe<float>(float x) {
    const unsigned b = __float_as_uint(x);
    return ((b & 0x7fffffffu) < (221u << 23)) && b != 0x80000000u;
}

// Per-tile max of a 32-bit key.  Full warp: one REDUX; 2 or 4 tiles: one
// REDUX per tile (others contribute 0); smaller tiles: butterfly.
template <int T>
__device__ __forceinline__ unsigned tile_max_key(unsigned key, int t) {
    if constexpr (T == 32) {
        return __reduce_max_sync(kFull, key);
    } else if constexpr (T >= 8) {
        unsigned out = 0;
#pragma unroll
        for (int i = 0; i < 32 / T; ++i) {
            const unsigned v = __reduce_max_sync(kFull, t == i ? key : 0u);
            if (t == i) out = v;
        }
        return out;
    } else {
        unsigned v = key;
#pragma unroll
        for (int off = T / 2; off >= 1; off >>= 1) v = max(v, __shfl_xor_sync(kFull, v, off));
        return v;
    }
}

template <typename R>
struct FastSmem {
    R slot[64];     // per lane: (a_kk, refined 1/a_kk) -- sub-warp tiles
    R row[2][32];   // pivot-row buffers (alternating steps), T elements per tile
};

// Compile-time options (defaults chosen by scripts/micro/getrf_bench.cu on the
// C3 order mix): kFastShflW32 -- full-warp tiles broadcast by SHFL instead of
// smem; kFastPreRcp -- every lane pre-refines 1/a_kk (shorter chain, more
// instructions).
constexpr int kFastShflW32 = 1, kFastPreRcp = 2, kFastHybrid = 4, kFastDblBuf = 8;
// Micro-benchmark-only ablations (wrong results; scripts/micro/getrf_bench.cu):
// skip the pivot-row publish / the division / the pivot search.
constexpr int kFastXNoPub = 16, kFastXNoDiv = 32, kFastXNoSearch = 64, kFastXAllLanes = 128, kFastXOnePair = 256;
#ifndef BJ_FAST_DEFAULT
#define BJ_FAST_DEFAULT 0
#endif

// Staging-buffer stride per tile: T*T elements rounded up to 16 bytes (the
// bulk copy needs 16-B aligned destinations); 32/T tiles fit in 1024 elements.
template <typename R>
__host__ __device__ constexpr int stage_stride(int T) {
    return (T * T + (16 / (int)sizeof(R)) - 1) / (16 / (int)sizeof(R)) * (16 / (int)sizeof(R));
}

// Per-lane view of one task (G = 32 / T blocks of one order): the lane's
// tile's block id and global position.  Fetched two tasks ahead.
struct FTask {
    int m;            // order (warp-uniform), 0 = no task
    bool ok;          // this lane's tile has a block
    int blk;
    int64_t lo;       // val_off[blk]
    int64_t vo;       // vec_off[blk]
};

// S: this tile's block staged in shared memory by the bulk copy (column-major,
// leading dimension M); `after_load` runs once the block is in registers
// (it re-arms the warp's staging buffer with the next task).
template <typename R, int M, int F, class AfterLoad>
__device__ __forceinline__ void getrf_fast_tile(R *__restrict__ A, const FTask &tk, const R *S,
                                                const int64_t *__restrict__ vec_off, int32_t *__restrict__ piv,
                                                int32_t *__restrict__ info, int32_t *__restrict__ safe_list,
                                                unsigned *__restrict__ safe_count, FastSmem<R> &sm,
                                                AfterLoad &&after_load) {
    constexpr int T = tile_width(M);
    constexpr bool W32 = (T == 32) && ((F & kFastShflW32) != 0);
    constexpr bool PRE = (F & kFastPreRcp) != 0;
    constexpr bool HYB = (T == 32) && !W32 && ((F & kFastHybrid) != 0);
    constexpr bool DBL = (F & kFastDblBuf) != 0;
    const int lane = threadIdx.x & 31;
    const int t = lane / T;
    const int r = lane % T;
    const int tbase = t * T;
    bool tile_ok = tk.ok;
    const int blk = tk.blk;
    R *Ab = A + tk.lo;

    R a[M];
    bool ok = true;
    static_for<0, M>([&](auto jc) {
        constexpr int j = decltype(jc)::value;
        a[j] = (tile_ok && r < M) ? S[r + j * M] : R(0);
        ok = ok && zero_mult_safe(a[j]);
    });
    after_load();
    // Tiles with an entry outside the fast path's precondition go to the safe kernel.
    if (tile_bits<T>(__ballot_sync(kFull, !ok), tbase) != 0u) {
        if (tile_ok && r == 0) safe_list[atomicAdd(safe_count, 1u)] = blk;
        tile_ok = false;
    }
    const bool row_ok = tile_ok && (r < M);

    int tag = row_ok ? 0 : -1;      // 0: candidate; k+1: pivot of step k; -1: inactive lane
    int inf = 0;
    bool redo = false;              // pivot ambiguity or IEEE slow-path quotient in this tile
    static_for<0, M>([&](auto kc) {
        constexpr int k = decltype(kc)::value;
        // Alternating buffers: step k+1 publishes into the other buffer, so
        // only the publish -> receive order needs a warp barrier (no barrier
        // between this step's broadcast loads and the next step's stores).
        R *buf = sm.row[DBL ? (k & 1) : 0] + tbase;
#ifdef BJ_TRACE
        if (blockIdx.x == 0 && threadIdx.x == 0) g_ftrace[k] = clock64();
#endif
        const bool cand = (tag == 0);
        // PRE: every lane refines 1/a_kk of its own candidate off the critical path.
        R y = R(0);
        if constexpr (PRE) {
            y = Num<R>::rcp_refine(a[k]);
            if constexpr (!W32 && !HYB) {
                if constexpr (sizeof(R) == 8) *reinterpret_cast<double2 *>(sm.slot + 2 * lane) = make_double2(a[k], y);
                else *reinterpret_cast<float2 *>(sm.slot + 2 * lane) = make_float2(a[k], y);
            }
        }
        // Fig. 1 bottom lines 5-7: key = candidate flag | top 26 bits of |a| | inverted lane.
        const unsigned hi = Num<R>::key_hi(a[k]);
        const unsigned key = cand ? (0x80000000u | (hi & 0x7fffffe0u) | (unsigned)(31 - r)) : 0u;
        const unsigned kmax = (F & kFastXNoSearch) ? (key | (unsigned)(31 - (k % T))) : tile_max_key<T>(key, t);
        int ipiv = (31 - (int)(kmax & 31u)) & (T - 1);   // (inactive tiles: in range, unused)
        // Another candidate with the same truncated key: the lane order may not
        // be the exact order (R1/R2).  No branch here: the tile is redone by
        // the safe kernel (flag checked once after the last step).
        redo = redo || (cand && ((key | 31u) == (kmax | 31u)) && r != ipiv);
        // line 12: the pivot (and its reciprocal)
        const bool isp = (r == ipiv) && row_ok;
        if (isp) tag = k + 1;                                   // line 9
        R d, yd, u1 = R(0);
        if constexpr (HYB) {
            // critical-path values straight from the pivot lane (warp-uniform
            // source), issued before the row publish; the rest of the pivot
            // row (columns >= k+2) goes through shared memory.
            d = __shfl_sync(kFull, a[k], ipiv);
            if constexpr (k + 1 < M) u1 = __shfl_sync(kFull, a[k + 1], ipiv);
            if constexpr (PRE) yd = __shfl_sync(kFull, y, ipiv);
            else yd = Num<R>::rcp_refine(d);
            if constexpr (k + 2 < M) {
                constexpr int j0 = (k + 2) & ~1;
                static_for<0, (M - j0 + 1) / 2>([&](auto pc) {
                    constexpr int j = j0 + 2 * decltype(pc)::value;
                    if constexpr (j + 1 < M) st_shared_pred(isp, buf + j, a[j], a[j + 1]);
                    else st_shared_pred(isp, buf + j, a[j]);
                });
            }
            __syncwarp();
        } else if constexpr (W32) {
            d = __shfl_sync(kFull, a[k], ipiv);
            if constexpr (PRE) yd = __shfl_sync(kFull, y, ipiv);
            else yd = Num<R>::rcp_refine(d);
        } else {
            // publish the pivot row (from column k: d is read back from it)
            if constexpr (sizeof(R) == 8 && T > 1) {
                constexpr int j0 = k & ~1;
                static_for<0, (M - j0 + 1) / 2>([&](auto pc) {
                    constexpr int j = j0 + 2 * decltype(pc)::value;
                    constexpr bool pub = (F & kFastXNoPub) == 0 && ((F & kFastXOnePair) == 0 || j == j0);
                    const bool who = (F & kFastXAllLanes) ? true : isp;
                    if constexpr (pub) {
                        if constexpr (j + 1 < M) st_shared_pred(who, buf + j, a[j], a[j + 1]);
                        else st_shared_pred(who, buf + j, a[j]);
                    }
                });
            } else if constexpr (sizeof(R) == 4 && T >= 4) {
                // fp32: 16-B quads (4x fewer one-lane stores than scalars)
                constexpr int j0 = k & ~3;
                static_for<0, (M - j0 + 3) / 4>([&](auto pc) {
                    constexpr int j = j0 + 4 * decltype(pc)::value;
                    if constexpr (j + 3 < M) {
                        st_shared_pred(isp, buf + j, a[j], a[j + 1], a[j + 2], a[j + 3]);
                    } else {
                        if constexpr (j + 1 < M) st_shared_pred(isp, buf + j, a[j], a[j + 1]);
                        else st_shared_pred(isp, buf + j, a[j]);
                        if constexpr (j + 2 < M) st_shared_pred(isp, buf + j + 2, a[j + 2]);
                    }
                });
            } else {
                static_for<k, M>([&](auto jc) {
                    constexpr int j = decltype(jc)::value;
                    st_shared_pred(isp, buf + j, a[j]);
                });
            }
            __syncwarp();
            if constexpr (PRE) {
                if constexpr (sizeof(R) == 8) {
                    const double2 p2 = *reinterpret_cast<const double2 *>(sm.slot + 2 * (tbase + ipiv));
                    d = p2.x;
                    yd = p2.y;
                } else {
                    const float2 p2 = *reinterpret_cast<const float2 *>(sm.slot + 2 * (tbase + ipiv));
                    d = p2.x;
                    yd = p2.y;
                }
            } else {
                d = buf[k];
                yd = (F & kFastXNoDiv) ? d : Num<R>::rcp_refine(d);
            }
        }
        const bool sing = (Num<R>::key_hi(d) == 0u) && (Num<R>::key_lo(d) == 0u);   // R4
        // line 13 (SCAL): rows that must not change divide 1 by 1 and use l = +0.
        const bool upd = (tag == 0) && !sing;
        bool bad = false;
        const R q = (F & kFastXNoDiv) ? a[k] * d : Num<R>::div_pre_flag(a[k], d, yd, bad);
        redo = redo || (upd && bad);
        const R l = upd ? q : R(0);
        if (upd) a[k] = q;
        if (sing && inf == 0) inf = k + 1;
        // lines 14-15 (GER), branch-free
        if constexpr (HYB) {
            if constexpr (k + 1 < M) a[k + 1] = Num<R>::fma(-l, u1, a[k + 1]);
            if constexpr (((k + 2) & 1) && k + 2 < M) a[k + 2] = Num<R>::fma(-l, buf[k + 2], a[k + 2]);
            constexpr int g0 = (k + 3) & ~1;
            static_for<0, (g0 < M ? (M - g0 + 1) / 2 : 0)>([&](auto pc) {
                constexpr int j = g0 + 2 * decltype(pc)::value;
                if constexpr (j + 1 < M) {
                    if constexpr (sizeof(R) == 8) {
                        const double2 u = *reinterpret_cast<const double2 *>(buf + j);
                        a[j] = Num<R>::fma(-l, u.x, a[j]);
                        a[j + 1] = Num<R>::fma(-l, u.y, a[j + 1]);
                    } else {
                        const float2 u = *reinterpret_cast<const float2 *>(buf + j);
                        a[j] = Num<R>::fma(-l, u.x, a[j]);
                        a[j + 1] = Num<R>::fma(-l, u.y, a[j + 1]);
                    }
                } else {
                    a[j] = Num<R>::fma(-l, buf[j], a[j]);
                }
            });
        } else if constexpr (W32) {
            static_for<k + 1, M>([&](auto jc) {
                constexpr int j = decltype(jc)::value;
                const R u = __shfl_sync(kFull, a[j], ipiv);
                a[j] = Num<R>::fma(-l, u, a[j]);
            });
        } else if constexpr (sizeof(R) == 8 && T > 1) {
            if constexpr ((k + 1) & 1) {
                if constexpr (k + 1 < M) a[k + 1] = Num<R>::fma(-l, buf[k + 1], a[k + 1]);
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
        } else if constexpr (sizeof(R) == 4 && T >= 4) {
            constexpr int g0 = (k + 4) & ~3;            // first quad after column k
            static_for<k + 1, (g0 < M ? g0 : M)>([&](auto jc) {
                constexpr int j = decltype(jc)::value;
                a[j] = Num<R>::fma(-l, buf[j], a[j]);
            });
            static_for<0, (g0 < M ? (M - g0 + 3) / 4 : 0)>([&](auto pc) {
                constexpr int j = g0 + 4 * decltype(pc)::value;
                if constexpr (j + 3 < M) {
                    const float4 u = *reinterpret_cast<const float4 *>(buf + j);
                    a[j] = Num<R>::fma(-l, u.x, a[j]);
                    a[j + 1] = Num<R>::fma(-l, u.y, a[j + 1]);
                    a[j + 2] = Num<R>::fma(-l, u.z, a[j + 2]);
                    a[j + 3] = Num<R>::fma(-l, u.w, a[j + 3]);
                } else {
                    static_for<j, M>([&](auto jc) {
                        constexpr int jj = decltype(jc)::value;
                        a[jj] = Num<R>::fma(-l, buf[jj], a[jj]);
                    });
                }
            });
        } else {
            static_for<k + 1, M>([&](auto jc) {
                constexpr int j = decltype(jc)::value;
                a[j] = Num<R>::fma(-l, buf[j], a[j]);
            });
        }
        if constexpr (!W32 && !DBL) __syncwarp();
    });
    // Tiles that hit a pivot ambiguity or a slow-path quotient are redone by
    // the safe kernel from the (still untouched) input.
    if constexpr ((F & (kFastXNoPub | kFastXNoDiv | kFastXNoSearch | kFastXAllLanes | kFastXOnePair)) != 0) redo = (tag == -7);   // ablation: keep the write-back
    if (tile_bits<T>(__ballot_sync(kFull, redo && tile_ok), tbase) != 0u) {
        if (tile_ok && r == 0) safe_list[atomicAdd(safe_count, 1u)] = blk;
        return;
    }
    // lines 18-19: combined row swap while off-loading L\U.
    if (row_ok) {
        const int pos = tag - 1;
        static_for<0, M>([&](auto jc) {
            constexpr int j = decltype(jc)::value;
            Ab[pos + j * M] = a[j];
        });
        piv[tk.vo + pos] = r;
    }
    if (tile_ok && r == 0) info[blk] = inf;
}

template <typename R, int M, int MHI, int F, class AfterLoad>
__device__ __forceinline__ void getrf_fast_dispatch(R *A, const FTask &tk, const R *S, const int64_t *vec_off,
                                                    int32_t *piv, int32_t *info, int32_t *safe_list,
                                                    unsigned *safe_count, FastSmem<R> &sm, AfterLoad &&after_load) {
    if (tk.m == M) {
        constexpr int T = tile_width(M);
        getrf_fast_tile<R, M, F>(A, tk, S + ((threadIdx.x & 31) / T) * stage_stride<R>(T), vec_off, piv, info,
                                 safe_list, safe_count, sm, after_load);
    } else {
        if constexpr (M < MHI)
            getrf_fast_dispatch<R, M + 1, MHI, F>(A, tk, S, vec_off, piv, info, safe_list, safe_count, sm,
                                                  after_load);
    }
}

// Task indices in two stages so no load waits on the one before it inside
// an iteration: getrf_fetch_idx (order[]) runs three tasks ahead,
// getrf_fetch_off (val_off/vec_off of the block found one iteration earlier)
// two tasks ahead.
template <int NM>
__device__ __forceinline__ FTask getrf_fetch_idx(int64_t task, int64_t ntask, int mlo, const int64_t *s_pref,
                                                 const int64_t *s_first, const int64_t *s_last,
                                                 const int32_t *__restrict__ order) {
    FTask tk;
    tk.m = 0;
    tk.ok = false;
    tk.blk = 0;
    tk.lo = 0;
    tk.vo = 0;
    if (task >= ntask) return tk;
    int i = 0;
    while (i + 1 < NM && s_pref[i + 1] <= task) ++i;
    const int m = mlo + i;
    const int64_t idx = s_first[i] + (task - s_pref[i]) * tiles_per_warp(m) + (threadIdx.x & 31) / tile_width(m);
    tk.m = m;
    tk.ok = idx < s_last[i];
    tk.blk = tk.ok ? __ldg(order + idx) : 0;
    return tk;
}
__device__ __forceinline__ void getrf_fetch_off(FTask &tk, const int64_t *__restrict__ val_off,
                                                const int64_t *__restrict__ vec_off) {
    tk.lo = tk.ok ? __ldg(val_off + tk.blk) : 0;
    tk.vo = tk.ok ? __ldg(vec_off + tk.blk) : 0;
}

// Stage task tk's blocks into the warp's buffer S: tile t's block (m*m
// elements, rounded up to 16 B -- the rounding stays inside the block's
// 16-B aligned slot) goes to S + t*stage_stride(T).  Lane 0 posts the byte count, then
// each tile's lane 0 issues one bulk copy.
template <typename R>
__device__ __forceinline__ void getrf_stage(R *A, const FTask &tk, R *S, uint64_t *bar) {
    if (tk.m == 0) return;
    const int lane = threadIdx.x & 31;
    const int T = tile_width(tk.m);
    const unsigned bytes = (unsigned)((tk.m * tk.m * (int)sizeof(R) + 15) & ~15);
    const unsigned lead = __ballot_sync(kFull, tk.ok && (lane % T) == 0);
    if (lane == 0) mbar_expect_tx(bar, bytes * __popc(lead));
    __syncwarp();
    if (tk.ok && (lane % T) == 0) bulk_g2s(S + (lane / T) * stage_stride<R>(T), A + tk.lo, bytes, bar);
}

// One size class [MLO, MHI].  Tasks enumerated bin by bin; warp w takes tasks
// w, w + nwarps, ...  Each warp owns an 8-KB staging buffer: while it factors
// task i from registers, the bulk copy of task i+1 is in flight (and task
// i+2's indices), so the block load no longer waits on HBM latency.
#ifndef BJ_FAST_MINB
#define BJ_FAST_MINB(R) (sizeof(R) == 8 ? 3 : 4)   // scripts/micro/getrf_bench.cu (B200): fp64 12 warps/SM beat 16, 20; fp32 16
#endif
template <typename R, int MLO, int MHI, int F = BJ_FAST_DEFAULT>
__global__ void __launch_bounds__(kFastThreads, BJ_FAST_MINB(R))
k_getrf_fast(R *A, const int64_t *__restrict__ val_off, const int64_t *__restrict__ vec_off,
             int32_t *__restrict__ piv, int32_t *__restrict__ info, const int32_t *__restrict__ order,
             const int64_t *__restrict__ bin_start, int32_t *__restrict__ safe_list,
             unsigned *__restrict__ safe_count) {
    constexpr int NM = MHI - MLO + 1;
    __shared__ int64_t s_pref[NM + 1], s_first[NM], s_last[NM];
    __shared__ __align__(16) FastSmem<R> s_warp[kFastThreads / 32];
    __shared__ __align__(128) R s_stage[kFastThreads / 32][32 * 32];
    __shared__ __align__(8) uint64_t s_bar[kFastThreads / 32];
    const int w = threadIdx.x >> 5;
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
    if ((threadIdx.x & 31) == 0) mbar_init(&s_bar[w], 1);
    __syncthreads();
    const int64_t ntask = s_pref[NM];
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    FastSmem<R> &sm = s_warp[w];
    R *S = s_stage[w];
    uint64_t *bar = &s_bar[w];
    // Warp index through a warp reduction: the compiler then treats task and
    // order m as warp-uniform and emits plain SHFL/REDUX/VOTE in the
    // size-specialised code instead of collective-emulation sequences.
    const int64_t warp = __reduce_max_sync(kFull, (unsigned)(((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5));
    FTask cur = getrf_fetch_idx<NM>(warp, ntask, MLO, s_pref, s_first, s_last, order);
    FTask nxt = getrf_fetch_idx<NM>(warp + nwarps, ntask, MLO, s_pref, s_first, s_last, order);
    FTask nn = getrf_fetch_idx<NM>(warp + 2 * nwarps, ntask, MLO, s_pref, s_first, s_last, order);
    getrf_fetch_off(cur, val_off, vec_off);
    getrf_fetch_off(nxt, val_off, vec_off);
    getrf_stage(A, cur, S, bar);
    unsigned parity = 0;
    for (int64_t task = warp; task < ntask; task += nwarps) {
        const FTask n3 = getrf_fetch_idx<NM>(task + 3 * nwarps, ntask, MLO, s_pref, s_first, s_last, order);
        getrf_fetch_off(nn, val_off, vec_off);
        mbar_wait_warp(bar, parity);
        parity ^= 1u;
        auto after_load = [&]() {
            __syncwarp();                 // every lane has its block in registers
            fence_proxy_async_smem();
            getrf_stage(A, nxt, S, bar);
        };
        getrf_fast_dispatch<R, MLO, MHI, F>(A, cur, S, vec_off, piv, info, safe_list, safe_count, sm, after_load);
        cur = nxt;
        nxt = nn;
        nn = n3;
    }
}

template <typename R, int MLO, int MHI>
bj_status launch_getrf_fast(R *A, const int64_t *val_off, const int64_t *vec_off, int32_t *piv, int32_t *info,
                            const PlanView &p, int32_t *safe_list, unsigned *safe_count, cudaStream_t s) {
    static int grid = 0;
    if (grid == 0) {
        int per_sm = 0;
        cudaFuncSetAttribute(k_getrf_fast<R, MLO, MHI>, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_getrf_fast<R, MLO, MHI>, kFastThreads, 0);
        grid = (per_sm < 1 ? 1 : per_sm) * sm_count();
    }
    k_getrf_fast<R, MLO, MHI><<<grid, kFastThreads, 0, s>>>(A, val_off, vec_off, piv, info, p.order, p.bin_start,
                                                            safe_list, safe_count);
    BJ_LAUNCH_CHECK();
    return BJ_OK;
}

// Safe path: blocks whose entries violate the fast path's precondition (-0,
// non-finite, |a| >= 2^990).  The plain algorithm of Fig. 1 bottom with the
// block in shared memory (row stride 33, lane r = row r, runtime m), explicit
// predication of pivoted rows, exact 64-bit pivot keys: bit-identical to the
// oracle for every input.  Rarely used, so it favours simplicity.
template <typename R>
__global__ void __launch_bounds__(128)
k_getrf_safe(R *A, const int32_t *__restrict__ sizes, const int64_t *__restrict__ val_off,
             const int64_t *__restrict__ vec_off, int32_t *__restrict__ piv, int32_t *__restrict__ info,
             const int32_t *__restrict__ list, const unsigned *__restrict__ count) {
    __shared__ R S[4][32 * 33];
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
            if (r == ipiv) tag = k + 1;
            const R d = s[ipiv + k * 33];
            if (!sing && tag == 0) {
                const R l = Num<R>::div(v, d);
                s[r + k * 33] = l;
                for (int j = k + 1; j < m; ++j) s[r + j * 33] = Num<R>::fma(-l, s[ipiv + j * 33], s[r + j * 33]);
            }
            if (sing && inf == 0) inf = k + 1;
            __syncwarp();
        }
        if (r < m) {
            const int pos = tag - 1;
            for (int j = 0; j < m; ++j) Ab[pos + j * m] = s[r + j * 33];
            piv[vec_off[blk] + pos] = r;
        }
        if (r == 0) info[blk] = inf;
        __syncwarp();
    }
}

}  // namespace bj
