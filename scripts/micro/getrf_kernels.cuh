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
//    no lane computes on padding (the reference pads to 32); the
//    code is fully specialised on m (static register indices);
//  * pivot search: unsigned max (REDUX for a full warp) over the high word of
//    |a| (bit 31 set for candidates, 0 for pivoted rows) within the tile, the
//    lowest lane among the maxima via a ballot; high-word ties are resolved on
//    the low word -> exactly the oracle's order and tie rule (R1, R2);
//  * implicit pivoting: a per-lane tag (step at which the row
//    was pivoted); the pivot row is never swapped: its lane publishes its
//    trailing part to a per-warp smem buffer (16-B stores) and the unpivoted
//    lanes read it back as 16-B broadcasts inside a divergent branch, so
//    pivoted rows need no selects;
//  * every lane publishes (a_kk, refined 1/a_kk) before the pivot search, the
//    pivot's pair is read back: the six dependent fp64 operations of the
//    reciprocal refinement leave the step's critical path; the quotient is
//    still the IEEE one (Num::div_pre, bit-identical to __ddiv_rn);
//  * combined row swap at write-back: lane r stores its row at
//    position tag-1 of every column (a permutation inside each column ->
//    coalesced) and perm[tag-1] = r; the next task's blocks are prefetched
//    into L2 (cp.async.bulk.prefetch) while this one is factored.
#include "common.cuh"
#include "internal.h"

namespace bj {

constexpr int kGetrfThreads = 128;

// Variant flags (compile-time; the library uses kGetrfDefault, the micro
// benchmark scripts/micro/getrf_bench.cu compares them).
constexpr int kVarSlot = 1;        // publish (a_kk, 1/a_kk) of every lane; pivot's read back
constexpr int kVarPrefetch = 2;    // L2 bulk prefetch of the next task's blocks
constexpr int kVarShfl = 4;        // full-warp tiles: broadcasts by warp-uniform SHFL
constexpr int kVarNoFallback = 8;  // benchmarking only: no smem fallback path (unsafe)
constexpr int kVarNoDiv = 16;      // sub-warp tiles: branch-free step (predicated publish, l=0 GER)
constexpr int kVarTrace = 32;      // benchmarking only: clock64 per step into g_trace

__device__ long long g_trace[64];
constexpr int kGetrfDefault = 0;   // fastest measured on the C3 order mix (scripts/micro/getrf_bench.cu)

template <typename R>
struct GetrfSmem {
    R row[32];                    // pivot-row broadcast buffer (T elements per tile)
    R slot[64];                   // per lane: (a_kk candidate, its refined reciprocal)
};

template <typename R, int M, int V>
__device__ __forceinline__ void getrf_tile(R *__restrict__ A, const int64_t *__restrict__ val_off,
                                           const int64_t *__restrict__ vec_off, int32_t *__restrict__ piv,
                                           int32_t *__restrict__ info, const int32_t *__restrict__ order,
                                           int64_t first, int64_t last, GetrfSmem<R> &sm) {
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
    R *buf = sm.row + tbase;               // this tile's pivot-row buffer (T elements, smem)

    // Load row r (column-major: lanes of a tile read consecutive addresses).
    R a[M];
    static_for<0, M>([&](auto jc) {
        constexpr int j = decltype(jc)::value;
        a[j] = row_ok ? Ab[r + j * M] : R(0);
    });

    int tag = row_ok ? 0 : -1;   // 0: candidate; k+1: pivot of step k; -1: padding lane
    int inf = 0;
    const bool tracer = ((V & kVarTrace) != 0) && blockIdx.x == 0 && threadIdx.x == 0;
    if constexpr ((V & kVarTrace) != 0) {
        if (tracer) g_trace[0] = clock64();
        R s0 = a[0];
        static_for<1, M>([&](auto jc) { s0 += a[decltype(jc)::value]; });   // force load completion
        if (tracer) g_trace[1] = clock64() + (s0 == 12345.0 ? 1 : 0);
    }
    static_for<0, M>([&](auto kc) {
        constexpr int k = decltype(kc)::value;
        if constexpr ((V & kVarTrace) != 0) {
            if (tracer) g_trace[2 + k] = clock64();
        }
        if constexpr ((V & kVarSlot) != 0) {
            // Every lane publishes (a_ik, refined 1/a_ik); the pivot lane's
            // pair is read back below -> the reciprocal refinement (six
            // dependent fp64 operations) leaves the step's critical path.
            const R y = Num<R>::rcp_refine(a[k]);
            if constexpr (sizeof(R) == 8) *reinterpret_cast<double2 *>(sm.slot + 2 * lane) = make_double2(a[k], y);
            else *reinterpret_cast<float2 *>(sm.slot + 2 * lane) = make_float2(a[k], y);
        }
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
        if constexpr ((V & kVarNoDiv) != 0) {
            // Branch-free step (valid under the fast_ok precondition, checked
            // by the caller): predicated 16-B publish, unpredicated GER with
            // the multiplier +0 on rows that must not change.
            const bool isp = (r == ipiv);
            if (isp) tag = k + 1;                       // line 9
            if constexpr (sizeof(R) == 8 && T > 1) {
                constexpr int j0 = k & ~1;
                static_for<0, (M - j0 + 1) / 2>([&](auto pc) {
                    constexpr int j = j0 + 2 * decltype(pc)::value;
                    if constexpr (j + 1 < M) st_shared_pred(isp, buf + j, a[j], a[j + 1]);
                    else st_shared_pred(isp, buf + j, a[j]);
                });
            } else {
                static_for<k, M>([&](auto jc) {
                    constexpr int j = decltype(jc)::value;
                    st_shared_pred(isp, buf + j, a[j]);
                });
            }
            __syncwarp();
            const R d = buf[k];                         // line 12
            const bool upd = (tag == 0) && !sing;
            const R q = Num<R>::div_pre_u(upd ? a[k] : R(1), d, Num<R>::rcp_refine(d));   // line 13
            const R l = upd ? q : R(0);
            if (upd) a[k] = q;
            if constexpr (sizeof(R) == 8) {             // lines 14-15, 16-B broadcast reads
                if constexpr ((k + 1) & 1) a[k + 1] = Num<R>::fma(-l, buf[k + 1], a[k + 1]);
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
        } else {
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
            R d, yd = R(0);                                 // line 12: the pivot (and 1/pivot)
            if constexpr ((V & kVarSlot) != 0) {
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
            }
            if (tag == 0 && !sing) {                        // lines 13-15 on the unpivoted rows
                const R l = ((V & kVarSlot) != 0) ? Num<R>::div_pre(a[k], d, yd)   // SCAL (IEEE division)
                                                  : Num<R>::div(a[k], d);
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

// "Safe for the zero-multiplier GER": finite, not -0, and small enough that
// 32 steps of partial pivoting (growth <= 2^31) cannot overflow.
template <typename R> __device__ __forceinline__ bool fast_ok(R x);
template <> __device__ __forceinline__ bool fast_ok<double>(double x) {
    const unsigned hi = (unsigned)__double2hiint(x), lo = (unsigned)__double2loint(x);
    return ((hi & 0x7fffffffu) < 0x7DD00000u) && !(hi == 0x80000000u && lo == 0u);
}
template <> __device__ __forceinline__ bool fast_ok<float>(float x) {
    const unsigned b = __float_as_uint(x);
    return ((b & 0x7fffffffu) < (221u << 23)) && b != 0x80000000u;
}

// Full-warp tile (17 <= m <= 32): one block per warp, lane r holds row r.
// Every broadcast (pivot value, its reciprocal, the pivot row) is a SHFL whose
// source lane (the pivot) is warp-uniform -- measured ~3x cheaper on B200
// than a shuffle with per-lane sources and ~3x cheaper than publishing the
// row through shared memory (a one-lane STS.128 costs ~4.4 SM cycles).
// The GER runs unpredicated on all lanes: rows that must not change (pivoted
// rows, padding lanes) use the multiplier +0, and fma(-0, u, a) == a bit for
// bit whenever u is finite and a != -0.  Both hold for every step when the
// block's entries are finite, not -0 and below 2^990 in magnitude (no new -0
// can arise, growth <= 2^31); blocks failing that check take the smem path.
// Software pipelining: step k updates column k+1 first, then starts the pivot
// search of step k+1 (REDUX/VOTE chain, reciprocal refinement) and only then
// issues the rest of its GER, whose independent SHFL/DFMA stream fills the
// latency of that chain.  Per-element operation order is unchanged.
// Returns false (nothing written) if the block needs the general path.
template <typename R, int M, int V>
__device__ __forceinline__ bool getrf_tile_w32(R *__restrict__ A, const int64_t *__restrict__ val_off,
                                               const int64_t *__restrict__ vec_off, int32_t *__restrict__ piv,
                                               int32_t *__restrict__ info, const int32_t *__restrict__ order,
                                               int64_t first, int64_t last) {
    const int r = threadIdx.x & 31;
    if (first >= last) return true;                  // warp-uniform
    const int blk = __ldg(order + first);
    const bool row_ok = r < M;
    R *Ab = A + __ldg(val_off + blk);

    R a[M];
    bool ok = true;
    static_for<0, M>([&](auto jc) {
        constexpr int j = decltype(jc)::value;
        a[j] = row_ok ? Ab[r + j * M] : R(0);
        ok = ok && fast_ok(a[j]);
    });
    if (!__all_sync(kFull, ok)) return false;

    int tag = row_ok ? 0 : -1;   // 0: candidate; k+1: pivot of step k; -1: padding lane
    int inf = 0;
    // pivot-search state of the current step
    unsigned kmax = 0, ball = 0;
    R y = R(0);
    // Fig. 1 bottom lines 5-7 (R1, R2), first half: key of column c, REDUX, VOTE.
    auto search_start = [&](auto cc) {
        constexpr int c = decltype(cc)::value;
        y = Num<R>::rcp_refine(a[c]);                   // the pivot lane's copy is used later
        const unsigned key = (tag == 0) ? (Num<R>::key_hi(a[c]) | 0x80000000u) : 0u;
        kmax = __reduce_max_sync(kFull, key);
        ball = __ballot_sync(kFull, key == kmax);
    };
    // second half: exact tie pass, pivot lane, SCAL; returns the multiplier.
    auto search_finish = [&](auto cc, int &ipiv, bool &sing) -> R {
        constexpr int c = decltype(cc)::value;
        sing = false;
        if constexpr (sizeof(R) == 8) {
            if (__popc(ball) > 1 || kmax == 0x80000000u) {      // warp-uniform, rare
                const unsigned key = (tag == 0) ? (Num<R>::key_hi(a[c]) | 0x80000000u) : 0u;
                const bool cand = (key == kmax);
                const unsigned lo = cand ? Num<R>::key_lo(a[c]) : 0u;
                const unsigned lmax = __reduce_max_sync(kFull, lo);
                ball = __ballot_sync(kFull, cand && lo == lmax);
                sing = (kmax == 0x80000000u) && (lmax == 0u);
            }
        } else {
            sing = (kmax == 0x80000000u);
        }
        ipiv = __ffs(ball) - 1;                         // warp-uniform
        if (r == ipiv) tag = c + 1;                     // line 9
        R l = R(0);
        if (!sing) {
            const bool upd = (tag == 0);
            const R d = __shfl_sync(kFull, a[c], ipiv);  // line 12
            const R yd = __shfl_sync(kFull, y, ipiv);
            const R q = Num<R>::div_pre(upd ? a[c] : R(1), d, yd);   // line 13 (SCAL)
            l = upd ? q : R(0);
            if (upd) a[c] = q;
        } else if (inf == 0) {
            inf = c + 1;                                // R4: skip SCAL and GER
        }
        return l;
    };

    int ipiv;
    bool sing;
    search_start(std::integral_constant<int, 0>{});
    R l = search_finish(std::integral_constant<int, 0>{}, ipiv, sing);
    static_for<0, M>([&](auto kc) {
        constexpr int k = decltype(kc)::value;
        if constexpr (k + 1 < M) {
            if (!sing) {                                // GER of column k+1 first
                const R u = __shfl_sync(kFull, a[k + 1], ipiv);
                a[k + 1] = Num<R>::fma(-l, u, a[k + 1]);
            }
            search_start(std::integral_constant<int, k + 1>{});
            if (!sing) {                                // rest of the GER (lines 14-15)
                static_for<k + 2, M>([&](auto jc) {
                    constexpr int j = decltype(jc)::value;
                    const R u = __shfl_sync(kFull, a[j], ipiv);
                    a[j] = Num<R>::fma(-l, u, a[j]);
                });
            }
            l = search_finish(std::integral_constant<int, k + 1>{}, ipiv, sing);
        }
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
    if (r == 0) info[blk] = inf;
    return true;
}

template <typename R, int M, int MHI, int V>
__device__ __forceinline__ void getrf_dispatch(int m, R *A, const int64_t *val_off, const int64_t *vec_off,
                                               int32_t *piv, int32_t *info, const int32_t *order,
                                               int64_t first, int64_t last, GetrfSmem<R> &sm) {
    if (m == M) {
        if constexpr (tile_width(M) == 32 && (V & kVarShfl) != 0) {
            const bool done = getrf_tile_w32<R, M, V>(A, val_off, vec_off, piv, info, order, first, last);
            if constexpr ((V & kVarNoFallback) == 0) {
                if (!done) getrf_tile<R, M, V>(A, val_off, vec_off, piv, info, order, first, last, sm);
            }
        } else {
            getrf_tile<R, M, V>(A, val_off, vec_off, piv, info, order, first, last, sm);
        }
    } else {
        if constexpr (M < MHI)
            getrf_dispatch<R, M + 1, MHI, V>(m, A, val_off, vec_off, piv, info, order, first, last, sm);
    }
}

// L2 prefetch of the blocks of task `task` (one bulk prefetch per tile).
template <int MLO, int MHI, typename R>
__device__ __forceinline__ void prefetch_task(const R *A, int64_t task, const int64_t *s_pref,
                                              const int64_t *s_first, const int64_t *s_last,
                                              const int32_t *__restrict__ order, const int64_t *__restrict__ val_off) {
    constexpr int NM = MHI - MLO + 1;
    if (task >= s_pref[NM]) return;
    int i = 0;
    while (i + 1 < NM && s_pref[i + 1] <= task) ++i;
    const int m = MLO + i;
    const int T = tile_width(m);
    const int lane = threadIdx.x & 31;
    const int64_t idx = s_first[i] + (task - s_pref[i]) * tiles_per_warp(m) + lane / T;
    if ((lane % T) == 0 && idx < s_last[i]) {
        const int blk = __ldg(order + idx);
        const R *p = A + __ldg(val_off + blk);
        const unsigned bytes = (unsigned)((m * m * (int)sizeof(R) + 15) & ~15);
        asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(p), "r"(bytes) : "memory");
    }
}

// One size class [MLO, MHI].  Tasks are enumerated bin by bin (all tasks of
// order MLO first); warp w takes tasks w, w + nwarps, ...
template <typename R, int MLO, int MHI, int V = kGetrfDefault>
__global__ void __launch_bounds__(kGetrfThreads, 4)
k_getrf_class(R *A, const int64_t *__restrict__ val_off, const int64_t *__restrict__ vec_off,
              int32_t *__restrict__ piv, int32_t *__restrict__ info, const int32_t *__restrict__ order,
              const int64_t *__restrict__ bin_start) {
    constexpr int NM = MHI - MLO + 1;
    __shared__ int64_t s_pref[NM + 1], s_first[NM], s_last[NM];
    __shared__ __align__(16) GetrfSmem<R> s_warp[kGetrfThreads / 32];
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
    GetrfSmem<R> &sm = s_warp[threadIdx.x >> 5];
    for (int64_t task = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; task < ntask; task += nwarps) {
        if constexpr ((V & kVarPrefetch) != 0)
            prefetch_task<MLO, MHI, R>(A, task + nwarps, s_pref, s_first, s_last, order, val_off);
        int i = 0;
        while (i + 1 < NM && s_pref[i + 1] <= task) ++i;
        const int m = MLO + i;
        const int64_t first = s_first[i] + (task - s_pref[i]) * tiles_per_warp(m);
        getrf_dispatch<R, MLO, MHI, V>(m, A, val_off, vec_off, piv, info, order, first, s_last[i], sm);
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
