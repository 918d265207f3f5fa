#pragma once
// getrf_pair.cuh -- hot-path row a3 for block orders 17..32: LU with implicit
// (swap-free) partial pivoting, Fig. 1 bottom, section III.A
// (P:400-464), one block per WARP PAIR with the columns split between the two
// warps.
//
// Why (B200 measurements, profiles/r02/): with one warp per block and the
// row in registers (lane r = row r) a 32x32 fp64 block needs 64
// registers per lane for the row alone, so only 12-16 warps fit on an SM.
// The pivot row must reach every lane at every step: through shared memory
// (one-lane STS.128 = 4.2 SM-cycles per 16 B, the r01 design, smem-pipe
// bound) or through SHFL from the warp-uniform pivot lane (cheap on the
// shuffle unit, but ptxas places each DFMA right after its SHFL, and 4
// warps per scheduler cannot hide the ~26-cycle latency).  Splitting the
// columns halves the registers per lane (lane r of warp `ROLE` holds row r,
// columns j = 2c + ROLE), so twice as many warps hide the SHFL latency; the
// SHFL count per block is unchanged (each warp broadcasts only its own
// columns of the pivot row, from its own lane ipiv).
//
// Step k is led by the warp that owns column k (k & 1): pivot search (one
// REDUX.MAX on a packed key), the pivot and its reciprocal by SHFL, the IEEE
// quotients l_r = a_rk / a_pk (Num::div_pre_flag), then l_r (0 for rows that
// must not change) and ipiv go to a two-slot shared-memory ring and the
// owner signals the partner with bar.arrive; the partner's bar.sync waits
// for it.  Both warps then update their own columns j > k with one FMA per
// element (zero-multiplier argument and its magnitude tests: getrf_fast.cuh).
// Each element sees exactly the oracle's operations in the oracle's order
// (R3, R5), so L\U, pivots and info are bit-identical; a pivot-search
// ambiguity in the truncated key, a slow-path quotient or a failed
// magnitude test sends the block to k_getrf_safe.
#include "getrf_fast.cuh"

namespace bj {

constexpr int kPairThreads = 64;             // one warp pair per CTA
constexpr int kPairBar = 1;                  // named barriers 1, 2, 3 (0 = __syncthreads)

template <typename R>
struct PairSmem {
    R l[2][32];                              // multipliers of steps k (slot k & 1)
    int ip[2];                               // ipiv | 32 * singular
    int flag[2];                             // per-warp "not fast" flags (load / end exchange)
};

// Named barriers of a pair (64 threads): base + 0 / base + 1 carry the step
// hand-over from warp 0 to warp 1 / from warp 1 to warp 0 (bar.arrive by the
// owner, bar.sync by the partner); base + 2 is the plain two-warp barrier.
// One id per direction: with a single id, a warp's arrive of step k and its
// own sync of step k+1 could complete a phase without the partner.
template <int ID> __device__ __forceinline__ void pair_arrive() { asm volatile("bar.arrive %0, 64;" ::"n"(ID) : "memory"); }
template <int ID> __device__ __forceinline__ void pair_sync() { asm volatile("bar.sync %0, 64;" ::"n"(ID) : "memory"); }

// One block of order M; this warp holds columns j = 2c + ROLE (c < NC) of
// every row.  S = the block staged in shared memory (column-major, ld M).
// `after_load` runs once both warps hold the block in registers.
template <typename R, int M, int ROLE, class AfterLoad>
__device__ __forceinline__ void getrf_pair_tile(R *__restrict__ A, const FTask &tk, const R *S,
                                                int32_t *__restrict__ piv, int32_t *__restrict__ info,
                                                int32_t *__restrict__ safe_list, unsigned *__restrict__ safe_count,
                                                PairSmem<R> &ps, AfterLoad &&after_load) {
    constexpr int bar_id = kPairBar;
    constexpr int NC = (M - ROLE + 1) / 2;
    const int r = threadIdx.x & 31;
    bool row_ok = tk.ok && r < M;

    R a[NC];
    bool ok = true;
    static_for<0, NC>([&](auto cc) {
        constexpr int c = decltype(cc)::value;
        a[c] = row_ok ? S[r + (2 * c + ROLE) * M] : R(0);
        ok = ok && fast_ok(a[c]);
    });
    // both warps loaded (the staging buffer may be re-armed) and agree on the input test
    const bool bad_in = __any_sync(kFull, !ok);
    if (r == 0) ps.flag[ROLE] = bad_in;
    pair_sync<bar_id + 2>();
    const bool skip = !tk.ok || ps.flag[0] || ps.flag[1];
    after_load();
    if (skip) {
        if (tk.ok && ROLE == 0 && r == 0) safe_list[atomicAdd(safe_count, 1u)] = tk.blk;
        pair_sync<bar_id + 2>();               // flags are read before the next task rewrites them
        return;
    }

    int tag = row_ok ? 0 : -1;      // 0: candidate; k+1: pivot of step k; -1: inactive lane
    int inf = 0;
    bool redo = false;
    const unsigned lanebits = 0x80000000u | (unsigned)(31 - r);
    static_for<0, M>([&](auto kc) {
        constexpr int k = decltype(kc)::value;
        constexpr int slot = k & 1;
        int ipiv;
        R l;
        if constexpr ((k & 1) == ROLE) {
            constexpr int kl = k / 2;
            const bool cand = (tag == 0);
            // Fig. 1 bottom lines 5-7: key = candidate flag | top 26 bits of |a| | inverted lane.
            const unsigned key = cand ? ((Num<R>::key_hi(a[kl]) & 0x7fffffe0u) | lanebits) : 0u;
            const unsigned kmax = __reduce_max_sync(kFull, key);
            ipiv = 31 - (int)(kmax & 31u);
            const R d = __shfl_sync(kFull, a[kl], ipiv);           // line 12: the pivot
            const R yd = Num<R>::rcp_refine(d);
            // a candidate strictly larger than the chosen pivot: the truncated key was ambiguous
            redo = redo || (cand && (fabs(a[kl]) > fabs(d)));
            const bool sing = (d == R(0));                          // R4
            if ((r == ipiv) && row_ok) tag = k + 1;                 // line 9
            const bool upd = (tag == 0) && !sing;
            bool bad = false;
            const R q = Num<R>::div_pre_flag(a[kl], d, yd, bad);    // line 13 (SCAL)
            redo = redo || (upd && bad);
            l = upd ? q : R(0);
            if (upd) a[kl] = q;
            if (sing && inf == 0) inf = k + 1;
            ps.l[slot][r] = l;                                      // the partner needs l, ipiv, R4
            if (r == 0) ps.ip[slot] = ipiv | (sing ? 32 : 0);
            pair_arrive<bar_id + ROLE>();
        } else {
            pair_sync<bar_id + 1 - ROLE>();
            l = ps.l[slot][r];
            const int ip = ps.ip[slot];
            ipiv = ip & 31;
            if ((r == ipiv) && row_ok) tag = k + 1;
            if ((ip & 32) && inf == 0) inf = k + 1;
        }
        // lines 14-15 (GER) on this warp's columns j > k, branch-free
        constexpr int c0 = (k + 1 - ROLE + 1) / 2;                 // first local column with 2c + ROLE > k
        static_for<c0, NC>([&](auto cc) {
            constexpr int c = decltype(cc)::value;
            a[c] = Num<R>::fma(-l, __shfl_sync(kFull, a[c], ipiv), a[c]);
        });
    });
    // output magnitude test (getrf_fast.cuh header) and the combined redo decision
    static_for<0, NC>([&](auto cc) { redo = redo || !fast_ok(a[decltype(cc)::value]); });
    const bool bad_out = __any_sync(kFull, redo && row_ok);
    if (r == 0) ps.flag[ROLE] = bad_out;
    pair_sync<bar_id + 2>();
    const bool again = ps.flag[0] || ps.flag[1];
    pair_sync<bar_id + 2>();                   // both read the flags before they are rewritten
    if (again) {
        if (ROLE == 0 && r == 0) safe_list[atomicAdd(safe_count, 1u)] = tk.blk;
        return;
    }
    // lines 18-19: combined row swap while off-loading L\U.
    R *Ab = A + tk.lo;
    if (row_ok) {
        const int pos = tag - 1;
        static_for<0, NC>([&](auto cc) {
            constexpr int c = decltype(cc)::value;
            Ab[pos + (2 * c + ROLE) * M] = a[c];
        });
        if (ROLE == 0) piv[tk.vo + pos] = r;
    }
    if (ROLE == 0 && r == 0) info[tk.blk] = inf;
}

template <typename R, int M, int MHI, int ROLE, class AfterLoad>
__device__ __forceinline__ void getrf_pair_dispatch(R *A, const FTask &tk, const R *S, int32_t *piv, int32_t *info,
                                                    int32_t *safe_list, unsigned *safe_count, PairSmem<R> &ps,
                                                    AfterLoad &&after_load) {
    if (tk.m == M) {
        getrf_pair_tile<R, M, ROLE>(A, tk, S, piv, info, safe_list, safe_count, ps, after_load);
    } else {
        if constexpr (M < MHI)
            getrf_pair_dispatch<R, M + 1, MHI, ROLE>(A, tk, S, piv, info, safe_list, safe_count, ps, after_load);
    }
}

#ifndef BJ_PAIR_MINB
#define BJ_PAIR_MINB 12
#endif
// Orders MLO..MHI (17..32), persistent, one warp pair per CTA: the pair takes
// tasks p, p + npairs, ... (one block each); warp 0 / 1 hold the even / odd
// columns.  Lane 0 of warp 0 keeps the task ring (cp.async, three tasks
// ahead) and stages the next block by bulk copy (TMA engine) into the pair's
// 8-KB buffer while the current one is factored.
template <typename R, int MLO, int MHI>
__global__ void __launch_bounds__(kPairThreads, BJ_PAIR_MINB)
k_getrf_pair(R *A, const int64_t *__restrict__ val_off, const int64_t *__restrict__ vec_off,
             int32_t *__restrict__ piv, int32_t *__restrict__ info, const int32_t *__restrict__ order,
             const int64_t *__restrict__ bin_start, int32_t *__restrict__ safe_list,
             unsigned *__restrict__ safe_count) {
    static_assert(MLO >= 17 && MHI <= 32, "full-warp orders only");
    constexpr int NM = MHI - MLO + 1;
    __shared__ int64_t s_pref[NM + 1], s_first[NM], s_last[NM];
    __shared__ __align__(128) R S[32 * 32];
    __shared__ __align__(16) PairSmem<R> ps;
    __shared__ __align__(16) int64_t r_lo[4], r_vo[4];
    __shared__ int32_t r_blk[4];
    __shared__ __align__(8) uint64_t bar;
    const int role = threadIdx.x >> 5;
    const int lane = threadIdx.x & 31;
    const bool leader = (threadIdx.x == 0);
    const int64_t npairs = gridDim.x;
    const int64_t pair = blockIdx.x;
    if (leader) {
        int64_t acc = 0;
        for (int i = 0; i < NM; ++i) {
            const int64_t b0 = bin_start[MLO + i], b1 = bin_start[MLO + i + 1];
            s_first[i] = b0;
            s_last[i] = b1;
            s_pref[i] = acc;
            acc += b1 - b0;
        }
        s_pref[NM] = acc;
        mbar_init(&bar, 1);
    }
    __syncthreads();
    const int64_t ntask = s_pref[NM];
    if (pair >= ntask) return;               // the whole CTA leaves
    auto order_of = [&](int64_t t) {
        int64_t idx = -1;
        const int m = t < ntask ? task_order<NM>(t, MLO, s_pref, s_first, s_last, idx) : 0;
        return m;
    };
    if (leader) {
        for (int q = 0; q < 3; ++q) {
            const int64_t t = pair + q * npairs;
            int64_t idx = -1;
            if (t < ntask) task_order<NM>(t, MLO, s_pref, s_first, s_last, idx);
            const int32_t blk = idx >= 0 ? __ldg(order + idx) : -1;
            r_blk[q] = blk;
            if (q < 2) {
                r_lo[q] = blk >= 0 ? __ldg(val_off + blk) : 0;
                r_vo[q] = blk >= 0 ? __ldg(vec_off + blk) : 0;
            }
        }
        const int m0 = order_of(pair);
        const unsigned bytes = (unsigned)((m0 * m0 * (int)sizeof(R) + 15) & ~15);
        mbar_expect_tx(&bar, bytes);
        bulk_g2s(S, A + r_lo[0], bytes, &bar);
    }
    __syncthreads();
    unsigned parity = 0;
    int q0 = 0;
    for (int64_t task = pair; task < ntask; task += npairs) {
        const int q1 = (q0 + 1) & 3, q2 = (q0 + 2) & 3, q3 = (q0 + 3) & 3;
        if (leader) {                        // ring: offsets of task+2, block id of task+3
            cp_async_wait_all();
            const int32_t b2 = r_blk[q2];
            if (b2 >= 0) {
                cp_async8(&r_lo[q2], val_off + b2);
                cp_async8(&r_vo[q2], vec_off + b2);
            }
            const int64_t t3 = task + 3 * npairs;
            int64_t idx = -1;
            if (t3 < ntask) task_order<NM>(t3, MLO, s_pref, s_first, s_last, idx);
            if (idx >= 0) cp_async4(&r_blk[q3], order + idx);
            else r_blk[q3] = -1;
            cp_async_commit();
        }
        mbar_wait_warp(&bar, parity);
        parity ^= 1u;
        FTask cur;
        cur.m = order_of(task);
        cur.blk = r_blk[q0];
        cur.ok = cur.blk >= 0;
        cur.lo = r_lo[q0];
        cur.vo = r_vo[q0];
        auto after_load = [&]() {
            if (leader) {
                const int64_t tn = task + npairs;
                const int mn = order_of(tn);
                if (mn != 0 && r_blk[q1] >= 0) {
                    fence_proxy_async_smem();
                    const unsigned bytes = (unsigned)((mn * mn * (int)sizeof(R) + 15) & ~15);
                    mbar_expect_tx(&bar, bytes);
                    bulk_g2s(S, A + r_lo[q1], bytes, &bar);
                } else {
                    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(&bar)) : "memory");
                }
            }
        };
        if (role == 0)
            getrf_pair_dispatch<R, MLO, MHI, 0>(A, cur, S, piv, info, safe_list, safe_count, ps, after_load);
        else
            getrf_pair_dispatch<R, MLO, MHI, 1>(A, cur, S, piv, info, safe_list, safe_count, ps, after_load);
        q0 = q1;
    }
    if (leader) cp_async_wait_all();
}

template <typename R, int MLO, int MHI>
bj_status launch_getrf_pair(R *A, const int64_t *val_off, const int64_t *vec_off, int32_t *piv, int32_t *info,
                            const PlanView &p, int32_t *safe_list, unsigned *safe_count, cudaStream_t s) {
    const int grid = persistent_grid(k_getrf_pair<R, MLO, MHI>, kPairThreads);
    k_getrf_pair<R, MLO, MHI><<<grid, kPairThreads, 0, s>>>(A, val_off, vec_off, piv, info, p.order, p.bin_start,
                                                            safe_list, safe_count);
    BJ_LAUNCH_CHECK();
    return BJ_OK;
}

}  // namespace bj
