#pragma once
// EXPERIMENT (not built into libbj.so): measured SLOWER than getrf_fast.cuh on
// B200 (scripts/micro/getrf_bench.cu r2: C2-like m=32 341 us vs 252 us; mix
// 17..32 3186 us vs 2543 us), kept for the record.
// getrf_r2.cuh -- hot-path row a3 for block orders 17..32: LU with implicit
// (swap-free) partial pivoting, Fig. 1 bottom, section III.A
// (P:400-464), with TWO rows per lane.
//
// Why (measured on B200, profiles/r01 and scripts/micro): with one row per
// lane (getrf_fast.cuh) the kernel is bound by the shared-memory (MIO) path
// that broadcasts each pivot row -- every lane must receive sum_k (m-k-1)
// values per block through LDS.128 broadcasts (2 wavefronts each) and the
// pivot lane publishes them with one-lane STS.128s; fewer resident warps even
// ran faster.  Here a tile of 16 lanes holds one block (lane q: rows q and
// q+16) and a warp factors two blocks in lockstep, so
//   * one LDS.128 broadcast feeds 2 FMAs per element (half the receive
//     wavefronts per block),
//   * the pivot row is first selected into one register set (FSEL, ALU pipe)
//     and published with one STS.128 per pair for both tiles at once (half the
//     publish instructions per block),
//   * every per-step scalar (reciprocal of the pivot, key decode, flags) is
//     shared by the two blocks.
// The arithmetic per element is unchanged -- same divisions, same FMAs in the
// same k order, same pivot keys and tie rule (R1-R5) -- so the factors are
// bit-identical to the oracle and to the one-row kernel; the same
// zero-multiplier precondition and deferral to k_getrf_safe apply.
#include "../../paper_conf_icpp_anztdfq17_b200/csrc/getrf_fast.cuh"

namespace bj {

constexpr int kR2Threads = 128;
#ifndef BJ_R2_MINB
#define BJ_R2_MINB 3
#endif
#ifndef BJ_R2_SELECT
#define BJ_R2_SELECT 0
#endif

template <typename R>
struct R2Smem {
    R row[2][36];   // pivot-row buffer per tile (tile 1 offset by 288 B: different banks)
};

template <typename R, int M, class AfterLoad>
__device__ __forceinline__ void getrf_r2_tile(R *__restrict__ A, const FTask &tk, const R *S,
                                              int32_t *__restrict__ piv, int32_t *__restrict__ info,
                                              int32_t *__restrict__ safe_list, unsigned *__restrict__ safe_count,
                                              R2Smem<R> &sm, AfterLoad &&after_load) {
    static_assert(M >= 17 && M <= 32, "two rows per lane: orders 17..32");
    const int lane = threadIdx.x & 31;
    const int t = lane >> 4;          // tile (block) of this lane
    const int q = lane & 15;
    const int r0 = q, r1 = q + 16;    // rows held by this lane
    bool tile_ok = tk.ok;
    const int blk = tk.blk;
    R *Ab = A + tk.lo;
    const bool v1 = r1 < M;           // second row exists

    R a0[M], a1[M];
    bool ok = true;
    static_for<0, M>([&](auto jc) {
        constexpr int j = decltype(jc)::value;
        a0[j] = tile_ok ? S[r0 + j * M] : R(0);
        a1[j] = (tile_ok && v1) ? S[r1 + j * M] : R(0);
        ok = ok && zero_mult_safe(a0[j]) && zero_mult_safe(a1[j]);
    });
    after_load();
    if ((__ballot_sync(kFull, !ok) >> (16 * t) & 0xffffu) != 0u) {
        if (tile_ok && q == 0) safe_list[atomicAdd(safe_count, 1u)] = blk;
        tile_ok = false;
    }
    R *buf = sm.row[t];

    // tag: 0 candidate, k+1 pivot of step k, -1 no row (or tile inactive)
    int tag0 = tile_ok ? 0 : -1;
    int tag1 = (tile_ok && v1) ? 0 : -1;
    int inf = 0;
    bool redo = false;
    static_for<0, M>([&](auto kc) {
        constexpr int k = decltype(kc)::value;
        const bool c0 = (tag0 == 0), c1 = (tag1 == 0);
        // Fig. 1 bottom lines 5-7: key = candidate | top 26 bits of |a| | inverted row.
        const unsigned k0 = c0 ? (0x80000000u | (Num<R>::key_hi(a0[k]) & 0x7fffffe0u) | (unsigned)(31 - r0)) : 0u;
        const unsigned k1 = c1 ? (0x80000000u | (Num<R>::key_hi(a1[k]) & 0x7fffffe0u) | (unsigned)(31 - r1)) : 0u;
        const unsigned kl = max(k0, k1);
        const unsigned m0 = __reduce_max_sync(kFull, t == 0 ? kl : 0u);
        const unsigned m1 = __reduce_max_sync(kFull, t == 1 ? kl : 0u);
        const unsigned kmax = t ? m1 : m0;
        const int ipiv = 31 - (int)(kmax & 31u);          // pivot row of this tile
        // another candidate with the same truncated key -> exact pass (R1, R2)
        redo = redo || (c0 && ((k0 | 31u) == (kmax | 31u)) && r0 != ipiv) ||
               (c1 && ((k1 | 31u) == (kmax | 31u)) && r1 != ipiv);
        const bool p0 = (r0 == ipiv) && tag0 == 0 && tile_ok;   // line 12: this lane holds the pivot
        const bool p1 = (r1 == ipiv) && tag1 == 0 && tile_ok;
        if (p0) tag0 = k + 1;                                      // line 9
        if (p1) tag1 = k + 1;
        // publish the pivot row (columns >= k, 16-B pairs)
        constexpr int j0 = k & ~1;
        static_for<0, (M - j0 + 1) / 2>([&](auto pc) {
            constexpr int j = j0 + 2 * decltype(pc)::value;
#if BJ_R2_SELECT
            // select into one register set (ALU), one store for both tiles
            const R x = p1 ? a1[j] : a0[j];
            if constexpr (j + 1 < M) {
                const R y = p1 ? a1[j + 1] : a0[j + 1];
                st_shared_pred(p0 || p1, buf + j, x, y);
            } else {
                st_shared_pred(p0 || p1, buf + j, x);
            }
#else
            // one predicated store per row slot (no selects)
            if constexpr (j + 1 < M) {
                st_shared_pred(p0, buf + j, a0[j], a0[j + 1]);
                st_shared_pred(p1, buf + j, a1[j], a1[j + 1]);
            } else {
                st_shared_pred(p0, buf + j, a0[j]);
                st_shared_pred(p1, buf + j, a1[j]);
            }
#endif
        });
        __syncwarp();
        const R d = buf[k];
        const R yd = Num<R>::rcp_refine(d);
        const bool sing = (Num<R>::key_hi(d) == 0u) && (Num<R>::key_lo(d) == 0u);   // R4
        // line 13 (SCAL): rows that must not change use l = +0
        const bool u0 = (tag0 == 0) && !sing, u1 = (tag1 == 0) && !sing;
        bool bad = false;
        const R q0 = Num<R>::div_pre_flag(a0[k], d, yd, bad);
        const bool b0 = bad;
        bad = false;
        const R q1 = Num<R>::div_pre_flag(a1[k], d, yd, bad);
        redo = redo || (u0 && b0) || (u1 && bad);
        const R l0 = u0 ? q0 : R(0), l1 = u1 ? q1 : R(0);
        if (u0) a0[k] = q0;
        if (u1) a1[k] = q1;
        if (sing && inf == 0) inf = k + 1;
        // lines 14-15 (GER), branch-free; one broadcast load feeds both rows
        if constexpr (sizeof(R) == 8) {
            if constexpr ((k + 1) & 1) {
                if constexpr (k + 1 < M) {
                    const R u = buf[k + 1];
                    a0[k + 1] = Num<R>::fma(-l0, u, a0[k + 1]);
                    a1[k + 1] = Num<R>::fma(-l1, u, a1[k + 1]);
                }
            }
            constexpr int g0 = (k + 2) & ~1;
            static_for<0, (M - g0 + 1) / 2>([&](auto pc) {
                constexpr int j = g0 + 2 * decltype(pc)::value;
                if constexpr (j + 1 < M) {
                    const double2 u = *reinterpret_cast<const double2 *>(buf + j);
                    a0[j] = Num<R>::fma(-l0, u.x, a0[j]);
                    a1[j] = Num<R>::fma(-l1, u.x, a1[j]);
                    a0[j + 1] = Num<R>::fma(-l0, u.y, a0[j + 1]);
                    a1[j + 1] = Num<R>::fma(-l1, u.y, a1[j + 1]);
                } else {
                    const R u = buf[j];
                    a0[j] = Num<R>::fma(-l0, u, a0[j]);
                    a1[j] = Num<R>::fma(-l1, u, a1[j]);
                }
            });
        } else {
            static_for<k + 1, M>([&](auto jc) {
                constexpr int j = decltype(jc)::value;
                const R u = buf[j];
                a0[j] = Num<R>::fma(-l0, u, a0[j]);
                a1[j] = Num<R>::fma(-l1, u, a1[j]);
            });
        }
        __syncwarp();
    });
    if ((__ballot_sync(kFull, redo && tile_ok) >> (16 * t) & 0xffffu) != 0u) {
        if (tile_ok && q == 0) safe_list[atomicAdd(safe_count, 1u)] = blk;
        return;
    }
    // lines 18-19: combined row swap while off-loading L\U
    if (tile_ok) {
        const int pos0 = tag0 - 1;
        static_for<0, M>([&](auto jc) {
            constexpr int j = decltype(jc)::value;
            Ab[pos0 + j * M] = a0[j];
        });
        piv[tk.vo + pos0] = r0;
        if (v1) {
            const int pos1 = tag1 - 1;
            static_for<0, M>([&](auto jc) {
                constexpr int j = decltype(jc)::value;
                Ab[pos1 + j * M] = a1[j];
            });
            piv[tk.vo + pos1] = r1;
        }
        if (q == 0) info[blk] = inf;
    }
}

template <typename R, int M, class AfterLoad>
__device__ __forceinline__ void getrf_r2_dispatch(R *A, const FTask &tk, const R *S, int32_t *piv, int32_t *info,
                                                  int32_t *safe_list, unsigned *safe_count, R2Smem<R> &sm,
                                                  AfterLoad &&after_load) {
    if (tk.m == M) {
        getrf_r2_tile<R, M>(A, tk, S + ((threadIdx.x & 31) >> 4) * (32 * 32), piv, info, safe_list, safe_count, sm,
                            after_load);
    } else {
        if constexpr (M < 32) getrf_r2_dispatch<R, M + 1>(A, tk, S, piv, info, safe_list, safe_count, sm, after_load);
    }
}

// Two blocks of order tk.m per warp: tile t (lanes 16t..16t+15) stages its
// block at S + t*1024 (16-B aligned).
template <typename R>
__device__ __forceinline__ void getrf_r2_stage(R *A, const FTask &tk, R *S, uint64_t *bar) {
    if (tk.m == 0) return;
    const int lane = threadIdx.x & 31;
    const unsigned bytes = (unsigned)((tk.m * tk.m * (int)sizeof(R) + 15) & ~15);
    const unsigned lead = __ballot_sync(kFull, tk.ok && (lane & 15) == 0);
    if (lane == 0) mbar_expect_tx(bar, bytes * __popc(lead));
    __syncwarp();
    if (tk.ok && (lane & 15) == 0) bulk_g2s(S + (lane >> 4) * (32 * 32), A + tk.lo, bytes, bar);
}

// Orders 17..32, two blocks per warp; the staging buffer holds both blocks
// of the next task while this one is factored from registers.
template <typename R>
__global__ void __launch_bounds__(kR2Threads, BJ_R2_MINB)
k_getrf_r2(R *A, const int64_t *__restrict__ val_off, const int64_t *__restrict__ vec_off,
           int32_t *__restrict__ piv, int32_t *__restrict__ info, const int32_t *__restrict__ order,
           const int64_t *__restrict__ bin_start, int32_t *__restrict__ safe_list,
           unsigned *__restrict__ safe_count) {
    constexpr int MLO = 17, NM = 16;
    extern __shared__ __align__(128) unsigned char r2_dyn[];
    __shared__ int64_t s_pref[NM + 1], s_first[NM], s_last[NM];
    __shared__ __align__(16) R2Smem<R> s_warp[kR2Threads / 32];
    __shared__ __align__(8) uint64_t s_bar[kR2Threads / 32];
    const int w = threadIdx.x >> 5;
    if (threadIdx.x == 0) {
        int64_t acc = 0;
        for (int i = 0; i < NM; ++i) {
            const int64_t b0 = bin_start[MLO + i], b1 = bin_start[MLO + i + 1];
            s_first[i] = b0;
            s_last[i] = b1;
            s_pref[i] = acc;
            acc += (b1 - b0 + 1) / 2;
        }
        s_pref[NM] = acc;
    }
    if ((threadIdx.x & 31) == 0) mbar_init(&s_bar[w], 1);
    __syncthreads();
    const int64_t ntask = s_pref[NM];
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    R2Smem<R> &sm = s_warp[w];
    R *S = reinterpret_cast<R *>(r2_dyn) + w * (2 * 32 * 32);
    uint64_t *bar = &s_bar[w];
    const int64_t warp = __reduce_max_sync(kFull, (unsigned)(((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5));
    auto fetch = [&](int64_t task) {
        FTask tk;
        tk.m = 0;
        tk.ok = false;
        tk.blk = 0;
        tk.lo = tk.vo = 0;
        if (task >= ntask) return tk;
        int i = 0;
        while (i + 1 < NM && s_pref[i + 1] <= task) ++i;
        const int64_t idx = s_first[i] + (task - s_pref[i]) * 2 + ((threadIdx.x & 31) >> 4);
        tk.m = MLO + i;
        tk.ok = idx < s_last[i];
        tk.blk = tk.ok ? __ldg(order + idx) : 0;
        tk.lo = tk.ok ? __ldg(val_off + tk.blk) : 0;
        tk.vo = tk.ok ? __ldg(vec_off + tk.blk) : 0;
        return tk;
    };
    FTask cur = fetch(warp);
    FTask nxt = fetch(warp + nwarps);
    getrf_r2_stage(A, cur, S, bar);
    unsigned parity = 0;
    for (int64_t task = warp; task < ntask; task += nwarps) {
        const FTask nn = fetch(task + 2 * nwarps);
        mbar_wait_warp(bar, parity);
        parity ^= 1u;
        auto after_load = [&]() {
            __syncwarp();
            fence_proxy_async_smem();
            getrf_r2_stage(A, nxt, S, bar);
        };
        getrf_r2_dispatch<R, MLO>(A, cur, S, piv, info, safe_list, safe_count, sm, after_load);
        cur = nxt;
        nxt = nn;
    }
}

constexpr size_t r2_dyn_smem(size_t elem) { return (size_t)(kR2Threads / 32) * 2 * 32 * 32 * elem; }

template <typename R>
bj_status launch_getrf_r2(R *A, const int64_t *val_off, const int64_t *vec_off, int32_t *piv, int32_t *info,
                          const PlanView &p, int32_t *safe_list, unsigned *safe_count, cudaStream_t s) {
    static int grid = 0;
    const size_t dyn = r2_dyn_smem(sizeof(R));
    if (grid == 0) {
        cudaFuncSetAttribute(k_getrf_r2<R>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)dyn);
        cudaFuncSetAttribute(k_getrf_r2<R>, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
        int per_sm = 0;
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_getrf_r2<R>, kR2Threads, dyn);
        grid = (per_sm < 1 ? 1 : per_sm) * sm_count();
    }
    k_getrf_r2<R><<<grid, kR2Threads, dyn, s>>>(A, val_off, vec_off, piv, info, p.order, p.bin_start, safe_list,
                                                safe_count);
    BJ_LAUNCH_CHECK();
    return BJ_OK;
}

}  // namespace bj
