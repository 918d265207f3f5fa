#pragma once
// getrf_fast.cuh -- hot-path row a3: variable-size batched LU with implicit
// (swap-free) partial pivoting, Fig. 1 bottom, section III.A
// (P:400-464).
//
// Design, driven by B200 measurements
// (scripts/micro/prims.cu -> profiles/r02/micro_prims.txt):
//  * blocks grouped by exact order m (plan, layout.cu); one persistent kernel
//    per size class {1-4, 5-8, 9-16, 17-32}; a warp takes a "task" of
//    G = 32/T same-order blocks, a block occupies a tile of T = pow2ceil(m)
//    lanes and lane r holds row r in registers (static indices: the code is
//    fully unrolled per m).  A is read from HBM once and no lane
//    computes on the reference's 32 x 32 padding.  The next
//    task's blocks are staged into shared memory by the bulk-copy (TMA)
//    engine while the current task is factored.
//  * Step k (Fig. 1 bottom lines 5-15):
//      - pivot search: one REDUX.MAX per tile on a key that packs the
//        candidate flag, the top 26 bits of |a| and the inverted lane, so the
//        max also names the pivot lane with the lowest-row tie rule (R1, R2).
//        A candidate whose exact |a| exceeds the chosen pivot's (possible
//        only when two values agree in those 26 bits) sets a per-tile redo
//        flag; the tile is then factored again by k_getrf_safe with exact
//        64-bit keys.  Exact ties are resolved by the lane order directly.
//      - broadcast of the pivot row: full-warp tiles (m = 17..32) use SHFL
//        from the warp-uniform pivot lane -- 0.27 SM-cycles per 32-bit word,
//        against 4.2 SM-cycles for a one-lane STS.128 plus 1.2 for the
//        LDS.128 broadcast (measured, micro_prims.txt); sub-warp tiles have a
//        different pivot lane per tile (SHFL at 1.0 SM-cycle per word), so
//        they publish through a per-warp shared-memory row buffer.
//      - SCAL: every candidate refines 1/a_kk of its own entry while the
//        search runs (full-warp tiles); the pivot's reciprocal travels with
//        the pivot, leaving the 3-operation IEEE quotient (Num::div_pre_flag,
//        bit-identical to __ddiv_rn / __fdiv_rn) on the critical path.
//      - GER: branch-free, one FMA per element: rows that must not change
//        (pivoted rows, padding lanes, singular steps R4) use the multiplier
//        +0, and fma(-0, u, a) == a bit for bit unless a == -0 (nvcc turns a
//        predicated DFMA into DFMA + 2 FSEL, 5 instead of 3 issue slots per
//        element).  No -0 can reach a frozen row: inputs hold none (the
//        input test), SCAL writes only column k (never touched again) and a
//        GER result is -0 only through underflow.  Underflow and the fast
//        quotient's domain are guarded by the OUTPUT test: every final L\U
//        entry is 0 or in [2^-450, 2^990) (fp32: [2^-39, 2^96); -0 allowed
//        in the L part, which GER never touches after SCAL).  Every product
//        l*u of two outputs is then 0 or >= 2^-900 with granularity
//        >= 2^-1004, so a GER result is exactly 0 (+0) or >= 2^-1005 in
//        magnitude -- even when the other operand is a subnormal input,
//        which a nonzero product swamps -- and never -0; a frozen row
//        gains +-0 and keeps every value but -0 bit for bit.  A quotient is
//        an output: a subnormal or huge dividend or pivot gives an output
//        outside the range (the tile is redone).  Inf / NaN anywhere stay
//        non-finite up to an output.  So the input test only has to reject
//        -0 (one LOP3 + one min per element); blocks holding one go to
//        k_getrf_safe at load time, blocks failing the output test are
//        redone by it.
//  * Partial pivoting grows entries by at most 2^31 in 32 steps, so every
//    fast-path intermediate is finite.
//  * Combined row swap at write-back: lane r stores its row at
//    position tag-1 of every column and perm[tag-1] = r.
#include "common.cuh"
#include "internal.h"
#include "getrs_tile.cuh"

namespace bj {

constexpr int kFastThreads = 128;

// Input test (header comment): 0 exactly for -0 (bits 0x8000...0).
__device__ __forceinline__ unsigned neg_zero_key(double x) {
    return ((unsigned)__double2hiint(x) ^ 0x80000000u) | (unsigned)__double2loint(x);
}
__device__ __forceinline__ unsigned neg_zero_key(float x) { return __float_as_uint(x) ^ 0x80000000u; }

// Output test with kOut2: +-0 or |x| in [2^-450, 2^990) (fp32 [2^-39, 2^96)).
template <typename R> __device__ __forceinline__ bool fast_ok_out(R x);
template <> __device__ __forceinline__ bool fast_ok_out<double>(double x) {
    const unsigned h = (unsigned)__double2hiint(x) & 0x7fffffffu, lo = (unsigned)__double2loint(x);
    return (h - 0x23D00000u < 0x7DD00000u - 0x23D00000u) || ((h | lo) == 0u);
}
template <> __device__ __forceinline__ bool fast_ok_out<float>(float x) {
    const unsigned b = __float_as_uint(x) & 0x7fffffffu;
    return (b - (88u << 23) < (223u << 23) - (88u << 23)) || b == 0u;
}

// Entries the fast path accepts in the final L\U (header comment): +0, or
// |x| in [2^-450, 2^990) (fp32 [2^-39, 2^96)).  -0 (outside the L part) and
// non-finite values fail.
template <typename R> __device__ __forceinline__ bool fast_ok(R x);
template <> __device__ __forceinline__ bool fast_ok<double>(double x) {
    const unsigned hi = (unsigned)__double2hiint(x), lo = (unsigned)__double2loint(x);
    return ((hi & 0x7fffffffu) - 0x23D00000u < 0x7DD00000u - 0x23D00000u) || ((hi | lo) == 0u);
}
template <> __device__ __forceinline__ bool fast_ok<float>(float x) {
    const unsigned b = __float_as_uint(x);
    return ((b & 0x7fffffffu) - (88u << 23) < (223u << 23) - (88u << 23)) || b == 0u;
}

// Row stride of the panel buffer: fp64 34 elements (272 B = 17 x 16 B, an
// odd number of 16-B units, so the STS.128 of the panel's pivot lanes hit
// distinct bank groups)
// (fp32: 36 elements = 144 B = 9 x 16 B).
template <typename R> __host__ __device__ constexpr int panel_stride() { return sizeof(R) == 8 ? 34 : 36; }
constexpr int kMaxPanel = 4;
template <typename R>
struct __align__(16) FastSmem {
    R row[32];                                    // pivot-row buffer, T elements per tile (sub-warp tiles)
    int pinv[32];                                 // fused solve: lane of the row at position k, per tile
    R panel[kMaxPanel][panel_stride<R>()];        // full-warp tiles: the panel's pivot rows (stale trailing part)
};
// bj_gesv_vbatched kernels of full-warp tiles: + the deferred-solve state
template <typename R>
struct __align__(16) FastSmemD : FastSmem<R> {     // 16-B multiple: the panel's STS.128 stay aligned
    int64_t plo[4], pvo[4];                       // pending blocks (val_off, vec_off)
    int keep;                                     // the last tile's block was kept (not sent to the safe path)
};

// Compile-time variants (scripts/micro/getrf_var.cu measures them):
//   kPre  -- every candidate refines 1/a_kk before the search (shorter chain,
//            more instructions); otherwise 1/d is refined after the broadcast.
//   kMin3 -- 3 CTAs (12 warps) per SM, 168 registers, instead of 4 (16 warps,
//            128 registers).
//   kVol  -- GER broadcast + FMA as volatile inline PTX (ptxas then keeps two
//            SHFL pairs in flight instead of one).
//   kPanel2/3/4 -- full-warp tiles: W-step panels (see getrf_w32_steps).
//   kMin5 / kMin6 -- 5 / 6 CTAs (20 / 24 warps) per SM (102 / 85 registers).
//   kMin4 -- 4 CTAs (16 warps) per SM (128 registers).
//   kNoinline -- per-order tiles out of line (one launch per order range).
//   kOut2 -- output test without the L-part position check (a -0 can only
//            be an L entry, header comment); changes the register allocation,
//            so it is chosen per order (micro_getrf_flags_per_order.txt).
constexpr int kPre = 1, kMin3 = 2, kVol = 4, kPanel2 = 8, kPanel3 = 16, kPanel4 = 32, kMin5 = 64, kMin6 = 128,
              kMin4 = 256, kNoinline = 512, kOut2 = 1024;
__host__ __device__ constexpr int panel_width(int F) {
    return (F & kPanel4) ? 4 : (F & kPanel3) ? 3 : (F & kPanel2) ? 2 : 1;
}
#ifndef BJ_FAST_DEFAULT
#define BJ_FAST_DEFAULT 8
#endif
// Per-order flags of the single-order kernels (profiles/r02/
// micro_getrf_flags_per_order.txt, 34.5k blocks per order): fp64 orders 25
// and 27..32 spill at 128 registers (16 warps/SM); with 168 registers at 12
// warps/SM they are 1-12 % faster.  kPre was slower for every order.
template <typename R, int M>
__host__ __device__ constexpr int fast_flags() {
    if (sizeof(R) == 4) return BJ_FAST_DEFAULT | kOut2;                    // fp32: 3-6 % faster, every order
    return (M >= 25 && M != 26)
               ? (BJ_FAST_DEFAULT | kMin3 | ((M == 25 || M == 27 || M == 31 || M == 32) ? kOut2 : 0))
               : (BJ_FAST_DEFAULT | ((M == 19 || M == 20) ? kOut2 : 0));
}
// Resident CTAs (of 4 warps) per SM: explicit flags, else by the registers
// the largest order of the class needs (row in registers + ~50).
template <typename R>
__host__ __device__ constexpr int fast_min_blocks(int F, int MHI) {
    return (F & kMin3) ? 3 : (F & kMin4) ? 4 : (F & kMin6) ? 6 : (F & kMin5) ? 5
         : (sizeof(R) == 8 || MHI > 26) ? 4 : 5;
}
// Staging buffer per warp: one task = 32/T blocks of order <= MHI.
template <typename R>
__host__ __device__ constexpr int stage_elems(int MLO, int MHI) {
    return MLO >= 17 ? (MHI * MHI + 16 / (int)sizeof(R) - 1) / (16 / (int)sizeof(R)) * (16 / (int)sizeof(R))
                     : 32 * 32;
}

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

// Broadcast of the pivot's value x to every lane of a full-warp tile.
template <typename R>
__device__ __forceinline__ R bcast(R x, int src) { return __shfl_sync(kFull, x, src); }
__device__ __forceinline__ double vbcast(double x, int src) {
    unsigned lo = __double2loint(x), hi = __double2hiint(x), rlo, rhi;
    asm volatile("shfl.sync.idx.b32 %0, %1, %2, 0x1f, -1;" : "=r"(rlo) : "r"(lo), "r"(src));
    asm volatile("shfl.sync.idx.b32 %0, %1, %2, 0x1f, -1;" : "=r"(rhi) : "r"(hi), "r"(src));
    return __hiloint2double(rhi, rlo);
}
__device__ __forceinline__ float vbcast(float x, int src) {
    float r;
    asm volatile("shfl.sync.idx.b32 %0, %1, %2, 0x1f, -1;" : "=f"(r) : "f"(x), "r"(src));
    return r;
}
__device__ __forceinline__ double vfma(double a, double b, double c) {
    double d;
    asm volatile("fma.rn.f64 %0, %1, %2, %3;" : "=d"(d) : "d"(a), "d"(b), "d"(c));
    return d;
}
__device__ __forceinline__ float vfma(float a, float b, float c) {
    float d;
    asm volatile("fma.rn.f32 %0, %1, %2, %3;" : "=f"(d) : "f"(a), "f"(b), "f"(c));
    return d;
}

// Steps of a full-warp tile (M = 17..32) in W-step panels.
//
// Every step needs the pivot row at every lane.  A one-lane STS.128 costs
// 4.2 SM-cycles whatever the number of active lanes (4 quarter-warp passes,
// micro_prims.txt), and SHFL-broadcast DFMA chains are latency-bound, so the
// panel amortises the publish over W pivot rows:
//   1. steps k0..k0+W-1 run on the panel columns only (pivot search, SCAL,
//      and the GER of the columns inside the panel, broadcast by SHFL);
//   2. the W pivot lanes store the trailing part of their rows -- untouched
//      since the panel began -- with the SAME predicated STS.128
//      instructions (one store stream for W rows);
//   3. every lane rebuilds the pivot rows' current values from them,
//      u_s = st_s - sum_{s'<s} l(p_s, k0+s') u_s'  (fma chain in ascending
//      s', exactly the updates pivot row p_s received in steps k0..k0+s-1),
//      and applies the W deferred updates to its own trailing columns in
//      ascending k.
// Every element therefore sees the oracle's operations in the oracle's
// order (R5): the rebuilt u_s is bit-identical to the pivot lane's own value.
// Rows that must not change use multiplier 0 (zero-multiplier argument,
// header comment).  Column k0+W, the next panel's first pivot column, is
// updated first.
template <typename R, int M, int W, bool PRE>
__device__ __forceinline__ void getrf_w32_steps(R (&a)[M], int &tag, unsigned &singmask, bool &redo, bool row_ok,
                                                int r, FastSmem<R> &sm) {
    constexpr int PS = panel_stride<R>();
    constexpr int V = 16 / (int)sizeof(R);                 // elements per 16-B store / load
    const unsigned lanebits = 0x80000000u | (unsigned)(31 - r);
    static_for<0, (M + W - 1) / W>([&](auto pc) {
        constexpr int k0 = decltype(pc)::value * W;
        constexpr int kend = (k0 + W < M) ? k0 + W : M;
        constexpr int nw = kend - k0;
        R lk[W];                                           // this lane's multipliers of the panel's steps
        int ipv[W];                                        // the panel's pivot lanes (warp-uniform)
        static_for<0, nw>([&](auto sc) {
            constexpr int sidx = decltype(sc)::value;
            constexpr int k = k0 + sidx;
            const bool cand = (tag == 0);
            // PRE: every lane refines 1/a_kk of its own entry while the search runs
            R y = R(0);
            if constexpr (PRE) y = Num<R>::rcp_refine(a[k]);
            // Fig. 1 bottom lines 5-7: key = candidate flag | top 26 bits of |a| | inverted lane.
            const unsigned key = cand ? ((Num<R>::key_hi(a[k]) & 0x7fffffe0u) | lanebits) : 0u;
            const unsigned kmax = __reduce_max_sync(kFull, key);
            const int ipiv = 31 - (int)(kmax & 31u);
            const R d = bcast(a[k], ipiv);                      // line 12: the pivot
            const R yd = PRE ? bcast(y, ipiv) : Num<R>::rcp_refine(d);
            // a candidate strictly larger than the chosen pivot: the truncated key was ambiguous
            redo = redo || (cand && (fabs(a[k]) > fabs(d)));
            if ((r == ipiv) && row_ok) tag = k + 1;             // line 9
            const bool sing = (d == R(0));                      // R4
            const bool upd = (tag == 0) && !sing;
            const R q = Num<R>::div_fastpath(a[k], d, yd);       // line 13 (SCAL); exact for kept blocks
            const R l = upd ? q : R(0);
            if (upd) a[k] = q;
            singmask |= sing ? (1u << k) : 0u;
            lk[sidx] = l;
            ipv[sidx] = ipiv;
            static_for<k + 1, kend>([&](auto jc) {              // lines 14-15 inside the panel
                constexpr int j = decltype(jc)::value;          // fma(l, -u, a) == fma(-l, u, a) bitwise
                a[j] = Num<R>::fma(l, -bcast(a[j], ipiv), a[j]);
            });
        });
        if constexpr (kend < M) {
            // 2. the panel's pivot lanes publish their stale trailing parts
            const int slot = tag - 1 - k0;
            const bool pub = row_ok && slot >= 0 && slot < nw;
            R *dst = sm.panel[pub ? slot : 0];
            __syncwarp();                                      // the previous panel's loads are done
            constexpr int j0 = kend & ~(V - 1);
            static_for<0, (M - j0 + V - 1) / V>([&](auto vc) {
                constexpr int j = j0 + V * decltype(vc)::value;
                if constexpr (sizeof(R) == 8) {
                    if constexpr (j + 1 < M) st_shared_pred(pub, dst + j, a[j], a[j + 1]);
                    else st_shared_pred(pub, dst + j, a[j]);
                } else {
                    if constexpr (j + 3 < M) st_shared_pred(pub, dst + j, a[j], a[j + 1], a[j + 2], a[j + 3]);
                    else {
                        if constexpr (j + 1 < M) st_shared_pred(pub, dst + j, a[j], a[j + 1]);
                        else st_shared_pred(pub, dst + j, a[j]);
                        if constexpr (j + 2 < M) st_shared_pred(pub, dst + j + 2, a[j + 2]);
                    }
                }
            });
            // multipliers among the panel's pivot rows: Lp[s][s'] = l(p_s, k0+s')
            R Lp[W][W];
            static_for<1, nw>([&](auto sc) {
                constexpr int sidx = decltype(sc)::value;
                static_for<0, sidx>([&](auto tc) {
                    constexpr int t = decltype(tc)::value;
                    Lp[sidx][t] = bcast(lk[t], ipv[sidx]);
                });
            });
            __syncwarp();
            // 3. rebuild the pivot rows and apply the W deferred updates, column by column
            static_for<kend, M>([&](auto jc) {
                constexpr int j = decltype(jc)::value;
                R u[W];
                static_for<0, nw>([&](auto sc) {
                    constexpr int sidx = decltype(sc)::value;
                    R v = sm.panel[sidx][j];
                    static_for<0, sidx>([&](auto tc) {
                        constexpr int t = decltype(tc)::value;
                        v = Num<R>::fma(Lp[sidx][t], -u[t], v);
                    });
                    u[sidx] = v;
                    a[j] = Num<R>::fma(lk[sidx], -v, a[j]);
                });
            });
        }
    });
}

// Fused setup (setup_fused.cuh): a block sent to the safe kernel must be in
// memory, but the fused path extracted it into shared memory only; the tile
// writes its original (S, column-major, ld M) to A first.
template <typename R, int M>
__device__ __forceinline__ void fused_spill(R *Ab, const R *S, bool tile_ok, int r, int T) {
    if (tile_ok)
        for (int i = r; i < M * M; i += T) Ab[i] = S[i];
    __syncwarp();
}

// Fused GETRS (bj_gesv_vbatched): the factors are still in registers -- lane
// r holds row r of the block, which is row pos = tag-1 of L\U -- so the solve
// of P:218-238 (b := P b, eager unit-lower solve, eager upper solve with
// division by U(k,k); Fig. 2 bottom, R8) needs no reload of the factors.
// Lane r starts with y_pos = b_r (b := P b), the position-k value is
// broadcast from the lane holding position k (inverse permutation in shared
// memory), and each lane updates only its own position, in the oracle's
// order; rows that must not change keep their value by selection (y may hold
// -0).  x may alias b exactly: every b is read before any x is written.
template <typename R, int M>
__device__ __forceinline__ void getrf_tile_solve(const R (&a)[M], int pos, bool row_ok, int r, int tbase,
                                                 const R *b, R *x, FastSmem<R> &sm) {
    R y = row_ok ? b[r] : R(0);
    __syncwarp();
    if (row_ok) sm.pinv[tbase + pos] = r;
    __syncwarp();
    static_for<0, M - 1>([&](auto kc) {                 // forward, unit lower
        constexpr int k = decltype(kc)::value;
        const R yk = __shfl_sync(kFull, y, tbase + sm.pinv[tbase + k]);
        const R t = Num<R>::fma(a[k], -yk, y);
        if (pos > k) y = t;
    });
    static_for<0, M>([&](auto kc) {                     // backward, upper
        constexpr int k = M - 1 - decltype(kc)::value;
        if (pos == k) y = Num<R>::div_pre(y, a[k], Num<R>::rcp_refine(a[k]));
        if constexpr (k > 0) {
            const R yk = __shfl_sync(kFull, y, tbase + sm.pinv[tbase + k]);
            const R t = Num<R>::fma(a[k], -yk, y);
            if (pos < k) y = t;
        }
    });
    if (row_ok) x[pos] = y;
}

// S: this tile's block staged in shared memory by the bulk copy (column-major,
// leading dimension M); `after_load` runs once the block is in registers
// (it re-arms the warp's staging buffer with the next task).
template <typename R, int M, int F, bool SOLVE, class AfterLoad, bool FUSED = false>
__device__ __forceinline__ void getrf_fast_tile(R *__restrict__ A, const FTask &tk, const R *S,
                                                int32_t *__restrict__ piv, int32_t *__restrict__ info,
                                                int32_t *__restrict__ safe_list, unsigned *__restrict__ safe_count,
                                                const R *b, R *x, FastSmem<R> &sm, AfterLoad &&after_load) {
    constexpr int T = tile_width(M);
    constexpr bool W32 = (T == 32);
    constexpr bool PRE = W32 && (F & kPre) != 0;
    const int lane = threadIdx.x & 31;
    const int t = lane / T;
    const int r = lane % T;
    const int tbase = t * T;
    bool tile_ok = tk.ok;
    const int blk = tk.blk;
    R *Ab = A + tk.lo;

    R a[M];
    unsigned nzmin = ~0u;                       // 0 iff the row holds a -0 (the input test)
    static_for<0, M>([&](auto jc) {
        constexpr int j = decltype(jc)::value;
        a[j] = (tile_ok && r < M) ? S[r + j * M] : R(0);
        nzmin = min(nzmin, neg_zero_key(a[j]));
    });
    const bool ok = nzmin != 0u;
    after_load();
    // Tiles with an entry outside the fast path's precondition go to the safe kernel.
    if (tile_bits<T>(__ballot_sync(kFull, !ok), tbase) != 0u) {
        if constexpr (FUSED) fused_spill<R, M>(Ab, S, tile_ok, r, T);
        if (tile_ok && r == 0) safe_list[atomicAdd(safe_count, 1u)] = blk;
        tile_ok = false;
    }
    const bool row_ok = tile_ok && (r < M);

    int tag = row_ok ? 0 : -1;      // 0: candidate; k+1: pivot of step k; -1: inactive lane
    unsigned singmask = 0;          // bit k: step k was singular (R4); info = first such step + 1
    bool redo = false;              // pivot ambiguity or failed magnitude test in this tile
    const unsigned lanebits = 0x80000000u | (unsigned)(31 - r);
    if constexpr (W32 && panel_width(F) > 1) {
        getrf_w32_steps<R, M, panel_width(F), (F & kPre) != 0>(a, tag, singmask, redo, row_ok, r, sm);
    } else static_for<0, M>([&](auto kc) {
        constexpr int k = decltype(kc)::value;
        const bool cand = (tag == 0);
        R y = R(0);
        if constexpr (PRE) y = Num<R>::rcp_refine(a[k]);
        // Fig. 1 bottom lines 5-7: key = candidate flag | top 26 bits of |a| | inverted lane.
        const unsigned key = cand ? ((Num<R>::key_hi(a[k]) & 0x7fffffe0u) | lanebits) : 0u;
        const unsigned kmax = tile_max_key<T>(key, t);
        const int ipiv = (31 - (int)(kmax & 31u)) & (T - 1);   // (inactive tiles: in range, unused)
        // line 12: the pivot d (and its reciprocal yd)
        R d, yd;
        if constexpr (W32) {
            d = bcast(a[k], ipiv);
            yd = PRE ? bcast(y, ipiv) : Num<R>::rcp_refine(d);
        } else {
            // publish the pivot row (from column k: d is read back from it)
            R *buf = sm.row + tbase;
            const bool isp = (r == ipiv) && row_ok;
            if constexpr (sizeof(R) == 8 && T > 1) {
                constexpr int j0 = k & ~1;
                static_for<0, (M - j0 + 1) / 2>([&](auto pc) {
                    constexpr int j = j0 + 2 * decltype(pc)::value;
                    if constexpr (j + 1 < M) st_shared_pred(isp, buf + j, a[j], a[j + 1]);
                    else st_shared_pred(isp, buf + j, a[j]);
                });
            } else if constexpr (sizeof(R) == 4 && T >= 4) {
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
            d = buf[k];
            yd = Num<R>::rcp_refine(d);
        }
        // A candidate strictly larger than the chosen pivot: the truncated
        // key was ambiguous -> exact redo (both finite here, R2 order).
        redo = redo || (cand && (fabs(a[k]) > fabs(d)));
        if ((r == ipiv) && row_ok) tag = k + 1;                    // line 9
        const bool sing = (d == R(0));                              // R4: all candidates +-0
        // line 13 (SCAL), then lines 14-15 (GER) on the rows still unpivoted
        const bool upd = (tag == 0) && !sing;
        const R q = Num<R>::div_fastpath(a[k], d, yd);          // exact for kept blocks (common.cuh)
        const R l = upd ? q : R(0);
        if (upd) a[k] = q;
        singmask |= sing ? (1u << k) : 0u;
        if constexpr (W32) {
            static_for<k + 1, M>([&](auto jc) {
                constexpr int j = decltype(jc)::value;
                if constexpr ((F & kVol) != 0) a[j] = vfma(-l, vbcast(a[j], ipiv), a[j]);
                else a[j] = Num<R>::fma(-l, bcast(a[j], ipiv), a[j]);
            });
        } else {
            const R *buf = sm.row + tbase;
            if constexpr (sizeof(R) == 8 && T > 1) {
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
            __syncwarp();
        }
    });
    // Output test of the zero-multiplier argument (header comment).  The L part
    // (columns < pos) may hold -0 (SCAL of a +0 entry by a negative pivot):
    // GER never touches a column after its SCAL, so those zeros are final.
    static_for<0, M>([&](auto jc) {
        constexpr int j = decltype(jc)::value;
        if constexpr ((F & kOut2) != 0) redo = redo || !fast_ok_out(a[j]);
        else redo = redo || !(fast_ok(a[j]) || (a[j] == R(0) && j < tag - 1));
    });
    // Tiles that hit a pivot ambiguity, a slow-path quotient or a failed
    // output test are redone by the safe kernel from the (still untouched)
    // input; the other tiles of the warp go on (the solve's shuffles need
    // every lane, so no lane returns early).
    const bool again = tile_bits<T>(__ballot_sync(kFull, redo && tile_ok), tbase) != 0u;
    if constexpr (FUSED) {
        if (again) fused_spill<R, M>(Ab, S, tile_ok, r, T);
    }
    if (again && tile_ok && r == 0) safe_list[atomicAdd(safe_count, 1u)] = blk;
    const bool keep = tile_ok && !again;
    const bool row_keep = keep && (r < M);
    // lines 18-19: combined row swap while off-loading L\U.
    const int pos = tag - 1;
    if (row_keep) {
        static_for<0, M>([&](auto jc) {
            constexpr int j = decltype(jc)::value;
            Ab[pos + j * M] = a[j];
        });
        piv[tk.vo + pos] = r;
    }
    if (keep && r == 0) info[blk] = __ffs((int)singmask);
    if constexpr (SOLVE) {
        if constexpr (W32) {
            // solved later by solve_pending (kernel loop); SOLVE && W32 only in FastSmemD kernels
            if (lane == 0) static_cast<FastSmemD<R> &>(sm).keep = keep ? 1 : 0;
        } else {
            getrf_tile_solve<R, M>(a, pos, row_keep, r, tbase, b + tk.vo, x + tk.vo, sm);
        }
    }
}

// Deferred solve of bj_gesv_vbatched for full-warp tiles (M = 17..32): the
// warp collects up to 4 blocks it has factored and kept (L\U and perm just
// written, still in L2) and solves them together with the GETRS tile of
// getrs_tile.cuh -- 8 lanes per block, 4 rows per lane -- reading the factors
// back through L2 (coherent loads).  The SIMT solve from the registers
// (getrf_tile_solve) costs every lane ~20 instructions per step for one FMA;
// this costs the GETRS kernel's instructions and no HBM re-read.  Same
// operations in the same order as GETRS: bit-identical.
template <typename R, int M>
__device__ __forceinline__ void solve_pending(const R *A, const int32_t *piv, const R *b, R *x,
                                              const FastSmemD<R> &sm, int npend) {
    constexpr int T = rs_lanes(M);
    static_assert(T == 8, "full-warp GETRF tiles pair with 8-lane GETRS tiles");
    const int lane = threadIdx.x & 31;
    const int t = lane / T, q = lane % T;
    const bool tile_ok = t < npend;
    const int tt = tile_ok ? t : npend - 1;               // clamped: a valid block, store skipped
    const int64_t lo = sm.plo[tt], vo = sm.pvo[tt];
    int pv[4];
#pragma unroll
    for (int s = 0; s < 4; ++s) {
        const int rr = q + s * T;
        pv[s] = rr < M ? __ldcg(piv + vo + rr) : 0;
    }
    getrs_rows<R, M, 6, true>(A + lo, piv + vo, b + vo, x + vo, tile_ok, q, pv);
}

// Out-of-line tile (kNoinline): each order gets its own register allocation
// inside one kernel launch for a whole order range (instead of one kernel per
// order, whose empty launches cost ~3 us each).
template <typename R, int M, int F, bool SOLVE, class AfterLoad>
__device__ __noinline__ void getrf_tile_call(R *A, FTask tk, const R *S, int32_t *piv, int32_t *info,
                                             int32_t *safe_list, unsigned *safe_count, const R *b, R *x,
                                             FastSmem<R> *sm, AfterLoad after_load) {
    getrf_fast_tile<R, M, F, SOLVE>(A, tk, S, piv, info, safe_list, safe_count, b, x, *sm, after_load);
}

template <typename R, int M, int MHI, int F, bool SOLVE, class AfterLoad>
__device__ __forceinline__ void getrf_fast_dispatch(R *A, const FTask &tk, const R *S, int32_t *piv, int32_t *info,
                                                    int32_t *safe_list, unsigned *safe_count, const R *b, R *x,
                                                    FastSmem<R> &sm, AfterLoad &&after_load) {
    if (tk.m == M) {
        constexpr int T = tile_width(M);
        if constexpr ((F & kNoinline) != 0)
            getrf_tile_call<R, M, F, SOLVE>(A, tk, S + ((threadIdx.x & 31) / T) * stage_stride<R>(T), piv, info,
                                            safe_list, safe_count, b, x, &sm, after_load);
        else
            getrf_fast_tile<R, M, F, SOLVE>(A, tk, S + ((threadIdx.x & 31) / T) * stage_stride<R>(T), piv, info,
                                            safe_list, safe_count, b, x, sm, after_load);
    } else {
        if constexpr (M < MHI)
            getrf_fast_dispatch<R, M + 1, MHI, F, SOLVE>(A, tk, S, piv, info, safe_list, safe_count, b, x, sm,
                                                         after_load);
    }
}

// Task schedule.  Tasks are enumerated bin by bin (orders MLO..MHI); warp w
// takes tasks w, w + nwarps, ...  task_order() gives the order m of a task and
// the index of this lane's tile's block in the plan's `order` array.
template <int NM>
__device__ __forceinline__ int task_order(int64_t task, int mlo, const int64_t *s_pref, const int64_t *s_first,
                                          const int64_t *s_last, int64_t &idx) {
    int i = 0;
    while (i + 1 < NM && s_pref[i + 1] <= task) ++i;
    const int m = mlo + i;
    idx = s_first[i] + (task - s_pref[i]) * tiles_per_warp(m) + (threadIdx.x & 31) / tile_width(m);
    if (idx >= s_last[i]) idx = -1;
    return m;
}

// Per-warp ring of upcoming tasks in shared memory, filled by cp.async
// (LDGSTS: global -> shared without registers), so the index chain
// order[] -> val_off/vec_off of tasks two and three ahead costs no registers
// during the factorization.  Slot s, tile t: the tile's block id (-1: no
// block), val_off and vec_off (written by the tile's lane 0).
template <int G>                             // G = blocks (tiles) per task
struct TaskRing {
    int64_t lo[4][G];
    int64_t vo[4][G];
    int32_t blk[4][G];
};
__device__ __forceinline__ void cp_async4(void *dst, const void *src) {
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(smem_u32(dst)), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async8(void *dst, const void *src) {
    asm volatile("cp.async.ca.shared.global [%0], [%1], 8;" ::"r"(smem_u32(dst)), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_group 0;" ::: "memory"); }

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

// Re-arm the warp's staging buffer with the next task once the current
// block is in registers (the `after_load` step of getrf_fast_tile).
template <typename R>
struct StageNext {
    R *A;
    FTask nxt;
    R *S;
    uint64_t *bar;
    __device__ __forceinline__ void operator()() const {
        __syncwarp();                     // every lane has its block in registers
        fence_proxy_async_smem();
        getrf_stage(A, nxt, S, bar);
    }
};

// One size class [MLO, MHI], persistent.  Each warp owns an 8-KB staging
// buffer: while it factors task i from registers, the bulk copy of task i+1
// is in flight (and the indices of tasks i+2, i+3 in the ring), so the block
// load does not wait on HBM latency.
template <typename R, int MLO, int MHI, int F = BJ_FAST_DEFAULT, bool SOLVE = false>
__global__ void __launch_bounds__(kFastThreads, fast_min_blocks<R>(F, MHI))
k_getrf_fast(R *A, const int64_t *__restrict__ val_off, const int64_t *__restrict__ vec_off,
             int32_t *__restrict__ piv, int32_t *__restrict__ info, const int32_t *__restrict__ order,
             const int64_t *__restrict__ bin_start, int32_t *__restrict__ safe_list,
             unsigned *__restrict__ safe_count, const R *b = nullptr, R *x = nullptr) {
    constexpr int NM = MHI - MLO + 1;
    __shared__ int64_t s_pref[NM + 1], s_first[NM], s_last[NM];
    // bj_gesv_vbatched on full-warp tiles: solves deferred in groups of 4 (solve_pending)
    constexpr bool DEFER = SOLVE && MLO >= 17;
    using Smem = std::conditional_t<DEFER, FastSmemD<R>, FastSmem<R>>;
    __shared__ __align__(16) Smem s_warp[kFastThreads / 32];
    __shared__ __align__(128) R s_stage[kFastThreads / 32][stage_elems<R>(MLO, MHI)];
    constexpr int G = tiles_per_warp(MLO);
    __shared__ __align__(16) TaskRing<G> s_ring[kFastThreads / 32];
    __shared__ __align__(8) uint64_t s_bar[kFastThreads / 32];
    const int w = threadIdx.x >> 5;
    const int lane = threadIdx.x & 31;
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
    if (lane == 0) mbar_init(&s_bar[w], 1);
    // Programmatic dependent launch: the next order's kernel may start filling
    // SMs as this one's CTAs retire (the kernels touch disjoint blocks); each
    // kernel waits for its predecessor before it exits, so stream order holds
    // transitively for whatever is launched after the chain.
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    __syncthreads();
    const int64_t ntask = s_pref[NM];
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    Smem &smd = s_warp[w];
    FastSmem<R> &sm = smd;
    R *S = s_stage[w];
    TaskRing<G> &ring = s_ring[w];
    uint64_t *bar = &s_bar[w];
    // Warp index through a warp reduction: the compiler then treats task and
    // order m as warp-uniform and emits plain SHFL/REDUX/VOTE in the
    // size-specialised code instead of collective-emulation sequences.
    const int64_t warp = __reduce_max_sync(kFull, (unsigned)(((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5));
    if (warp >= ntask) {
        asm volatile("griddepcontrol.wait;" ::: "memory");
        return;
    }
    // prologue: indices of tasks 0..2 and offsets of tasks 0..1 (plain loads)
    // a lane's tile for a task of order m is lane / tile_width(m); ring
    // entries are written by the tile's first lane (lane % T == 0)
    auto tile_of = [&](int64_t t) {
        int64_t idx;
        const int m = t < ntask ? task_order<NM>(t, MLO, s_pref, s_first, s_last, idx) : MLO;
        return lane / tile_width(m);
    };
    auto writer = [&](int64_t t) {
        int64_t idx;
        const int m = t < ntask ? task_order<NM>(t, MLO, s_pref, s_first, s_last, idx) : MLO;
        return (lane % tile_width(m)) == 0;
    };
    for (int q = 0; q < 3; ++q) {
        const int64_t t = warp + q * nwarps;
        int64_t idx = -1;
        if (t < ntask) task_order<NM>(t, MLO, s_pref, s_first, s_last, idx);
        if (writer(t)) {
            const int g = tile_of(t);
            const int32_t blk = idx >= 0 ? __ldg(order + idx) : -1;
            ring.blk[q][g] = blk;
            if (q < 2) {
                ring.lo[q][g] = blk >= 0 ? __ldg(val_off + blk) : 0;
                ring.vo[q][g] = blk >= 0 ? __ldg(vec_off + blk) : 0;
            }
        }
    }
    auto slot_task = [&](int64_t t, int q) {
        FTask tk;
        int64_t idx;
        tk.m = t < ntask ? task_order<NM>(t, MLO, s_pref, s_first, s_last, idx) : 0;
        const int g = tile_of(t);
        tk.blk = ring.blk[q][g];
        tk.ok = tk.m != 0 && tk.blk >= 0;
        tk.lo = ring.lo[q][g];
        tk.vo = ring.vo[q][g];
        return tk;
    };
    __syncwarp();
    getrf_stage(A, slot_task(warp, 0), S, bar);
    unsigned parity = 0;
    int q0 = 0;
    static_assert(!DEFER || MLO == MHI, "one order per full-warp kernel");
    int npend = 0;
    for (int64_t task = warp; task < ntask; task += nwarps) {
        const int q1 = (q0 + 1) & 3, q2 = (q0 + 2) & 3, q3 = (q0 + 3) & 3;
        // ring: offsets of task+2 (its block id landed one iteration ago), block id of task+3
        cp_async_wait_all();
        __syncwarp();                        // ring entries of other lanes (tile writers) visible
        {
            const int64_t t2 = task + 2 * nwarps, t3 = task + 3 * nwarps;
            if (writer(t2)) {
                const int g = tile_of(t2);
                const int32_t b2 = ring.blk[q2][g];
                if (b2 >= 0) {
                    cp_async8(&ring.lo[q2][g], val_off + b2);
                    cp_async8(&ring.vo[q2][g], vec_off + b2);
                }
            }
            if (writer(t3)) {
                const int g = tile_of(t3);
                int64_t idx = -1;
                if (t3 < ntask) task_order<NM>(t3, MLO, s_pref, s_first, s_last, idx);
                if (idx >= 0) cp_async4(&ring.blk[q3][g], order + idx);
                else ring.blk[q3][g] = -1;
            }
            cp_async_commit();
        }
        mbar_wait_warp(bar, parity);
        parity ^= 1u;
        const FTask cur = slot_task(task, q0);
        const StageNext<R> after_load{A, slot_task(task + nwarps, q1), S, bar};
        getrf_fast_dispatch<R, MLO, MHI, F, SOLVE>(A, cur, S, piv, info, safe_list, safe_count, b, x, sm,
                                                   after_load);
        if constexpr (DEFER) {
            __syncwarp();                            // sm.keep, L\U and perm of this task written
            const bool kept = cur.ok && smd.keep != 0;
            if (kept && lane == 0) {
                smd.plo[npend] = cur.lo;
                smd.pvo[npend] = cur.vo;
            }
            npend += kept ? 1 : 0;
            if (npend == 4) {
                __syncwarp();
                solve_pending<R, MLO>(A, piv, b, x, smd, npend);
                npend = 0;
            }
        }
        q0 = q1;
    }
    if constexpr (DEFER) {
        if (npend > 0) {
            __syncwarp();
            solve_pending<R, MLO>(A, piv, b, x, smd, npend);
        }
    }
    cp_async_wait_all();
    asm volatile("griddepcontrol.wait;" ::: "memory");
}

// Launch with programmatic stream serialization (PDL, see k_getrf_fast).
template <typename R, int MLO, int MHI, bool SOLVE>
bj_status launch_getrf_fast(R *A, const int64_t *val_off, const int64_t *vec_off, int32_t *piv, int32_t *info,
                            const PlanView &p, int32_t *safe_list, unsigned *safe_count, const R *b, R *x,
                            cudaStream_t s) {
    // sub-warp classes: the position-free output test (micro: 9..16 -1.5 %, 5..8 -2.5 %)
    auto kern = k_getrf_fast<R, MLO, MHI, (MLO == MHI ? fast_flags<R, MLO>() : (BJ_FAST_DEFAULT | kOut2)), SOLVE>;
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(persistent_grid(kern, kFastThreads, true));
    cfg.blockDim = dim3(kFastThreads);
    cfg.dynamicSmemBytes = 0;
    cfg.stream = s;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    BJ_CUDA_TRY(cudaLaunchKernelEx(&cfg, kern, A, val_off, vec_off, piv, info, (const int32_t *)p.order,
                                   (const int64_t *)p.bin_start, safe_list, safe_count, b, x));
    ::bj::count_launch();
    return BJ_OK;
}

// Safe path: blocks whose entries violate the fast path's precondition, or
// whose pivot search was ambiguous in the truncated key.  The plain algorithm
// of Fig. 1 bottom with the block in shared memory (row stride 33, lane r =
// row r, runtime m), explicit predication of pivoted rows, exact 64-bit pivot
// keys, IEEE division: bit-identical to the oracle for every input.  Rarely
// used, so it favours simplicity.
template <typename R>
__global__ void __launch_bounds__(128)
k_getrf_safe(R *A, const int32_t *__restrict__ sizes, const int64_t *__restrict__ val_off,
             const int64_t *__restrict__ vec_off, int32_t *__restrict__ piv, int32_t *__restrict__ info,
             const int32_t *__restrict__ list, const unsigned *__restrict__ count, const R *b = nullptr,
             R *x = nullptr) {
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
            // exact key (R2) by three warp reductions: the largest high word
            // of |v| among candidates (+1 so a zero candidate beats a
            // non-candidate), the largest low word among those, the lowest
            // lane among the maxima (R1)
            const bool cand = (tag == 0);
            const unsigned khi = cand ? Num<R>::key_hi(v) + 1u : 0u;
            const unsigned mhi = __reduce_max_sync(kFull, khi);
            const unsigned klo = (cand && khi == mhi) ? Num<R>::key_lo(v) : 0u;
            const unsigned mlo = __reduce_max_sync(kFull, klo);
            const unsigned who = (cand && khi == mhi && klo == mlo) ? (unsigned)r : 31u;
            const int ipiv = (int)__reduce_min_sync(kFull, who);
            const bool sing = (mhi == 1u) && (mlo == 0u);
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
        if (b != nullptr && r == 0) {
            // fused solve (bj_gesv_vbatched): plain scalar GETRS from the factors
            // just written (R8), same operations as the oracle's
            const int64_t vo = vec_off[blk];
            const int32_t *p = piv + vo;
            R v[kMaxM];
            for (int i = 0; i < m; ++i) v[i] = b[vo + p[i]];
            for (int k = 0; k + 1 < m; ++k)
                for (int i = k + 1; i < m; ++i) v[i] = Num<R>::fma(-Ab[i + k * m], v[k], v[i]);
            for (int k = m - 1; k >= 0; --k) {
                v[k] = Num<R>::div(v[k], Ab[k + k * m]);
                for (int i = 0; i < k; ++i) v[i] = Num<R>::fma(-Ab[i + k * m], v[k], v[i]);
            }
            for (int i = 0; i < m; ++i) x[vo + i] = v[i];
        }
        __syncwarp();
    }
}

}  // namespace bj
