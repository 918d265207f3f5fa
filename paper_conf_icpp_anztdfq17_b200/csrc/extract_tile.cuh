#pragma once
// extract_tile.cuh -- hot-path row a2, the per-block extraction step shared by
// bj_extract (extract.cu) and the fused setup (setup_fused.cuh): section III.C
// (Fig. 3), warp-cooperative scan of one diagonal block's CSR rows
// into a zero-filled shared-memory tile.
#include <climits>

#include "common.cuh"

namespace bj {

constexpr int64_t kHeavy = 8192;     // stored entries per block above which the CTA path is used

// One diagonal block (rows bs..be-1, m = be - bs in 1..32, entries
// [e0, e1) of the CSR, at most kHeavy) extracted by one warp into the
// zero-filled shared-memory tile T (column-major, leading dimension m).
// rpv: lane j < m holds row_ptr[bs + j].  Shared with the fused setup kernel
// (getrf_fused.cu), which factors the tile in place of a staged block.
template <typename R>
__device__ __forceinline__ void extract_block_warp(const int32_t *__restrict__ col_idx, const R *__restrict__ values,
                                                   int64_t col_offset, int bs, int m, int64_t rpv, int64_t e0,
                                                   int64_t e1, R *T) {
    const int lane = threadIdx.x & 31;
    const int be = bs + m;
    const int q = 16 / (int)sizeof(R);
    const int np = (m * m + q - 1) / q * q;
    for (int i = lane; i < np; i += 32) T[i] = R(0);
    __syncwarp();
    const int64_t cb = (int64_t)bs + col_offset, ce = (int64_t)be + col_offset;
    // The block's rows are one contiguous entry range [e0, e1): the warp
    // scans it in 32-entry chunks (coalesced col-indices),
    // kU chunks per round so kU loads per lane are in flight, and the
    // value loads of one round overlap the col-index loads of the next.
    // Row of entry e: rows starting at or before the chunk start (ballot)
    // plus row starts inside the chunk at or before e (one REDUX.OR mask).
    const int rel = lane < m ? (int)(rpv - e0) : INT_MAX;   // row start, relative
    const int len = (int)(e1 - e0);
    // The row-start mask counts each start position once, so a block with
    // an empty row (two rows starting at the same entry) takes the plain
    // row-by-row scan instead (rare: FEM-like matrices have none).
    const int rel_next = __shfl_down_sync(kFull, rel, 1);
    const bool has_empty = __any_sync(kFull, lane < m && (lane + 1 < m ? rel_next == rel : rel == len));
    if (has_empty) {
        for (int r = 0; r < m; ++r) {
            const int rs = __shfl_sync(kFull, rel, r);
            const int re = r + 1 < m ? __shfl_sync(kFull, rel, r + 1) : len;
            for (int e = rs + lane; e < re; e += 32) {
                const int64_t c = __ldg(col_idx + e0 + e);
                if (c >= cb && c < ce) T[r + (int)(c - cb) * m] = __ldg(values + e0 + e);
            }
        }
    } else {
        const int nch = (len + 31) >> 5;
        constexpr int kU = 8;
        int32_t cc[kU];
        auto load_cols = [&](int c0) {
#pragma unroll
            for (int u = 0; u < kU; ++u) {
                const int e = ((c0 + u) << 5) + lane;
                cc[u] = e < len ? __ldg(col_idx + e0 + e) : -1;
            }
        };
        load_cols(0);
        for (int c0 = 0; c0 < nch; c0 += kU) {
            int32_t cv[kU];
#pragma unroll
            for (int u = 0; u < kU; ++u) cv[u] = cc[u];
            if (c0 + kU < nch) load_cols(c0 + kU);
            // all value loads of the round first (in-order issue: a store that
            // waits on its load would otherwise serialise the chunks), then
            // the scatter into the smem tile
            R vv[kU];
            int at[kU];
#pragma unroll
            for (int u = 0; u < kU; ++u) {
                const int E = (c0 + u) << 5;
                at[u] = -1;
                if (E < len) {                                        // warp-uniform
                    const int row0 = __popc(__ballot_sync(kFull, rel <= E)) - 1;
                    const unsigned starts =
                        __reduce_or_sync(kFull, (rel > E && rel < E + 32) ? 1u << (rel - E) : 0u);
                    const int row = row0 + __popc(starts & ((2u << lane) - 1u));
                    const int64_t c = cv[u];
                    if (c >= cb && c < ce) {
                        at[u] = row + (int)(c - cb) * m;
                        vv[u] = __ldg(values + e0 + E + lane);
                    }
                }
            }
#pragma unroll
            for (int u = 0; u < kU; ++u)
                if (at[u] >= 0) T[at[u]] = vv[u];
        }
    }
    __syncwarp();
}

}  // namespace bj
