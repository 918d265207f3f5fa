// supervar.cu -- supervariable blocking on the GPU:
// CSR sparsity pattern -> block_ptr of the block-Jacobi diagonal blocks.
//
// PAPER.md section II.A, P:186-193 (supervariables = variables sharing the same
// column-nonzero pattern; adjacent supervariables clustered up to an upper
// bound on the block size) and P:837-843 (the experiments vary only that
// bound).  The clustering rule is unstated; readings R20-R22:
// consecutive rows with identical stored column sequences form a supervariable
// (R20); supervariables longer than the bound are cut into bound-row pieces
// plus a remainder (R22); pieces are clustered greedily in row order (R21).
//
// GPU formulation (none of it is in the paper):
//   1. k_sv_flags: one warp per row compares the row's column sequence with
//      the previous row's (coalesced 32-wide chunks, ballot) -> svpos[i] = i at
//      a supervariable start, else 0.
//   2. inclusive max-scan -> svstart[i] (start row of i's supervariable).
//   3. k_unit_pos: unit boundary at i iff (i - svstart[i]) % bound == 0 (R22);
//      unit[n] = n.  Inclusive max-scan -> prevB[x] = largest boundary <= x.
//   4. The greedy walk (R21) is the chain p -> next(p) = prevB[min(p+bound, n)]
//      from p = 0 (every unit has <= bound rows, so next(p) > p).  Rows are cut
//      into segments of kSegRows.  The chain enters segment t at an offset
//      e in [0, bound) (the previous node is < t*kSegRows and next() advances
//      at most `bound` rows), so k_sv_table lets lane e of warp t walk the
//      segment from t*kSegRows + e and record (exit offset, node count): the
//      segment's transfer function for every possible entry.
//   5. k_sv_compose (one CTA) composes the transfer functions in row order
//      from entry 0 -- a table lookup per segment, staged through shared
//      memory -- giving each segment's true entry and node count.  (Chains
//      from different starts need not merge -- uniform 3-row supervariables
//      give parallel chains -- so guessing entries and iterating is O(nseg)
//      passes; the tables make it one pass.)
//   6. exclusive sum of the per-segment counts, then each segment re-walks
//      from its entry and writes its nodes into block_ptr.
#include <cub/cub.cuh>

#include "common.cuh"
#include "internal.h"

namespace bj {

namespace {

constexpr int kSegRows = 2048;
constexpr int kComposeSegs = 256;   // segments staged per shared-memory chunk
constexpr int kFlagThreads = 256;

struct MaxI32 {
    __device__ __forceinline__ int32_t operator()(int32_t a, int32_t b) const { return a > b ? a : b; }
};

__global__ void k_sv_flags(const int64_t *__restrict__ row_ptr, const int32_t *__restrict__ col_idx, int32_t n,
                           int32_t *__restrict__ svpos) {
    const int lane = threadIdx.x & 31;
    const int64_t warps = (int64_t)gridDim.x * (blockDim.x >> 5);
    for (int64_t i = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; i < n; i += warps) {
        bool start = (i == 0);
        if (!start) {
            const int64_t a0 = row_ptr[i - 1], a1 = row_ptr[i], a2 = row_ptr[i + 1];
            const int64_t len = a2 - a1;
            if (len != a1 - a0) {
                start = true;
            } else {
                // no early exit: every chunk's loads are independent and in flight together
                bool diff = false;
#pragma unroll 4
                for (int64_t k = lane; k < len; k += 32) diff |= __ldg(col_idx + a0 + k) != __ldg(col_idx + a1 + k);
                start = __any_sync(kFull, diff);
            }
        }
        if (lane == 0) svpos[i] = start ? (int32_t)i : 0;
    }
}

__global__ void k_unit_pos(const int32_t *__restrict__ svstart, int32_t n, int32_t bound,
                           int32_t *__restrict__ unit) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i <= n; i += (int64_t)gridDim.x * blockDim.x)
        unit[i] = (i == n || ((int32_t)i - svstart[i]) % bound == 0) ? (int32_t)i : 0;
}

// Segment t covers rows [t*kSegRows, (t+1)*kSegRows): write the chain nodes
// from its entry at off[t]; the last segment appends block_ptr[nb] = n.
__global__ void k_sv_walk(const int32_t *__restrict__ prevB, int32_t n, int32_t bound, int32_t nseg,
                          const int32_t *__restrict__ entry, const int32_t *__restrict__ off,
                          int32_t *__restrict__ block_ptr) {
    const int32_t t = blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= nseg) return;
    const int64_t end64 = (int64_t)(t + 1) * kSegRows;
    const int32_t end = end64 < n ? (int32_t)end64 : n;
    int32_t p = entry[t], c = 0;
    int32_t *dst = block_ptr + off[t];
    while (p < end) {
        dst[c++] = p;
        const int64_t q = (int64_t)p + bound;
        p = prevB[q < n ? q : n];
    }
    if (t == nseg - 1) dst[c] = n;
}

// Lane e of warp t walks segment t from row t*kSegRows + e (e < bound);
// table[t*32 + e] = (node count << 8) | exit offset into segment t+1.
__global__ void k_sv_table(const int32_t *__restrict__ prevB, int32_t n, int32_t bound, int32_t nseg,
                           int32_t *__restrict__ table) {
    const int lane = threadIdx.x & 31;
    const int64_t t = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    if (t >= nseg || lane >= bound) return;
    const int64_t base = t * kSegRows, end64 = base + kSegRows;
    const int32_t end = end64 < n ? (int32_t)end64 : n;
    int32_t p = (int32_t)(base + lane), c = 0;
    while (p < end) {
        ++c;
        const int64_t q = (int64_t)p + bound;
        p = prevB[q < n ? q : n];
    }
    table[t * 32 + lane] = (c << 8) | (int32_t)(p - end);   // p - end < bound
}

// One CTA: compose the segment transfer functions from entry offset 0.
__global__ void k_sv_compose(const int32_t *__restrict__ table, int32_t nseg, int32_t *__restrict__ entry,
                             int32_t *__restrict__ count) {
    __shared__ int32_t tab[kComposeSegs * 32];
    int32_t e = 0;   // valid in thread 0
    for (int64_t t0 = 0; t0 < nseg; t0 += kComposeSegs) {
        const int32_t nt = (int32_t)((nseg - t0) < kComposeSegs ? (nseg - t0) : kComposeSegs);
        __syncthreads();
        for (int i = threadIdx.x; i < nt * 32; i += blockDim.x) tab[i] = table[t0 * 32 + i];
        __syncthreads();
        if (threadIdx.x == 0) {
            for (int32_t k = 0; k < nt; ++k) {
                const int32_t v = tab[k * 32 + e];
                entry[t0 + k] = (int32_t)((t0 + k) * kSegRows) + e;
                count[t0 + k] = v >> 8;
                e = v & 0xff;
            }
        }
    }
}

}  // namespace

bj_status supervariable_run(const bj_csr &A, int32_t bound, int32_t *block_ptr, int64_t *nblocks_h,
                            cudaStream_t s) {
    const int32_t n = (int32_t)A.nrows;
    if (n == 0) {
        BJ_CUDA_TRY(cudaMemsetAsync(block_ptr, 0, sizeof(int32_t), s));
        BJ_CUDA_TRY(cudaStreamSynchronize(s));
        *nblocks_h = 0;
        return BJ_OK;
    }
    const int32_t nseg = (int32_t)((n + (int64_t)kSegRows - 1) / kSegRows);
    // scratch: svpos/unit/table [n+1], svstart/prevB [n+1], entry, count, off [nseg]
    size_t scan_bytes = 0, sum_bytes = 0;
    cub::DeviceScan::InclusiveScan(nullptr, scan_bytes, (int32_t *)nullptr, (int32_t *)nullptr, MaxI32(), n + 1, s);
    cub::DeviceScan::ExclusiveSum(nullptr, sum_bytes, (int32_t *)nullptr, (int32_t *)nullptr, nseg, s);
    const size_t tmp_bytes = (scan_bytes > sum_bytes ? scan_bytes : sum_bytes) + 256;
    const size_t vec_bytes = ((sizeof(int32_t) * ((size_t)n + 1) + 255) / 256) * 256;
    const size_t seg_bytes = ((sizeof(int32_t) * (size_t)nseg + 255) / 256) * 256;
    char *scratch = nullptr;
    BJ_CUDA_TRY(cudaMallocAsync((void **)&scratch, 2 * vec_bytes + 3 * seg_bytes + 256 + tmp_bytes, s));
    int32_t *a = reinterpret_cast<int32_t *>(scratch);
    int32_t *b = reinterpret_cast<int32_t *>(scratch + vec_bytes);
    int32_t *entry = reinterpret_cast<int32_t *>(scratch + 2 * vec_bytes);
    int32_t *count = reinterpret_cast<int32_t *>(scratch + 2 * vec_bytes + seg_bytes);
    int32_t *off = reinterpret_cast<int32_t *>(scratch + 2 * vec_bytes + 2 * seg_bytes);
    void *tmp = scratch + 2 * vec_bytes + 3 * seg_bytes + 256;
    bj_status st = BJ_OK;
    int32_t h_last[2] = {0, 0};
    const int grid = 8 * sm_count();   // 64 warps per SM for the latency-bound row compare
    const int sgrid = (nseg + 127) / 128;

    k_sv_flags<<<grid, kFlagThreads, 0, s>>>(A.row_ptr, A.col_idx, n, a);
    BJ_LAUNCH_CHECK();
    if (cub::DeviceScan::InclusiveScan(tmp, scan_bytes, a, b, MaxI32(), n, s) != cudaSuccess) st = BJ_ERR_CUDA;
    k_unit_pos<<<grid, 256, 0, s>>>(b, n, bound, a);
    BJ_LAUNCH_CHECK();
    if (cub::DeviceScan::InclusiveScan(tmp, scan_bytes, a, b, MaxI32(), n + 1, s) != cudaSuccess) st = BJ_ERR_CUDA;
    k_sv_table<<<(int)(((int64_t)nseg * 32 + 127) / 128), 128, 0, s>>>(b, n, bound, nseg, a);
    BJ_LAUNCH_CHECK();
    k_sv_compose<<<1, 1024, 0, s>>>(a, nseg, entry, count);
    BJ_LAUNCH_CHECK();
    if (st == BJ_OK && cub::DeviceScan::ExclusiveSum(tmp, sum_bytes, count, off, nseg, s) != cudaSuccess)
        st = BJ_ERR_CUDA;
    if (st == BJ_OK) {
        k_sv_walk<<<sgrid, 128, 0, s>>>(b, n, bound, nseg, entry, off, block_ptr);
        BJ_LAUNCH_CHECK();
        if (cudaMemcpyAsync(&h_last[0], off + (nseg - 1), sizeof(int32_t), cudaMemcpyDeviceToHost, s) != cudaSuccess ||
            cudaMemcpyAsync(&h_last[1], count + (nseg - 1), sizeof(int32_t), cudaMemcpyDeviceToHost, s) !=
                cudaSuccess)
            st = BJ_ERR_CUDA;
    }
    if (cudaFreeAsync(scratch, s) != cudaSuccess) st = BJ_ERR_CUDA;
    if (cudaStreamSynchronize(s) != cudaSuccess) st = BJ_ERR_CUDA;
    if (st == BJ_OK) *nblocks_h = (int64_t)h_last[0] + h_last[1];
    return st;
}

}  // namespace bj
