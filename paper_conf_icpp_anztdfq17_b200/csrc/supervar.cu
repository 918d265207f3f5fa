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
//      from p = 0 (every unit has <= bound rows, so next(p) > p).  The rows
//      are cut into segments of kSegRows; one thread walks each segment from
//      a guessed entry node, and the exit node of segment t becomes the entry
//      of t+1.  Iterated to a fixpoint (entry[0] = 0 is exact, so by induction
//      the fixpoint is the true chain; chains from different starts merge
//      quickly because next() is monotone, so 2 passes are typical).
//   5. exclusive sum of per-segment node counts, then each segment writes its
//      nodes into block_ptr.
#include <cub/cub.cuh>

#include "common.cuh"
#include "internal.h"

namespace bj {

namespace {

constexpr int kSegRows = 512;
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
                for (int64_t k = lane; k - lane < len; k += 32) {
                    const bool diff = k < len && col_idx[a0 + k] != col_idx[a1 + k];
                    if (__any_sync(kFull, diff)) { start = true; break; }
                }
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

// Segment t covers rows [t*kSegRows, (t+1)*kSegRows).  Walks the chain from
// entry[t]; the first node >= the segment end is the entry of segment t+1.
// write == nullptr: fixpoint pass (counts + exits); else write the nodes.
__global__ void k_sv_walk(const int32_t *__restrict__ prevB, int32_t n, int32_t bound, int32_t nseg,
                          const int32_t *entry, int32_t *entry_next,   // may alias (in-place pass)
                          int32_t *__restrict__ count, int32_t *__restrict__ changed,
                          const int32_t *__restrict__ off, int32_t *__restrict__ block_ptr) {
    const int32_t t = blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= nseg) return;
    const int64_t end64 = (int64_t)(t + 1) * kSegRows;
    const int32_t end = end64 < n ? (int32_t)end64 : n;
    int32_t p = entry[t], c = 0;
    int32_t *dst = block_ptr ? block_ptr + off[t] : nullptr;
    while (p < end) {
        if (dst) dst[c] = p;
        ++c;
        const int64_t q = (int64_t)p + bound;
        p = prevB[q < n ? q : n];
    }
    if (!block_ptr) {
        count[t] = c;
        if (t + 1 < nseg) {
            if (entry_next[t + 1] != p) { entry_next[t + 1] = p; *changed = 1; }
        }
    } else if (t == nseg - 1) {
        block_ptr[off[t] + c] = n;
    }
}

// Initial guess of segment entries: a boundary node in [t*kSegRows, +bound].
__global__ void k_sv_guess(const int32_t *__restrict__ prevB, int32_t n, int32_t bound, int32_t nseg,
                           int32_t *__restrict__ entry) {
    const int32_t t = blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= nseg) return;
    if (t == 0) { entry[0] = 0; return; }
    const int64_t q = (int64_t)t * kSegRows + bound;
    entry[t] = prevB[q < n ? q : n];
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
    // scratch: svpos/unit [n+1], svstart/prevB [n+1], entry, count, off [nseg], changed
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
    int32_t *changed = reinterpret_cast<int32_t *>(scratch + 2 * vec_bytes + 3 * seg_bytes);
    void *tmp = scratch + 2 * vec_bytes + 3 * seg_bytes + 256;
    bj_status st = BJ_OK;
    int32_t h_changed = 1, h_last[2] = {0, 0};
    const int grid = 4 * sm_count();
    const int sgrid = (nseg + 127) / 128;

    k_sv_flags<<<grid, kFlagThreads, 0, s>>>(A.row_ptr, A.col_idx, n, a);
    BJ_LAUNCH_CHECK();
    if (cub::DeviceScan::InclusiveScan(tmp, scan_bytes, a, b, MaxI32(), n, s) != cudaSuccess) st = BJ_ERR_CUDA;
    k_unit_pos<<<grid, 256, 0, s>>>(b, n, bound, a);
    BJ_LAUNCH_CHECK();
    if (cub::DeviceScan::InclusiveScan(tmp, scan_bytes, a, b, MaxI32(), n + 1, s) != cudaSuccess) st = BJ_ERR_CUDA;
    k_sv_guess<<<sgrid, 128, 0, s>>>(b, n, bound, nseg, entry);
    BJ_LAUNCH_CHECK();
    for (int it = 0; st == BJ_OK && h_changed && it <= nseg; ++it) {
        if (cudaMemsetAsync(changed, 0, sizeof(int32_t), s) != cudaSuccess) { st = BJ_ERR_CUDA; break; }
        // entries are updated in place: a pass may read an entry a neighbour
        // just fixed, which only speeds convergence; the fixpoint is the same.
        k_sv_walk<<<sgrid, 128, 0, s>>>(b, n, bound, nseg, entry, entry, count, changed, nullptr, nullptr);
        BJ_LAUNCH_CHECK();
        if (cudaMemcpyAsync(&h_changed, changed, sizeof(int32_t), cudaMemcpyDeviceToHost, s) != cudaSuccess ||
            cudaStreamSynchronize(s) != cudaSuccess) { st = BJ_ERR_CUDA; break; }
    }
    if (st == BJ_OK) {
        if (cub::DeviceScan::ExclusiveSum(tmp, sum_bytes, count, off, nseg, s) != cudaSuccess) st = BJ_ERR_CUDA;
    }
    if (st == BJ_OK) {
        k_sv_walk<<<sgrid, 128, 0, s>>>(b, n, bound, nseg, entry, entry, count, changed, off, block_ptr);
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
