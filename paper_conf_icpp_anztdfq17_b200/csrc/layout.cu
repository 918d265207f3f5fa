// layout.cu -- hot-path row a1: batch layout (vec_off / val_off scans) and the
// size-bucket plan (stable device counting sort of block ids by order m).
//
// The paper pads every block to 32 x 32; here blocks are packed
// back to back (16-byte aligned starts) and grouped by exact order so the
// size-specialised kernels never compute on padding.
#include "scan.cuh"
#include "internal.h"

namespace bj {

// ---------------------------------------------------------------- layout
struct SizesLayoutF {
    const int32_t *sizes;
    int64_t *vec, *val;
    int q;
    __device__ I64x2 value(int64_t i) const {
        long long m = max(sizes[i], 0);
        long long sq = m * m;
        return I64x2{m, (sq + q - 1) / q * q};
    }
    __device__ void store(int64_t i, I64x2 p) const { vec[i] = p.a; val[i] = p.b; }
    bj_status store_empty(cudaStream_t s) const {
        BJ_CUDA_TRY(cudaMemsetAsync(vec, 0, sizeof(int64_t), s));
        BJ_CUDA_TRY(cudaMemsetAsync(val, 0, sizeof(int64_t), s));
        return BJ_OK;
    }
};

struct BlockPtrLayoutF {
    const int32_t *bp;
    int32_t *sizes;
    int64_t *vec, *val;
    int64_t n;
    int q;
    __device__ I64x2 value(int64_t i) const {
        long long m = max(bp[i + 1] - bp[i], 0);
        long long sq = m * m;
        return I64x2{m, (sq + q - 1) / q * q};
    }
    __device__ void store(int64_t i, I64x2 p) const {
        vec[i] = p.a;
        val[i] = p.b;
        if (i < n) sizes[i] = bp[i + 1] - bp[i];
    }
    bj_status store_empty(cudaStream_t s) const {
        BJ_CUDA_TRY(cudaMemsetAsync(vec, 0, sizeof(int64_t), s));
        BJ_CUDA_TRY(cudaMemsetAsync(val, 0, sizeof(int64_t), s));
        return BJ_OK;
    }
};

bj_status layout_sizes(int64_t nb, const int32_t *sizes, int elem, int64_t *vec, int64_t *val,
                       cudaStream_t s) {
    return run_scan(SizesLayoutF{sizes, vec, val, 16 / elem}, nb, s);
}

bj_status layout_block_ptr(int64_t nb, const int32_t *bp, int elem, int32_t *sizes, int64_t *vec,
                           int64_t *val, cudaStream_t s) {
    return run_scan(BlockPtrLayoutF{bp, sizes, vec, val, nb, 16 / elem}, nb, s);
}

// ---------------------------------------------------------------- plan
// Tiles of kPlanTile consecutive blocks; per tile a histogram over the 34
// bins, a global (bin, tile) prefix, then a stable scatter.
constexpr int kPlanThreads = 256;
constexpr int kPlanRounds = 8;
constexpr int kPlanTile = kPlanThreads * kPlanRounds;

__global__ void __launch_bounds__(kPlanThreads)
k_plan_hist(const int32_t *__restrict__ sizes, int64_t n, int64_t *__restrict__ hist) {
    __shared__ int cnt[kBins];
    for (int i = threadIdx.x; i < kBins; i += blockDim.x) cnt[i] = 0;
    __syncthreads();
    const int64_t base = (int64_t)blockIdx.x * kPlanTile;
    for (int j = 0; j < kPlanRounds; ++j) {
        int64_t i = base + j * kPlanThreads + threadIdx.x;
        if (i < n) atomicAdd(&cnt[size_bin(sizes[i])], 1);
    }
    __syncthreads();
    for (int b = threadIdx.x; b < kBins; b += blockDim.x) hist[(int64_t)blockIdx.x * kBins + b] = cnt[b];
}

// Single CTA, one warp per bin.  Pass 1: bin totals (each lane sums a
// strided subset of the tiles, warp reduction) -> bin starts.  Pass 2:
// exclusive scan of hist[.][bin] over the tiles starting at the bin's start,
// so hist becomes the absolute start of (tile, bin) in `order` directly.
__global__ void __launch_bounds__(1024) k_plan_offsets(int64_t *hist, int64_t ntiles, int64_t *bin_start) {
    __shared__ int64_t tot[kBins];
    __shared__ int64_t base[kBins + 1];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, nw = blockDim.x >> 5;
    for (int b = w; b < kBins; b += nw) {
        int64_t acc = 0;
        for (int64_t T0 = 0; T0 < ntiles; T0 += 32 * 16) {    // 16 independent loads in flight per lane
            int64_t cs[16];
#pragma unroll
            for (int j = 0; j < 16; ++j) {
                const int64_t t = T0 + 32 * j + lane;
                cs[j] = t < ntiles ? hist[t * kBins + b] : 0;
            }
#pragma unroll
            for (int j = 0; j < 16; ++j) acc += cs[j];
        }
#pragma unroll
        for (int off = 16; off >= 1; off >>= 1) acc += __shfl_xor_sync(kFull, acc, off);
        if (lane == 0) tot[b] = acc;
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        int64_t s = 0;
        for (int i = 0; i < kBins; ++i) {
            base[i] = s;
            bin_start[i] = s;
            s += tot[i];
        }
        bin_start[kBins] = s;
    }
    __syncthreads();
    constexpr int kAhead = 16;       // 32-tile chunks whose counts are loaded before the scans
    for (int b = w; b < kBins; b += nw) {
        int64_t carry = base[b];
        for (int64_t T0 = 0; T0 < ntiles; T0 += 32 * kAhead) {
            int64_t cs[kAhead];
#pragma unroll
            for (int j = 0; j < kAhead; ++j) {
                const int64_t t = T0 + 32 * j + lane;
                cs[j] = t < ntiles ? hist[t * kBins + b] : 0;
            }
#pragma unroll
            for (int j = 0; j < kAhead; ++j) {
                const int64_t t = T0 + 32 * j + lane;
                const int64_t c = cs[j];
                int64_t inc = c;
#pragma unroll
                for (int off = 1; off < 32; off <<= 1) {
                    const int64_t v = __shfl_up_sync(kFull, inc, off);
                    if (lane >= off) inc += v;
                }
                if (t < ntiles) hist[t * kBins + b] = carry + inc - c;
                carry += __shfl_sync(kFull, inc, 31);
            }
        }
    }
}

__global__ void __launch_bounds__(kPlanThreads)
k_plan_scatter(const int32_t *__restrict__ sizes, int64_t n, const int64_t *__restrict__ tile_off,
               int32_t *__restrict__ order) {
    constexpr int NW = kPlanThreads / 32;
    __shared__ int64_t run[kBins];               // offset of the next item of each bin
    __shared__ int rtot[kBins];
    __shared__ int wpre[NW][kBins];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    for (int b = threadIdx.x; b < kBins; b += blockDim.x) run[b] = tile_off[(int64_t)blockIdx.x * kBins + b];
    const int64_t base = (int64_t)blockIdx.x * kPlanTile;
    const unsigned lt = (1u << lane) - 1u;
    for (int j = 0; j < kPlanRounds; ++j) {
        for (int b = threadIdx.x; b < NW * kBins; b += blockDim.x) (&wpre[0][0])[b] = 0;
        __syncthreads();
        const int64_t i = base + (int64_t)j * kPlanThreads + threadIdx.x;
        const int bin = i < n ? size_bin(sizes[i]) : -1;
        const unsigned peers = __match_any_sync(kFull, bin);
        const int rank = __popc(peers & lt);     // stable rank inside the warp
        if (bin >= 0 && rank == 0) wpre[w][bin] = __popc(peers);
        __syncthreads();
        if (threadIdx.x < kBins) {               // exclusive prefix over warps, per bin
            const int b = threadIdx.x;
            int acc = 0;
            for (int ww = 0; ww < NW; ++ww) {
                const int c = wpre[ww][b];
                wpre[ww][b] = acc;
                acc += c;
            }
            rtot[b] = acc;
        }
        __syncthreads();
        if (bin >= 0) order[run[bin] + wpre[w][bin] + rank] = (int32_t)i;
        __syncthreads();
        if (threadIdx.x < kBins) run[threadIdx.x] += rtot[threadIdx.x];
    }
}

bj_status build_plan(int64_t nb, const int32_t *sizes, int32_t *order, int64_t *bin_start,
                     cudaStream_t s) {
    if (nb == 0) {
        BJ_CUDA_TRY(cudaMemsetAsync(bin_start, 0, sizeof(int64_t) * (kBins + 1), s));
        return BJ_OK;
    }
    const int64_t ntiles = (nb + kPlanTile - 1) / kPlanTile;
    AsyncScratch scratch(s);                 // released on every return path
    BJ_CUDA_TRY(cudaMallocAsync((void **)&scratch.p, sizeof(int64_t) * kBins * ntiles, s));
    int64_t *hist = reinterpret_cast<int64_t *>(scratch.p);
    k_plan_hist<<<(unsigned)ntiles, kPlanThreads, 0, s>>>(sizes, nb, hist);
    BJ_LAUNCH_CHECK();
    k_plan_offsets<<<1, 1024, 0, s>>>(hist, ntiles, bin_start);
    BJ_LAUNCH_CHECK();
    k_plan_scatter<<<(unsigned)ntiles, kPlanThreads, 0, s>>>(sizes, nb, hist, order);
    BJ_LAUNCH_CHECK();
    return BJ_OK;
}

}  // namespace bj
