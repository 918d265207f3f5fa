// scan.cuh -- device exclusive scans used by the layout / plan / synth steps.
// Three-phase reduce-then-scan over tiles of 2048 items (256 threads x 8).
// Two int64 sequences are scanned at once (vec_off and val_off of a1).
#pragma once

#include "common.cuh"

namespace bj {

constexpr int kScanThreads = 256;
constexpr int kScanItems = 8;
constexpr int kScanTile = kScanThreads * kScanItems;

struct I64x2 { long long a, b; };

__device__ __forceinline__ I64x2 add2(I64x2 x, I64x2 y) { return {x.a + y.a, x.b + y.b}; }

// Block-wide exclusive scan of one I64x2 per thread; returns the exclusive
// prefix and sets `total` (every thread) to the block total.
__device__ __forceinline__ I64x2 block_exclusive_scan(I64x2 v, I64x2 &total) {
    constexpr int NW = kScanThreads / 32;
    __shared__ I64x2 warp_sums[NW + 1];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    I64x2 inc = v;
#pragma unroll
    for (int off = 1; off < 32; off <<= 1) {
        long long a = __shfl_up_sync(kFull, inc.a, off);
        long long b = __shfl_up_sync(kFull, inc.b, off);
        if (lane >= off) { inc.a += a; inc.b += b; }
    }
    if (lane == 31) warp_sums[w] = inc;
    __syncthreads();
    if (threadIdx.x == 0) {
        I64x2 acc{0, 0};
        for (int i = 0; i < NW; ++i) {
            I64x2 t = warp_sums[i];
            warp_sums[i] = acc;
            acc = add2(acc, t);
        }
        warp_sums[NW] = acc;
    }
    __syncthreads();
    const I64x2 base = warp_sums[w];
    total = warp_sums[NW];
    __syncthreads();
    return I64x2{base.a + inc.a - v.a, base.b + inc.b - v.b};
}

template <class F>
__global__ void __launch_bounds__(kScanThreads) k_scan_reduce(F f, int64_t n, I64x2 *partial) {
    I64x2 tot;
    const int64_t base = (int64_t)blockIdx.x * kScanTile + (int64_t)threadIdx.x * kScanItems;
    I64x2 s{0, 0};
#pragma unroll
    for (int j = 0; j < kScanItems; ++j) {
        int64_t i = base + j;
        if (i < n) s = add2(s, f.value(i));
    }
    block_exclusive_scan(s, tot);
    if (threadIdx.x == 0) partial[blockIdx.x] = tot;
}

// Single CTA: exclusive scan of the tile partials in place.
static __global__ void __launch_bounds__(kScanThreads) k_scan_partials(I64x2 *partial, int64_t ntiles) {
    I64x2 tot;
    I64x2 carry{0, 0};
    for (int64_t c0 = 0; c0 < ntiles; c0 += kScanThreads) {
        int64_t i = c0 + threadIdx.x;
        I64x2 v = i < ntiles ? partial[i] : I64x2{0, 0};
        I64x2 ex = block_exclusive_scan(v, tot);
        if (i < ntiles) partial[i] = add2(ex, carry);
        carry = add2(carry, tot);
    }
}

template <class F>
__global__ void __launch_bounds__(kScanThreads) k_scan_down(F f, int64_t n, const I64x2 *partial) {
    // Thread t scans items t*8 .. t*8+7 of the tile; the prefixes go through
    // shared memory so the stores of vec/val are coalesced (consecutive
    // threads -> consecutive items) instead of 8-element strided.
    __shared__ long long oa[kScanTile], ob[kScanTile];
    I64x2 tot;
    const int64_t tile0 = (int64_t)blockIdx.x * kScanTile;
    const int64_t base = tile0 + (int64_t)threadIdx.x * kScanItems;
    I64x2 v[kScanItems];
    I64x2 s{0, 0};
#pragma unroll
    for (int j = 0; j < kScanItems; ++j) {
        int64_t i = base + j;
        v[j] = i < n ? f.value(i) : I64x2{0, 0};
        s = add2(s, v[j]);
    }
    I64x2 ex = add2(block_exclusive_scan(s, tot), partial[blockIdx.x]);
#pragma unroll
    for (int j = 0; j < kScanItems; ++j) {
        oa[threadIdx.x * kScanItems + j] = ex.a;
        ob[threadIdx.x * kScanItems + j] = ex.b;
        if (base + j == n - 1) f.store(n, add2(ex, v[j]));      // totals
        ex = add2(ex, v[j]);
    }
    __syncthreads();
    for (int k = threadIdx.x; k < kScanTile; k += kScanThreads) {
        const int64_t i = tile0 + k;
        if (i < n) f.store(i, I64x2{oa[k], ob[k]});
    }
}

// Host driver: exclusive scan of f.value(0..n-1) written through f.store(i,
// prefix) for i = 0..n (f.store(n, totals) receives the totals).  Scratch is
// stream-ordered (cudaMallocAsync).
template <class F>
bj_status run_scan(F f, int64_t n, cudaStream_t s) {
    if (n == 0) return f.store_empty(s);
    const int64_t ntiles = (n + kScanTile - 1) / kScanTile;
    AsyncScratch scratch(s);                 // released on every return path
    BJ_CUDA_TRY(cudaMallocAsync((void **)&scratch.p, sizeof(I64x2) * ntiles, s));
    I64x2 *partial = reinterpret_cast<I64x2 *>(scratch.p);
    k_scan_reduce<F><<<(unsigned)ntiles, kScanThreads, 0, s>>>(f, n, partial);
    BJ_LAUNCH_CHECK();
    k_scan_partials<<<1, kScanThreads, 0, s>>>(partial, ntiles);
    BJ_LAUNCH_CHECK();
    k_scan_down<F><<<(unsigned)ntiles, kScanThreads, 0, s>>>(f, n, partial);
    BJ_LAUNCH_CHECK();
    return BJ_OK;
}

}  // namespace bj
