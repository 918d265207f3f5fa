// extract.cu -- hot-path row a2: CSR -> dense diagonal blocks, section III.C
// (Fig. 3).
//
// As in the paper, all lanes of a warp cooperate on one row at a time so the
// col-indices are read coalesced, and hits are staged in shared memory
// (P:594-603).  B200 changes:
//  * a warp owns a whole diagonal block: its smem tile is zero-filled, hits are
//    scattered into it, and the finished block (incl. the 16-B pad) is written
//    with 16-byte stores -> the dense output is written exactly once, no
//    separate zero-fill pass over HBM;
//  * load balance for skewed rows: blocks whose rows hold more than
//    kHeavy stored entries are deferred to a second kernel in which a whole CTA
//    (256 threads) scans the block's entry range, each thread locating its row
//    by binary search over the block's row pointers in smem;
//  * persistent grid, blocks taken in row order (streaming CSR reads).
#include "common.cuh"
#include "internal.h"
#include "extract_tile.cuh"

namespace bj {

constexpr int kExtractWarps = 4;
constexpr int kExtractThreads = 32 * kExtractWarps;
constexpr int kHeavyThreads = 256;

template <typename R>
__device__ __forceinline__ void write_tile(R *__restrict__ dst, const R *src, int nelem_padded) {
    // nelem_padded * sizeof(R) is a multiple of 16 and dst is 16-B aligned.
    const int n16 = nelem_padded * (int)sizeof(R) / 16;
    const int4 *s4 = reinterpret_cast<const int4 *>(src);
    int4 *d4 = reinterpret_cast<int4 *>(dst);
    for (int i = threadIdx.x & 31; i < n16; i += 32) d4[i] = s4[i];
}

// mlo_skip: blocks of order >= mlo_skip (and at most kHeavy entries) are left
// to the fused setup kernel (0 = extract every block).
template <typename R>
__global__ void __launch_bounds__(kExtractThreads)
k_extract_warp(const int64_t *__restrict__ row_ptr, const int32_t *__restrict__ col_idx,
               const R *__restrict__ values, int64_t col_offset, const int32_t *__restrict__ block_ptr,
               int64_t nb, const int64_t *__restrict__ val_off, R *__restrict__ out,
               int32_t *__restrict__ heavy, unsigned long long *__restrict__ nheavy, int mlo_skip) {
    __shared__ __align__(16) R tile[kExtractWarps][kMaxM * kMaxM];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    R *T = tile[w];
    const int64_t nwarps = ((int64_t)gridDim.x * kExtractThreads) >> 5;
    // Block descriptors are pipelined across iterations: block_ptr two blocks
    // ahead, row_ptr one block ahead, so a block's scan starts without
    // waiting on its index chain.
    const int64_t b0 = __reduce_max_sync(kFull, (unsigned)(((int64_t)blockIdx.x * kExtractThreads + threadIdx.x) >> 5));
    auto ld_bp = [&](int64_t b, int &bs, int &be) {
        bs = b < nb ? __ldg(block_ptr + b) : 0;
        be = b < nb ? __ldg(block_ptr + b + 1) : 0;
    };
    auto ld_rp = [&](int bs, int be, int64_t &rpv, int64_t &e1) {
        const int m = be - bs;
        rpv = (m > 0 && m <= kMaxM && lane < m) ? __ldg(row_ptr + bs + lane) : 0;
        e1 = (m > 0 && m <= kMaxM) ? __ldg(row_ptr + be) : 0;
    };
    int n_bs, n_be, nn_bs, nn_be;
    int64_t n_rpv, n_e1;
    ld_bp(b0, n_bs, n_be);
    ld_rp(n_bs, n_be, n_rpv, n_e1);
    ld_bp(b0 + nwarps, nn_bs, nn_be);
    for (int64_t b = b0; b < nb; b += nwarps) {
        const int bs = n_bs, be = n_be;
        const int64_t rpv = n_rpv, e1 = n_e1;
        n_bs = nn_bs;
        n_be = nn_be;
        ld_rp(n_bs, n_be, n_rpv, n_e1);
        ld_bp(b + 2 * nwarps, nn_bs, nn_be);
        const int m = be - bs;
        if (m <= 0 || m > kMaxM) continue;                     // nothing to write / invalid order
        // lane j < m holds row_ptr[bs + j]; every lane holds row_ptr[be]
        const int64_t e0 = __shfl_sync(kFull, rpv, 0);
        if (e1 - e0 > kHeavy) {
            if (lane == 0) heavy[atomicAdd(nheavy, 1ull)] = (int32_t)b;
            continue;
        }
        if (mlo_skip > 0 && m >= mlo_skip) continue;           // the fused setup extracts it
        const int q = 16 / (int)sizeof(R);
        const int np = (m * m + q - 1) / q * q;
        extract_block_warp<R>(col_idx, values, col_offset, bs, m, rpv, e0, e1, T);
        write_tile(out + __ldg(val_off + b), T, np);
        __syncwarp();
    }
}

template <typename R>
__global__ void __launch_bounds__(kHeavyThreads)
k_extract_heavy(const int64_t *__restrict__ row_ptr, const int32_t *__restrict__ col_idx,
                const R *__restrict__ values, int64_t col_offset, const int32_t *__restrict__ block_ptr,
                const int64_t *__restrict__ val_off, R *__restrict__ out, const int32_t *__restrict__ heavy,
                const unsigned long long *__restrict__ nheavy) {
    __shared__ __align__(16) R T[kMaxM * kMaxM];
    __shared__ int64_t rp[kMaxM + 1];
    const int64_t nh = (int64_t)*nheavy;
    for (int64_t h = blockIdx.x; h < nh; h += gridDim.x) {
        const int b = heavy[h];
        const int bs = block_ptr[b], be = block_ptr[b + 1], m = be - bs;
        const int q = 16 / (int)sizeof(R);
        const int np = (m * m + q - 1) / q * q;
        for (int i = threadIdx.x; i < np; i += blockDim.x) T[i] = R(0);
        if (threadIdx.x <= m) rp[threadIdx.x] = row_ptr[bs + threadIdx.x];
        __syncthreads();
        const int64_t e0 = rp[0], e1 = rp[m];
        const int64_t cb = (int64_t)bs + col_offset, ce = (int64_t)be + col_offset;
        for (int64_t e = e0 + threadIdx.x; e < e1; e += blockDim.x) {
            const int64_t c = __ldg(col_idx + e);
            if (c >= cb && c < ce) {
                int lo = 0, hi = m;                                 // row: rp[lo] <= e < rp[lo+1]
                while (hi - lo > 1) {
                    const int mid = (lo + hi) >> 1;
                    if (rp[mid] <= e) lo = mid; else hi = mid;
                }
                T[lo + (int)(c - cb) * m] = __ldg(values + e);
            }
        }
        __syncthreads();
        const int n16 = np * (int)sizeof(R) / 16;
        const int4 *s4 = reinterpret_cast<const int4 *>(T);
        int4 *d4 = reinterpret_cast<int4 *>(out + val_off[b]);
        for (int i = threadIdx.x; i < n16; i += blockDim.x) d4[i] = s4[i];
        __syncthreads();
    }
}

template <typename R>
bj_status extract_run(const bj_csr &A, const int32_t *block_ptr, int64_t nb, const int64_t *val_off, R *out,
                      cudaStream_t s, int mlo_skip) {
    if (nb == 0) return BJ_OK;
    const int grid = persistent_grid(k_extract_warp<R>, kExtractThreads);
    const int hgrid = 2 * sm_count();
    int32_t *heavy = nullptr;
    unsigned long long *nheavy = nullptr;
    const size_t hbytes = sizeof(int32_t) * (size_t)nb;
    AsyncScratch scratch(s);
    BJ_CUDA_TRY(cudaMallocAsync((void **)&scratch.p, 16 + hbytes, s));
    nheavy = reinterpret_cast<unsigned long long *>(scratch.p);
    heavy = reinterpret_cast<int32_t *>(scratch.p + 16);
    BJ_CUDA_TRY(cudaMemsetAsync(nheavy, 0, sizeof(unsigned long long), s));
    const R *vals = static_cast<const R *>(A.values);
    k_extract_warp<R><<<grid, kExtractThreads, 0, s>>>(A.row_ptr, A.col_idx, vals, A.col_offset, block_ptr, nb,
                                                       val_off, out, heavy, nheavy, mlo_skip);
    BJ_LAUNCH_CHECK();
    k_extract_heavy<R><<<hgrid, kHeavyThreads, 0, s>>>(A.row_ptr, A.col_idx, vals, A.col_offset, block_ptr,
                                                       val_off, out, heavy, nheavy);
    BJ_LAUNCH_CHECK();
    return BJ_OK;
}

template bj_status extract_run<double>(const bj_csr &, const int32_t *, int64_t, const int64_t *, double *,
                                       cudaStream_t, int);
template bj_status extract_run<float>(const bj_csr &, const int32_t *, int64_t, const int64_t *, float *,
                                      cudaStream_t, int);

}  // namespace bj
