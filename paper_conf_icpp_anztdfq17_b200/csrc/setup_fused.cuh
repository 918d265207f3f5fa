#pragma once
// setup_fused.cuh -- NEXT(1) of SURVEY 8(f): the block-Jacobi setup with the
// diagonal-block extraction (row a2) fused into the factorization (row a3).
// As in the paper's own pipeline (the extracted elements "are
// copied into registers of the thread that will handle the respective row in
// the factorization process"), a warp extracts its block from the CSR into a
// shared-memory tile (extract_tile.cuh) and factors it from there with the
// GETRF tile of getrf_fast.cuh -- the dense block is never written to and
// re-read from HBM (-2 s m^2 bytes per block).  Outputs are bit-identical to
// bj_extract followed by bj_getrf_vbatched: the same extraction, the same
// factorization code.  One kernel per order 17..32 (the full-warp tiles);
// blocks of other orders, and blocks with more than kHeavy stored entries,
// take the separate extract + factor path (api.cu).
#include "extract_tile.cuh"
#include "getrf_fast.cuh"

namespace bj {

template <typename R, int M>
__global__ void __launch_bounds__(kFastThreads, fast_min_blocks<R>(fast_flags<R, M>(), M))
k_setup_fused(const int64_t *__restrict__ row_ptr, const int32_t *__restrict__ col_idx,
              const R *__restrict__ values, int64_t col_offset, const int32_t *__restrict__ block_ptr, R *A,
              const int64_t *__restrict__ val_off, const int64_t *__restrict__ vec_off, int32_t *__restrict__ piv,
              int32_t *__restrict__ info, const int32_t *__restrict__ order, const int64_t *__restrict__ bin_start,
              int32_t *__restrict__ safe_list, unsigned *__restrict__ safe_count) {
    static_assert(M >= 17 && M <= 32, "full-warp orders");
    __shared__ __align__(16) FastSmem<R> s_warp[kFastThreads / 32];
    __shared__ __align__(16) R s_tile[kFastThreads / 32][stage_elems<R>(M, M)];
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    FastSmem<R> &sm = s_warp[w];
    R *S = s_tile[w];
    const int64_t first = bin_start[M], ntask = bin_start[M + 1] - first;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    const int64_t warp = __reduce_max_sync(kFull, (unsigned)(((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5));
    // index chain one task ahead: order -> block_ptr -> row_ptr
    auto fetch = [&](int64_t t, int &blk, int &bs, int64_t &rpv, int64_t &e1) {
        blk = t < ntask ? __ldg(order + first + t) : -1;
        bs = blk >= 0 ? __ldg(block_ptr + blk) : 0;
        rpv = (blk >= 0 && lane < M) ? __ldg(row_ptr + bs + lane) : 0;
        e1 = blk >= 0 ? __ldg(row_ptr + bs + M) : 0;
    };
    int n_blk, n_bs;
    int64_t n_rpv, n_e1;
    fetch(warp, n_blk, n_bs, n_rpv, n_e1);
    for (int64_t t = warp; t < ntask; t += nwarps) {
        const int blk = n_blk, bs = n_bs;
        const int64_t rpv = n_rpv, e1 = n_e1;
        fetch(t + nwarps, n_blk, n_bs, n_rpv, n_e1);
        const int64_t e0 = __shfl_sync(kFull, rpv, 0);
        FTask tk;
        tk.m = M;
        tk.ok = true;
        tk.blk = blk;
        tk.lo = __ldg(val_off + blk);
        tk.vo = __ldg(vec_off + blk);
        if (e1 - e0 > kHeavy) {              // extracted by k_extract_heavy; factored by the safe kernel
            if (lane == 0) safe_list[atomicAdd(safe_count, 1u)] = blk;
            continue;
        }
        extract_block_warp<R>(col_idx, values, col_offset, bs, M, rpv, e0, e1, S);
        auto nothing = [] {};
        getrf_fast_tile<R, M, fast_flags<R, M>(), false, decltype(nothing) &, true>(
            A, tk, S, piv, info, safe_list, safe_count, nullptr, nullptr, sm, nothing);
        __syncwarp();                        // the tile is read before the next extraction rewrites it
    }
    asm volatile("griddepcontrol.wait;" ::: "memory");
}

template <typename R, int M>
bj_status launch_setup_fused(const bj_csr &Acsr, const int32_t *block_ptr, R *A, const int64_t *val_off,
                             const int64_t *vec_off, int32_t *piv, int32_t *info, const PlanView &p,
                             int32_t *safe_list, unsigned *safe_count, cudaStream_t s) {
    auto kern = k_setup_fused<R, M>;
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(persistent_grid(kern, kFastThreads, true));
    cfg.blockDim = dim3(kFastThreads);
    cfg.stream = s;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    BJ_CUDA_TRY(cudaLaunchKernelEx(&cfg, kern, (const int64_t *)Acsr.row_ptr, (const int32_t *)Acsr.col_idx,
                                   (const R *)Acsr.values, (int64_t)Acsr.col_offset, block_ptr, A, val_off, vec_off,
                                   piv, info, (const int32_t *)p.order, (const int64_t *)p.bin_start, safe_list,
                                   safe_count));
    ::bj::count_launch();
    return BJ_OK;
}

}  // namespace bj
