// api.cu -- the C ABI (include/bj.h): argument checking, plans, handles,
// workspaces and dispatch to the kernel translation units.  No arithmetic of
// the method lives here; there is no CPU or library fallback.
#include <algorithm>
#include <mutex>
#include <new>
#include <unordered_map>
#include <vector>
#include <stdlib.h>
#include <string.h>

#include "common.cuh"
#include "internal.h"

namespace bj {

static thread_local int64_t g_launches = 0;
void count_launch(int n) { g_launches += n; }

int sm_count() {
    int dev = 0;
    cudaGetDevice(&dev);
    static int cached[64] = {0};
    if (dev < 0 || dev >= 64) dev = 0;
    if (cached[dev] == 0) {
        int n = 0;
        cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
        cached[dev] = n > 0 ? n : 1;
    }
    return cached[dev];
}

// persistent_grid's cache (common.cuh): (kernel address, device, block size) -> grid
namespace {
struct GridKey {
    const void *k;
    int dev, threads;
    bool operator==(const GridKey &o) const { return k == o.k && dev == o.dev && threads == o.threads; }
};
struct GridKeyHash {
    size_t operator()(const GridKey &g) const {
        return std::hash<const void *>()(g.k) ^ ((size_t)g.dev * 0x9E3779B97F4A7C15ull) ^ ((size_t)g.threads << 40);
    }
};
std::mutex g_grid_mutex;
std::unordered_map<GridKey, int, GridKeyHash> g_grid_cache;
}  // namespace
int grid_cache_get(const void *kernel, int dev, int threads) {
    std::lock_guard<std::mutex> lock(g_grid_mutex);
    auto it = g_grid_cache.find(GridKey{kernel, dev, threads});
    return it == g_grid_cache.end() ? 0 : it->second;
}
void grid_cache_put(const void *kernel, int dev, int threads, int grid) {
    std::lock_guard<std::mutex> lock(g_grid_mutex);
    g_grid_cache[GridKey{kernel, dev, threads}] = grid;
}

static int elem_size(bj_dtype d) { return d == BJ_F64 ? 8 : d == BJ_F32 ? 4 : 0; }
static bool aligned16(const void *p) { return ((uintptr_t)p & 15u) == 0; }

static bj_status check_batch(const bj_batch *b, bool need_values) {
    if (!b || b->nblocks < 0 || elem_size(b->dtype) == 0) return BJ_ERR_ARG;
    if (b->nblocks > 0 && (!b->sizes || !b->vec_off || !b->val_off)) return BJ_ERR_ARG;
    if (need_values && b->nblocks > 0 && !b->values) return BJ_ERR_ARG;
    if (b->values && !aligned16(b->values)) return BJ_ERR_ALIGN;
    if (b->nblocks >= (int64_t)1 << 31) return BJ_ERR_ARG;   // block ids are int32
    return BJ_OK;
}

}  // namespace bj

using namespace bj;

struct bj_plan {
    int64_t nblocks = 0;
    int32_t *order = nullptr;
    int64_t *bin_start = nullptr;
    cudaStream_t stream = nullptr;     // creation stream: the plan's memory is freed on it
    PlanView view() const { return PlanView{nblocks, order, bin_start}; }
};

struct bj_handle {
    bool ready = false;
    bool inverse = false;              // NEXT(3): factors hold explicit inverses (apply = GEMV)
    bj_batch factors{};
    int32_t *pivots = nullptr;
    bj_plan plan;
    int64_t nrows = 0;
};

struct bj_workspace {
    char *dev = nullptr;
    size_t cap = 0;
};

// The library's scratch and plan memory comes from the device's default
// stream-ordered pool; keep freed memory in the pool (no release at stream
// syncs) so per-call allocations never reach the driver on the hot path.
static void pool_keep_memory() {
    static bool done[64] = {false};            // per device
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64 || done[dev]) return;
    done[dev] = true;
    cudaMemPool_t pool;
    if (cudaDeviceGetDefaultMemPool(&pool, dev) == cudaSuccess) {
        uint64_t keep = UINT64_MAX;
        cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &keep);
    }
}

static bj_status plan_alloc_build(bj_plan *p, int64_t nb, const int32_t *sizes, cudaStream_t s) {
    pool_keep_memory();
    p->nblocks = nb;
    p->stream = s;
    BJ_CUDA_TRY(cudaMallocAsync((void **)&p->order, sizeof(int32_t) * (size_t)(nb > 0 ? nb : 1), s));
    BJ_CUDA_TRY(cudaMallocAsync((void **)&p->bin_start, sizeof(int64_t) * (kBins + 1), s));
    return build_plan(nb, sizes, p->order, p->bin_start, s);
}

static void plan_free_async(bj_plan *p, cudaStream_t s) {
    if (p->order) cudaFreeAsync(p->order, s);
    if (p->bin_start) cudaFreeAsync(p->bin_start, s);
    p->order = nullptr;
    p->bin_start = nullptr;
}

extern "C" {

const char *bj_status_string(bj_status st) {
    switch (st) {
    case BJ_OK: return "BJ_OK";
    case BJ_ERR_ARG: return "BJ_ERR_ARG: invalid argument";
    case BJ_ERR_BLOCK_SIZE: return "BJ_ERR_BLOCK_SIZE: block order outside 0..32";
    case BJ_ERR_ALIGN: return "BJ_ERR_ALIGN: pointer not 16-byte aligned";
    case BJ_ERR_CUDA: return "BJ_ERR_CUDA: CUDA runtime error";
    case BJ_ERR_NOMEM: return "BJ_ERR_NOMEM: allocation failed";
    case BJ_ERR_STATE: return "BJ_ERR_STATE: object not ready";
    case BJ_ERR_COMM: return "BJ_ERR_COMM: communication callback failed";
    }
    return "unknown bj_status";
}

const char *bj_version(void) { return "bj-b200 0.1 (sm_100a)"; }

int64_t bj_launch_count(void) { return g_launches; }
void bj_launch_count_reset(void) { g_launches = 0; }

bj_status bj_layout(int64_t nblocks, const int32_t *sizes, bj_dtype dtype, int64_t *vec_off, int64_t *val_off,
                    bj_stream_t stream) {
    pool_keep_memory();
    const int es = elem_size(dtype);
    if (nblocks < 0 || es == 0 || !vec_off || !val_off || (nblocks > 0 && !sizes)) return BJ_ERR_ARG;
    return layout_sizes(nblocks, sizes, es, vec_off, val_off, (cudaStream_t)stream);
}

bj_status bj_layout_from_block_ptr(int64_t nblocks, const int32_t *block_ptr, bj_dtype dtype, int32_t *sizes,
                                   int64_t *vec_off, int64_t *val_off, bj_stream_t stream) {
    pool_keep_memory();
    const int es = elem_size(dtype);
    if (nblocks < 0 || es == 0 || !block_ptr || !vec_off || !val_off || (nblocks > 0 && !sizes)) return BJ_ERR_ARG;
    return layout_block_ptr(nblocks, block_ptr, es, sizes, vec_off, val_off, (cudaStream_t)stream);
}

bj_status bj_plan_create(bj_plan **plan, int64_t nblocks, const int32_t *sizes, bj_stream_t stream) {
    if (!plan || nblocks < 0 || (nblocks > 0 && !sizes) || nblocks >= (int64_t)1 << 31) return BJ_ERR_ARG;
    bj_plan *p = new (std::nothrow) bj_plan();
    if (!p) return BJ_ERR_NOMEM;
    bj_status st = plan_alloc_build(p, nblocks, sizes, (cudaStream_t)stream);
    if (st != BJ_OK) {
        plan_free_async(p, (cudaStream_t)stream);
        delete p;
        return st;
    }
    *plan = p;
    return BJ_OK;
}

bj_status bj_plan_destroy(bj_plan *plan) {
    if (!plan) return BJ_ERR_ARG;
    // stream-ordered: after every call already enqueued on the creation stream
    plan_free_async(plan, plan->stream);
    delete plan;
    return BJ_OK;
}

bj_status bj_extract(const bj_csr *A, const int32_t *block_ptr, bj_batch *out, bj_stream_t stream) {
    pool_keep_memory();
    if (!A || !block_ptr) return BJ_ERR_ARG;
    bj_status st = check_batch(out, true);
    if (st != BJ_OK) return st;
    if (A->dtype != out->dtype || A->nrows < 0 || A->nnz < 0 || !A->row_ptr) return BJ_ERR_ARG;
    if (A->nnz > 0 && (!A->col_idx || !A->values)) return BJ_ERR_ARG;
    cudaStream_t s = (cudaStream_t)stream;
    if (out->dtype == BJ_F64)
        return extract_run<double>(*A, block_ptr, out->nblocks, out->val_off, (double *)out->values, s);
    return extract_run<float>(*A, block_ptr, out->nblocks, out->val_off, (float *)out->values, s);
}

bj_status bj_supervariable_blocking(const bj_csr *A, int32_t max_block, int32_t *block_ptr, int64_t *nblocks_h,
                                    bj_stream_t stream) {
    if (!A || !block_ptr || !nblocks_h || max_block < 1 || max_block > kMaxM) return BJ_ERR_ARG;
    if (A->nrows < 0 || A->nrows > 2147483646LL || A->nnz < 0 || !A->row_ptr) return BJ_ERR_ARG;
    if (A->nnz > 0 && !A->col_idx) return BJ_ERR_ARG;
    pool_keep_memory();
    return supervariable_run(*A, max_block, block_ptr, nblocks_h, (cudaStream_t)stream);
}

bj_status bj_getrf_vbatched(bj_batch *blocks, int32_t *pivots, int32_t *info, const bj_plan *plan,
                            bj_stream_t stream) {
    pool_keep_memory();
    bj_status st = check_batch(blocks, true);
    if (st != BJ_OK) return st;
    if (blocks->nblocks > 0 && (!pivots || !info)) return BJ_ERR_ARG;
    if (plan && plan->nblocks != blocks->nblocks) return BJ_ERR_ARG;
    if (blocks->nblocks == 0) return BJ_OK;
    cudaStream_t s = (cudaStream_t)stream;
    bj_plan tmp;
    const bj_plan *p = plan;
    if (!p) {
        if ((st = plan_alloc_build(&tmp, blocks->nblocks, blocks->sizes, s)) != BJ_OK) {
            plan_free_async(&tmp, s);
            return st;
        }
        p = &tmp;
    }
    if (blocks->dtype == BJ_F64)
        st = getrf_run<double>((double *)blocks->values, blocks->val_off, blocks->vec_off, pivots, info, p->view(),
                               blocks->sizes, s);
    else
        st = getrf_run<float>((float *)blocks->values, blocks->val_off, blocks->vec_off, pivots, info, p->view(),
                              blocks->sizes, s);
    if (!plan) plan_free_async(&tmp, s);
    return st;
}

bj_status bj_getrs_vbatched(const bj_batch *lu, const int32_t *pivots, const void *b, void *x, const bj_plan *plan,
                            bj_stream_t stream) {
    pool_keep_memory();
    bj_status st = check_batch(lu, true);
    if (st != BJ_OK) return st;
    if (lu->nblocks > 0 && (!pivots || !b || !x)) return BJ_ERR_ARG;
    if (plan && plan->nblocks != lu->nblocks) return BJ_ERR_ARG;
    if (lu->nblocks == 0) return BJ_OK;
    cudaStream_t s = (cudaStream_t)stream;
    bj_plan tmp;
    const bj_plan *p = plan;
    if (!p) {
        if ((st = plan_alloc_build(&tmp, lu->nblocks, lu->sizes, s)) != BJ_OK) {
            plan_free_async(&tmp, s);
            return st;
        }
        p = &tmp;
    }
    if (lu->dtype == BJ_F64)
        st = getrs_run<double>((const double *)lu->values, lu->val_off, lu->vec_off, pivots, (const double *)b,
                               (double *)x, p->view(), s);
    else
        st = getrs_run<float>((const float *)lu->values, lu->val_off, lu->vec_off, pivots, (const float *)b,
                              (float *)x, p->view(), s);
    if (!plan) plan_free_async(&tmp, s);
    return st;
}

bj_status bj_gesv_vbatched(bj_batch *blocks, int32_t *pivots, int32_t *info, const void *b, void *x,
                           const bj_plan *plan, bj_stream_t stream) {
    pool_keep_memory();
    bj_status st = check_batch(blocks, true);
    if (st != BJ_OK) return st;
    if (blocks->nblocks > 0 && (!pivots || !info || !b || !x)) return BJ_ERR_ARG;
    if (plan && plan->nblocks != blocks->nblocks) return BJ_ERR_ARG;
    if (blocks->nblocks == 0) return BJ_OK;
    cudaStream_t s = (cudaStream_t)stream;
    bj_plan tmp;
    const bj_plan *p = plan;
    if (!p) {
        if ((st = plan_alloc_build(&tmp, blocks->nblocks, blocks->sizes, s)) != BJ_OK) {
            plan_free_async(&tmp, s);
            return st;
        }
        p = &tmp;
    }
    if (blocks->dtype == BJ_F64)
        st = gesv_run<double>((double *)blocks->values, blocks->val_off, blocks->vec_off, pivots, info, p->view(),
                              blocks->sizes, (const double *)b, (double *)x, s);
    else
        st = gesv_run<float>((float *)blocks->values, blocks->val_off, blocks->vec_off, pivots, info, p->view(),
                             blocks->sizes, (const float *)b, (float *)x, s);
    if (!plan) plan_free_async(&tmp, s);
    return st;
}

bj_status bj_getri_vbatched(bj_batch *blocks, int32_t *pivots, int32_t *info, const bj_plan *plan,
                            bj_stream_t stream) {
    pool_keep_memory();
    bj_status st = check_batch(blocks, true);
    if (st != BJ_OK) return st;
    if (blocks->nblocks > 0 && (!pivots || !info)) return BJ_ERR_ARG;
    if (plan && plan->nblocks != blocks->nblocks) return BJ_ERR_ARG;
    if (blocks->nblocks == 0) return BJ_OK;
    cudaStream_t s = (cudaStream_t)stream;
    bj_plan tmp;
    const bj_plan *p = plan;
    if (!p) {
        if ((st = plan_alloc_build(&tmp, blocks->nblocks, blocks->sizes, s)) != BJ_OK) {
            plan_free_async(&tmp, s);
            return st;
        }
        p = &tmp;
    }
    if (blocks->dtype == BJ_F64)
        st = getri_run<double>((double *)blocks->values, blocks->val_off, blocks->vec_off, pivots, info, p->view(),
                               blocks->sizes, s);
    else
        st = getri_run<float>((float *)blocks->values, blocks->val_off, blocks->vec_off, pivots, info, p->view(),
                              blocks->sizes, s);
    if (!plan) plan_free_async(&tmp, s);
    return st;
}

bj_status bj_gemv_vbatched(const bj_batch *inv, const void *x, void *y, const bj_plan *plan, bj_stream_t stream) {
    pool_keep_memory();
    bj_status st = check_batch(inv, true);
    if (st != BJ_OK) return st;
    if (inv->nblocks > 0 && (!x || !y)) return BJ_ERR_ARG;
    if (plan && plan->nblocks != inv->nblocks) return BJ_ERR_ARG;
    if (inv->nblocks == 0) return BJ_OK;
    cudaStream_t s = (cudaStream_t)stream;
    bj_plan tmp;
    const bj_plan *p = plan;
    if (!p) {
        if ((st = plan_alloc_build(&tmp, inv->nblocks, inv->sizes, s)) != BJ_OK) {
            plan_free_async(&tmp, s);
            return st;
        }
        p = &tmp;
    }
    if (inv->dtype == BJ_F64)
        st = gemv_run<double>((const double *)inv->values, inv->val_off, inv->vec_off, (const double *)x,
                              (double *)y, p->view(), s);
    else
        st = gemv_run<float>((const float *)inv->values, inv->val_off, inv->vec_off, (const float *)x, (float *)y,
                             p->view(), s);
    if (!plan) plan_free_async(&tmp, s);
    return st;
}

bj_status bj_create(bj_handle **handle) {
    if (!handle) return BJ_ERR_ARG;
    bj_handle *h = new (std::nothrow) bj_handle();
    if (!h) return BJ_ERR_NOMEM;
    *handle = h;
    return BJ_OK;
}

static bj_status setup_common(bj_handle *h, const bj_csr *A, const int32_t *block_ptr, bj_batch *factors,
                              int32_t *pivots, int32_t *info, bj_stream_t stream, bool inverse) {
    pool_keep_memory();
    if (!h || !A || !block_ptr || !factors) return BJ_ERR_ARG;
    bj_status st = check_batch(factors, true);
    if (st != BJ_OK) return st;
    if (A->dtype != factors->dtype) return BJ_ERR_ARG;
    if (factors->nblocks > 0 && (!pivots || !info)) return BJ_ERR_ARG;
    cudaStream_t s = (cudaStream_t)stream;
    const int64_t nb = factors->nblocks;
    const int es = elem_size(factors->dtype);
    h->ready = false;
    if ((st = layout_block_ptr(nb, block_ptr, es, factors->sizes, factors->vec_off, factors->val_off, s)) != BJ_OK)
        return st;
    if (A->nrows < 0 || A->nnz < 0 || !A->row_ptr || (A->nnz > 0 && (!A->col_idx || !A->values))) return BJ_ERR_ARG;
    plan_free_async(&h->plan, s);
    if ((st = plan_alloc_build(&h->plan, nb, factors->sizes, s)) != BJ_OK) return st;
    if (inverse) {
        if ((st = bj_extract(A, block_ptr, factors, stream)) != BJ_OK) return st;
        st = bj_getri_vbatched(factors, pivots, info, &h->plan, stream);
    } else if (factors->dtype == BJ_F64) {          // NEXT(1): extraction fused into GETRF
        st = setup_run<double>(*A, block_ptr, (double *)factors->values, factors->val_off, factors->vec_off,
                               pivots, info, h->plan.view(), factors->sizes, s);
    } else {
        st = setup_run<float>(*A, block_ptr, (float *)factors->values, factors->val_off, factors->vec_off,
                              pivots, info, h->plan.view(), factors->sizes, s);
    }
    if (st != BJ_OK) return st;
    h->factors = *factors;
    h->pivots = pivots;
    h->nrows = A->nrows;
    h->inverse = inverse;
    h->ready = true;
    return BJ_OK;
}

bj_status bj_setup(bj_handle *h, const bj_csr *A, const int32_t *block_ptr, bj_batch *factors, int32_t *pivots,
                   int32_t *info, bj_stream_t stream) {
    return setup_common(h, A, block_ptr, factors, pivots, info, stream, false);
}

bj_status bj_setup_inverse(bj_handle *h, const bj_csr *A, const int32_t *block_ptr, bj_batch *inverses,
                           int32_t *pivots, int32_t *info, bj_stream_t stream) {
    return setup_common(h, A, block_ptr, inverses, pivots, info, stream, true);
}

bj_status bj_apply(bj_handle *h, const void *x, void *y, bj_stream_t stream) {
    pool_keep_memory();
    if (!h || !x || !y) return BJ_ERR_ARG;
    if (!h->ready) return BJ_ERR_STATE;
    if (h->inverse) return bj_gemv_vbatched(&h->factors, x, y, &h->plan, stream);
    return bj_getrs_vbatched(&h->factors, h->pivots, x, y, &h->plan, stream);
}

bj_status bj_destroy(bj_handle *h) {
    if (!h) return BJ_ERR_ARG;
    if (h->plan.order) cudaFree(h->plan.order);
    if (h->plan.bin_start) cudaFree(h->plan.bin_start);
    delete h;
    return BJ_OK;
}

bj_status bj_partition(int64_t nblocks, const int32_t *sizes_h, int G, int64_t *bounds_h) {
    if (nblocks < 0 || G < 1 || !bounds_h || (nblocks > 0 && !sizes_h)) return BJ_ERR_ARG;
    int64_t total = 0;
    for (int64_t i = 0; i < nblocks; ++i) total += (int64_t)sizes_h[i] * sizes_h[i];
    bounds_h[0] = 0;
    bounds_h[G] = nblocks;
    // single sweep: boundary r is the first i with G*P(i) >= r*total
    int64_t P = 0, i = 0;
    for (int r = 1; r < G; ++r) {
        const __int128 target = (__int128)r * total;
        while (i < nblocks && (__int128)G * P < target) {
            P += (int64_t)sizes_h[i] * sizes_h[i];
            ++i;
        }
        bounds_h[r] = i;
    }
    return BJ_OK;
}

bj_status bj_workspace_create(bj_workspace **ws) {
    if (!ws) return BJ_ERR_ARG;
    bj_workspace *w = new (std::nothrow) bj_workspace();
    if (!w) return BJ_ERR_NOMEM;
    *ws = w;
    return BJ_OK;
}

bj_status bj_workspace_destroy(bj_workspace *ws) {
    if (!ws) return BJ_ERR_ARG;
    if (ws->dev) cudaFree(ws->dev);
    delete ws;
    return BJ_OK;
}

static size_t up256(size_t x) { return (x + 255) & ~(size_t)255; }

bj_status bj_gesv_host(bj_workspace *ws, int64_t nb, const int32_t *sizes_h, int64_t nvalues, const void *blocks_h,
                       int64_t nvec, const void *b_h, void *x_h, int32_t *pivots_h, int32_t *info_h, bj_dtype dtype,
                       bj_stream_t stream) {
    pool_keep_memory();
    const int es = elem_size(dtype);
    if (!ws || nb < 0 || nvalues < 0 || nvec < 0 || es == 0) return BJ_ERR_ARG;
    if (nb > 0 && (!sizes_h || !blocks_h || !b_h || !x_h)) return BJ_ERR_ARG;
    if (nb == 0) return BJ_OK;
    {   // the caller's buffers must hold the layout of sizes_h (host arithmetic, no copy yet)
        const int64_t q = 16 / es;
        int64_t need_val = 0, need_vec = 0;
        for (int64_t i = 0; i < nb; ++i) {
            const int64_t m = sizes_h[i] > 0 ? sizes_h[i] : 0;
            need_val += (m * m + q - 1) / q * q;
            need_vec += m;
        }
        if (nvalues < need_val || nvec < need_vec) return BJ_ERR_ARG;
    }
    cudaStream_t s = (cudaStream_t)stream;
    // Chunked pipeline: the batch is cut into K contiguous chunks; the copy
    // engines move chunk c+1 in (stream sh) and chunk c-1 out (stream sd) while
    // chunk c is factored and solved on the caller's stream, so PCIe time
    // hides the compute.  Each chunk is an independent sub-batch (own layout
    // and plan); the results are those of the whole batch (blocks are
    // independent).
    int K = (int)std::min<int64_t>(4, std::max<int64_t>(1, nb / 65536));
    if (const char *ev_k = getenv("BJ_GESV_HOST_CHUNKS")) {     // experiment hook (bench / tests)
        const int k = atoi(ev_k);
        if (k >= 1 && k <= 64) K = (int)std::min<int64_t>(k, nb);
    }
    std::vector<int64_t> V(nb + 1), E(nb + 1), cb(K + 1);
    {
        const int64_t q = 16 / es;
        V[0] = E[0] = 0;
        for (int64_t i = 0; i < nb; ++i) {
            const int64_t m = sizes_h[i] > 0 ? sizes_h[i] : 0;
            V[i + 1] = V[i] + (m * m + q - 1) / q * q;
            E[i + 1] = E[i] + m;
        }
        for (int c = 0; c <= K; ++c) cb[c] = nb * c / K;
    }
    const size_t o_sizes = 0;
    const size_t o_vec = o_sizes + up256(sizeof(int32_t) * nb);
    const size_t o_val = o_vec + up256(sizeof(int64_t) * (nb + K));
    const size_t o_A = o_val + up256(sizeof(int64_t) * (nb + K));
    const size_t o_b = o_A + up256((size_t)es * nvalues);
    const size_t o_x = o_b + up256((size_t)es * nvec);
    const size_t o_piv = o_x + up256((size_t)es * nvec);
    const size_t o_info = o_piv + up256(sizeof(int32_t) * nvec);
    const size_t o_order = o_info + up256(sizeof(int32_t) * nb);
    const size_t o_bins = o_order + up256(sizeof(int32_t) * nb);
    const size_t need = o_bins + up256(sizeof(int64_t) * (kBins + 1) * K);
    if (need > ws->cap) {
        if (ws->dev) BJ_CUDA_TRY(cudaFree(ws->dev));
        ws->dev = nullptr;
        ws->cap = 0;
        if (cudaMalloc((void **)&ws->dev, need) != cudaSuccess) return BJ_ERR_NOMEM;
        ws->cap = need;
    }
    char *d = ws->dev;
    int32_t *sizes = (int32_t *)(d + o_sizes);
    int64_t *vec = (int64_t *)(d + o_vec), *val = (int64_t *)(d + o_val);
    int32_t *piv = (int32_t *)(d + o_piv), *info = (int32_t *)(d + o_info);
    char *A = d + o_A, *bd = d + o_b, *xd = d + o_x;
    int32_t *order = (int32_t *)(d + o_order);
    int64_t *bins = (int64_t *)(d + o_bins);
    cudaStream_t sh = nullptr, sd = nullptr;
    std::vector<cudaEvent_t> ev(2 * (size_t)K + 1, nullptr);
    auto cleanup = [&]() {
        if (sd) cudaStreamSynchronize(sd);
        if (sh) cudaStreamSynchronize(sh);
        cudaStreamSynchronize(s);
        for (auto e : ev)
            if (e) cudaEventDestroy(e);
        if (sh) cudaStreamDestroy(sh);
        if (sd) cudaStreamDestroy(sd);
    };
    bj_status st = BJ_OK;
    do {
        if (cudaStreamCreateWithFlags(&sh, cudaStreamNonBlocking) != cudaSuccess ||
            cudaStreamCreateWithFlags(&sd, cudaStreamNonBlocking) != cudaSuccess) { st = BJ_ERR_CUDA; break; }
        for (auto &e : ev)
            if (cudaEventCreateWithFlags(&e, cudaEventDisableTiming) != cudaSuccess) { st = BJ_ERR_CUDA; break; }
        if (st != BJ_OK) break;
        // the workspace may still be in use by work the caller queued earlier on s
        if (cudaEventRecord(ev[2 * K], s) != cudaSuccess || cudaStreamWaitEvent(sh, ev[2 * K], 0) != cudaSuccess) {
            st = BJ_ERR_CUDA;
            break;
        }
        const char *Ah = (const char *)blocks_h, *bh = (const char *)b_h;
        for (int c = 0; c < K && st == BJ_OK; ++c) {          // inputs, chunk by chunk
            const int64_t b0 = cb[c], b1 = cb[c + 1];
            if (cudaMemcpyAsync(sizes + b0, sizes_h + b0, sizeof(int32_t) * (b1 - b0), cudaMemcpyHostToDevice, sh) ||
                cudaMemcpyAsync(A + es * V[b0], Ah + es * V[b0], (size_t)es * (V[b1] - V[b0]), cudaMemcpyHostToDevice, sh) ||
                cudaMemcpyAsync(bd + es * E[b0], bh + es * E[b0], (size_t)es * (E[b1] - E[b0]), cudaMemcpyHostToDevice, sh) ||
                cudaEventRecord(ev[c], sh))
                st = BJ_ERR_CUDA;
        }
        for (int c = 0; c < K && st == BJ_OK; ++c) {          // compute, chunk by chunk
            const int64_t b0 = cb[c], b1 = cb[c + 1], n = b1 - b0;
            if (n == 0) { if (cudaEventRecord(ev[K + c], s)) st = BJ_ERR_CUDA; continue; }
            if (cudaStreamWaitEvent(s, ev[c], 0)) { st = BJ_ERR_CUDA; break; }
            int64_t *vc = vec + b0 + c, *lc = val + b0 + c;
            if ((st = layout_sizes(n, sizes + b0, es, vc, lc, s)) != BJ_OK) break;
            bj_plan p;
            p.nblocks = n;
            p.order = order + b0;
            p.bin_start = bins + (size_t)c * (kBins + 1);
            if ((st = build_plan(n, sizes + b0, p.order, p.bin_start, s)) != BJ_OK) break;
            bj_batch batch{n, sizes + b0, vc, lc, A + es * V[b0], dtype};
            // separate calls: measured faster than the fused bj_gesv_vbatched on
            // B200 (the solve is latency-bound)
            if ((st = bj_getrf_vbatched(&batch, piv + E[b0], info + b0, &p, stream)) != BJ_OK) break;
            if ((st = bj_getrs_vbatched(&batch, piv + E[b0], bd + es * E[b0], xd + es * E[b0], &p, stream)) != BJ_OK)
                break;
            if (cudaEventRecord(ev[K + c], s)) st = BJ_ERR_CUDA;
        }
        for (int c = 0; c < K && st == BJ_OK; ++c) {          // outputs, chunk by chunk
            const int64_t b0 = cb[c], b1 = cb[c + 1];
            if (cudaStreamWaitEvent(sd, ev[K + c], 0) ||
                cudaMemcpyAsync((char *)x_h + es * E[b0], xd + es * E[b0], (size_t)es * (E[b1] - E[b0]),
                                cudaMemcpyDeviceToHost, sd) ||
                (pivots_h && cudaMemcpyAsync(pivots_h + E[b0], piv + E[b0], sizeof(int32_t) * (E[b1] - E[b0]),
                                             cudaMemcpyDeviceToHost, sd)) ||
                (info_h && cudaMemcpyAsync(info_h + b0, info + b0, sizeof(int32_t) * (b1 - b0),
                                           cudaMemcpyDeviceToHost, sd)))
                st = BJ_ERR_CUDA;
        }
    } while (0);
    cleanup();
    if (st != BJ_OK) return st;
    if (cudaGetLastError() != cudaSuccess) return BJ_ERR_CUDA;
    return BJ_OK;
}

}  // extern "C"
