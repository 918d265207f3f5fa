// synth.cu -- device-side seeded input generators (bench / test inputs only;
// not part of the method).  Bit-identical to the host module bj_synth/ (the
// same splitmix64 counter streams); checked in tests/test_gpu_parity.py
// (test_device_generator_matches_host_generator) and tests/test_gpu_extract.py.
#include "bj_synth.h"
#include "scan.cuh"

namespace bj {
namespace synth {

constexpr unsigned long long GOLDEN = 0x9E3779B97F4A7C15ull;
constexpr unsigned long long SALT = 0x632BE59BD9B4E019ull;
constexpr unsigned long long HUB_THRESHOLD = 9007199254740ull;
constexpr long long HUB_CAP = 100000;
constexpr long long HUB_VAL_K = 1073741;
constexpr int SEED_VALUES = 2, SEED_RHS = 3, SEED_SKEW = 4, SEED_HUBCOL = 5, SEED_HUBVAL = 6, SEED_INT = 7;

__host__ __device__ inline unsigned long long mix64(unsigned long long z) {
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}
__host__ __device__ inline unsigned long long seed_key(unsigned long long seed) { return mix64(seed * GOLDEN + SALT); }
__device__ inline unsigned long long hash64(unsigned long long sk, unsigned long long idx) {
    return mix64(sk + (idx + 1ull) * GOLDEN);
}
__device__ inline double uniform_pm1(unsigned long long h) {
    const double u = (double)(h >> 11) * 0x1p-53;
    return __dadd_rn(__dmul_rn(2.0, u), -1.0);       // exact
}
__device__ inline long long uniform_int(unsigned long long h, long long lo, long long hi) {
    const unsigned long long span = (unsigned long long)(hi - lo + 1);
    return lo + (long long)(((h >> 32) * span) >> 32);
}

__global__ void k_sizes(int64_t n, int64_t first, int lo, int hi, unsigned long long sk, int32_t *sizes) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        sizes[i] = (int32_t)uniform_int(hash64(sk, (unsigned long long)(first + i)), lo, hi);
}

template <typename R>
__global__ void k_blocks(int64_t nb, int64_t first, int kind, const int32_t *__restrict__ sizes,
                         const int64_t *__restrict__ val_off, R *__restrict__ values) {
    const unsigned long long sk = seed_key(kind == 0 ? SEED_VALUES : SEED_INT);
    const int lane = threadIdx.x & 31;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t b = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; b < nb; b += nw) {
        const int m = max(sizes[b], 0);
        const int64_t o = val_off[b], o1 = val_off[b + 1];
        const int mm = m > 32 ? 0 : m * m;
        for (int64_t e = lane; e < o1 - o; e += 32) {
            R v = R(0);
            if (e < mm) {
                const int r = (int)(e % m), c = (int)(e / m);
                const unsigned long long key = (unsigned long long)(first + b) * 1024ull + (unsigned long long)(c * 32 + r);
                const unsigned long long h = hash64(sk, key);
                const double d = kind == 0 ? uniform_pm1(h) : (double)uniform_int(h, -3, 3);
                v = (R)d;
            }
            values[o + e] = v;
        }
    }
}

template <typename R>
__global__ void k_rhs(int64_t nb, int64_t first, const int32_t *__restrict__ sizes,
                      const int64_t *__restrict__ vec_off, R *__restrict__ b) {
    const unsigned long long sk = seed_key(SEED_RHS);
    const int lane = threadIdx.x & 31;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t i = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; i < nb; i += nw) {
        const int m = max(sizes[i], 0);
        for (int r = lane; r < m; r += 32)
            b[vec_off[i] + r] = (R)uniform_pm1(hash64(sk, (unsigned long long)(first + i) * 32ull + r));
    }
}

// ---------------------------------------------------------------- FEM grid
struct Grid {
    int nx, ny, nz;
    int skew;
    long long n, band, W, P;
};

__host__ inline Grid make_grid(int nx, int ny, int nz, int skew) {
    Grid g;
    g.nx = nx; g.ny = ny; g.nz = nz;
    g.n = 3LL * nx * ny * nz;
    g.band = 3LL * (1 + nx + (long long)nx * ny) + 2;
    g.W = g.n - (2 * g.band + 1);
    g.skew = skew && g.W > 0;
    g.P = 1;
    if (g.W > 0) {
        const long long primes[] = {1000003, 1000033, 1000037, 1000039, 1000081};
        for (long long p : primes)
            if (g.W % p != 0) { g.P = p; break; }
    }
    return g;
}

__device__ inline long long icbrt(unsigned long long v) {
    long long x = (long long)cbrt((double)v);
    while (x > 0 && (unsigned long long)x * x * x > v) --x;
    while ((unsigned long long)(x + 1) * (x + 1) * (x + 1) <= v) ++x;
    return x;
}

__device__ inline long long n_extra(const Grid &g, long long r) {
    if (!g.skew) return 0;
    const unsigned long long sk = seed_key(SEED_SKEW);
    if ((hash64(sk, 2ull * r) >> 11) >= HUB_THRESHOLD) return 0;
    const unsigned long long uu = 1ull + (hash64(sk, 2ull * r + 1ull) >> 44);
    const unsigned long long v = (1000000ull << 40) / (uu * uu);
    long long k = icbrt(v);
    if (k > HUB_CAP) k = HUB_CAP;
    if (k > g.W) k = g.W;
    return k;
}

__device__ inline int n_neighbors(const Grid &g, long long r) {
    const long long node = r / 3;
    const int x = (int)(node % g.nx), y = (int)((node / g.nx) % g.ny), z = (int)(node / ((long long)g.nx * g.ny));
    const int cx = 1 + (x > 0) + (x < g.nx - 1);
    const int cy = 1 + (y > 0) + (y < g.ny - 1);
    const int cz = 1 + (z > 0) + (z < g.nz - 1);
    return cx * cy * cz;
}

struct FemRowPtrF {
    Grid g;
    long long r0;
    int64_t *row_ptr;
    __device__ I64x2 value(int64_t i) const {
        const long long r = r0 + i;
        return I64x2{3LL * n_neighbors(g, r) + n_extra(g, r), 0};
    }
    __device__ void store(int64_t i, I64x2 p) const { row_ptr[i] = p.a; }
    bj_status store_empty(cudaStream_t s) const {
        BJ_CUDA_TRY(cudaMemsetAsync(row_ptr, 0, sizeof(int64_t), s));
        return BJ_OK;
    }
};

template <typename R>
__global__ void k_fem_fill(Grid g, long long r0, long long nrows, const int64_t *__restrict__ row_ptr,
                           int32_t *__restrict__ col_idx, R *__restrict__ values) {
    const unsigned long long skv = seed_key(SEED_VALUES), skc = seed_key(SEED_HUBCOL), skh = seed_key(SEED_HUBVAL);
    const int lane = threadIdx.x & 31;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t i = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; i < nrows; i += nw) {
        const long long r = r0 + i;
        const long long node = r / 3;
        const int x = (int)(node % g.nx), y = (int)((node / g.nx) % g.ny), z = (int)(node / ((long long)g.nx * g.ny));
        const int dz = lane / 9 - 1, dy = (lane / 3) % 3 - 1, dx = lane % 3 - 1;
        const bool valid = lane < 27 && x + dx >= 0 && x + dx < g.nx && y + dy >= 0 && y + dy < g.ny &&
                           z + dz >= 0 && z + dz < g.nz;
        const unsigned ball = __ballot_sync(kFull, valid);
        const int pos = 3 * __popc(ball & ((1u << lane) - 1u));
        const int64_t base = row_ptr[i];
        double off_sum = 0.0;
        int diag_slot = -1;
        if (valid) {
            const long long nd = (x + dx) + (long long)g.nx * ((y + dy) + (long long)g.ny * (z + dz));
            for (int d = 0; d < 3; ++d) {
                const long long c = 3 * nd + d;
                col_idx[base + pos + d] = (int32_t)c;
                if (c == r) {
                    diag_slot = pos + d;
                } else {
                    const unsigned long long h = hash64(skv, ((unsigned long long)r << 32) + (unsigned long long)c);
                    const double v = -((double)(h >> 44) + 1.0) * 0x1p-20;
                    off_sum += -v;
                    values[base + pos + d] = (R)v;
                }
            }
        }
        const int nst = 3 * __popc(ball);
        const long long k = n_extra(g, r);
        if (k > 0) {
            const long long h0 = (long long)(hash64(skc, (unsigned long long)r) % (unsigned long long)g.W);
            for (long long j = lane; j < k; j += 32) {
                const long long t = (h0 + j * g.P) % g.W;
                const long long c = (r + g.band + 1 + t) % g.n;
                const unsigned long long eh = hash64(skh, ((unsigned long long)r << 32) + (unsigned long long)c) >> 40;
                const double v = (double)((long long)(eh % (unsigned long long)(2 * HUB_VAL_K + 1)) - HUB_VAL_K) * 0x1p-30;
                col_idx[base + nst + j] = (int32_t)c;
                values[base + nst + j] = (R)v;
                off_sum += fabs(v);
            }
        }
        // every partial sum is exact (all terms on the 2^-30 grid, |sum| < 2^8)
#pragma unroll
        for (int o = 16; o >= 1; o >>= 1) off_sum += __shfl_xor_sync(kFull, off_sum, o);
        if (diag_slot >= 0) values[base + diag_slot] = (R)(1.0 + off_sum);
    }
}

static int grid_for(int64_t items, int per_block) {
    int64_t g = (items + per_block - 1) / per_block;
    const int64_t cap = 8LL * sm_count();
    if (g > cap) g = cap;
    return (int)(g < 1 ? 1 : g);
}

}  // namespace synth
}  // namespace bj

using namespace bj;
using namespace bj::synth;

extern "C" bj_status bj_synth_sizes(int64_t nblocks, int64_t first, int lo, int hi, uint64_t seed, int32_t *sizes,
                                    bj_stream_t stream) {
    if (nblocks < 0 || (nblocks > 0 && !sizes) || hi < lo) return BJ_ERR_ARG;
    if (nblocks == 0) return BJ_OK;
    k_sizes<<<grid_for(nblocks, 256), 256, 0, (cudaStream_t)stream>>>(nblocks, first, lo, hi, seed_key(seed), sizes);
    BJ_LAUNCH_CHECK();
    return BJ_OK;
}

extern "C" bj_status bj_synth_blocks(const bj_batch *batch, int64_t first, int kind, bj_stream_t stream) {
    if (!batch || batch->nblocks < 0 || (kind != 0 && kind != 1)) return BJ_ERR_ARG;
    if (batch->nblocks == 0) return BJ_OK;
    const int g = grid_for(batch->nblocks * 32, 256);
    if (batch->dtype == BJ_F64)
        k_blocks<double><<<g, 256, 0, (cudaStream_t)stream>>>(batch->nblocks, first, kind, batch->sizes,
                                                               batch->val_off, (double *)batch->values);
    else if (batch->dtype == BJ_F32)
        k_blocks<float><<<g, 256, 0, (cudaStream_t)stream>>>(batch->nblocks, first, kind, batch->sizes,
                                                              batch->val_off, (float *)batch->values);
    else
        return BJ_ERR_ARG;
    BJ_LAUNCH_CHECK();
    return BJ_OK;
}

extern "C" bj_status bj_synth_rhs(const bj_batch *batch, int64_t first, void *b, bj_stream_t stream) {
    if (!batch || !b || batch->nblocks < 0) return BJ_ERR_ARG;
    if (batch->nblocks == 0) return BJ_OK;
    const int g = grid_for(batch->nblocks * 32, 256);
    if (batch->dtype == BJ_F64)
        k_rhs<double><<<g, 256, 0, (cudaStream_t)stream>>>(batch->nblocks, first, batch->sizes, batch->vec_off,
                                                            (double *)b);
    else if (batch->dtype == BJ_F32)
        k_rhs<float><<<g, 256, 0, (cudaStream_t)stream>>>(batch->nblocks, first, batch->sizes, batch->vec_off,
                                                           (float *)b);
    else
        return BJ_ERR_ARG;
    BJ_LAUNCH_CHECK();
    return BJ_OK;
}

extern "C" bj_status bj_synth_fem_row_ptr(int nx, int ny, int nz, int skew, int64_t r0, int64_t r1,
                                          int64_t *row_ptr, bj_stream_t stream) {
    if (nx <= 0 || ny <= 0 || nz <= 0 || r0 < 0 || r1 < r0 || !row_ptr) return BJ_ERR_ARG;
    const Grid g = make_grid(nx, ny, nz, skew);
    if (r1 > g.n) return BJ_ERR_ARG;
    return run_scan(FemRowPtrF{g, r0, row_ptr}, r1 - r0, (cudaStream_t)stream);
}

extern "C" bj_status bj_synth_fem_fill(int nx, int ny, int nz, int skew, int64_t r0, int64_t r1,
                                       const int64_t *row_ptr, int32_t *col_idx, void *values, bj_dtype dtype,
                                       bj_stream_t stream) {
    if (nx <= 0 || ny <= 0 || nz <= 0 || r0 < 0 || r1 < r0 || !row_ptr || !col_idx || !values) return BJ_ERR_ARG;
    const Grid g = make_grid(nx, ny, nz, skew);
    if (r1 > g.n) return BJ_ERR_ARG;
    if (r1 == r0) return BJ_OK;
    const int gr = grid_for((r1 - r0) * 32, 256);
    if (dtype == BJ_F64)
        k_fem_fill<double><<<gr, 256, 0, (cudaStream_t)stream>>>(g, r0, r1 - r0, row_ptr, col_idx, (double *)values);
    else if (dtype == BJ_F32)
        k_fem_fill<float><<<gr, 256, 0, (cudaStream_t)stream>>>(g, r0, r1 - r0, row_ptr, col_idx, (float *)values);
    else
        return BJ_ERR_ARG;
    BJ_LAUNCH_CHECK();
    return BJ_OK;
}
