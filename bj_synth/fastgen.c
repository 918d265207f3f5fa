/*
 * bj_synth/fastgen.c -- host-side C implementation of the SAME counter-based
 * input generators as bj_synth/__init__.py (numpy), for the full-size parity
 * tests and the CPU-baseline samples (the numpy version needs ~1 min per 1M
 * blocks and cannot build a 2M-row FEM CSR in reasonable time).
 *
 * Input generation only: no arithmetic of the method lives here.  Every value
 * depends only on (seed, global index); tests/test_synth.py checks this file
 * bit for bit against the numpy generator it mirrors.
 *
 * Build: gcc -std=gnu99 -O2 -fopenmp -fPIC -shared (bj_synth.build()).
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>

#define EXPORT __attribute__((visibility("default")))

static const uint64_t GOLDEN = 0x9E3779B97F4A7C15ULL;
static const uint64_t SALT = 0x632BE59BD9B4E019ULL;
static const uint64_t HUB_THRESHOLD = 9007199254740ULL;
static const int64_t HUB_CAP = 100000;
static const int64_t HUB_VAL_K = 1073741;
enum { SEED_VALUES = 2, SEED_RHS = 3, SEED_SKEW = 4, SEED_HUBCOL = 5, SEED_HUBVAL = 6, SEED_INT = 7 };

static inline uint64_t mix64(uint64_t z) {
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
    return z ^ (z >> 31);
}
static inline uint64_t seed_key(uint64_t seed) { return mix64(seed * GOLDEN + SALT); }
static inline uint64_t hash64(uint64_t sk, uint64_t idx) { return mix64(sk + (idx + 1ULL) * GOLDEN); }
static inline double uniform_pm1(uint64_t h) { return 2.0 * ((double)(h >> 11) * 0x1p-53) - 1.0; }
static inline int64_t uniform_int(uint64_t h, int64_t lo, int64_t hi) {
    const uint64_t span = (uint64_t)(hi - lo + 1);
    return lo + (int64_t)(((h >> 32) * span) >> 32);
}

/* block_values(): element (r, c) of global block g has key g*1024 + c*32 + r;
 * kind 0 = U[-1,1) (seed 2), 1 = U{-3..3} (seed 7); fp32 = rounded fp64 draw.
 * The padding between blocks is written as +0. */
#define BLOCK_VALUES(NAME, T)                                                                 \
EXPORT void NAME(int64_t nb, int64_t first, int kind, const int32_t *sizes,                 \
                 const int64_t *val_off, const int64_t *ids, T *out) {                       \
    const uint64_t sk = seed_key(kind == 0 ? SEED_VALUES : SEED_INT);                         \
    int64_t b;                                                                                \
    _Pragma("omp parallel for schedule(static, 4096)")                                        \
    for (b = 0; b < nb; ++b) {                                                                \
        const int m = sizes[b] > 0 ? sizes[b] : 0;                                            \
        const uint64_t g = (uint64_t)(ids ? ids[b] : first + b);                              \
        T *o = out + val_off[b];                                                              \
        int64_t e, n = val_off[b + 1] - val_off[b];                                           \
        for (e = 0; e < n; ++e) o[e] = (T)0;                                                  \
        for (int c = 0; c < m; ++c)                                                           \
            for (int r = 0; r < m; ++r) {                                                     \
                const uint64_t h = hash64(sk, g * 1024ULL + (uint64_t)(c * 32 + r));          \
                const double v = kind == 0 ? uniform_pm1(h) : (double)uniform_int(h, -3, 3); \
                o[r + (int64_t)c * m] = (T)v;                                                 \
            }                                                                                 \
    }                                                                                         \
}
BLOCK_VALUES(bjs_block_values_d, double)
BLOCK_VALUES(bjs_block_values_s, float)

/* rhs_values(): element r of global block g has key g*32 + r (seed 3). */
#define RHS_VALUES(NAME, T)                                                                   \
EXPORT void NAME(int64_t nb, int64_t first, const int32_t *sizes, const int64_t *vec_off,   \
                 const int64_t *ids, T *out) {                                               \
    const uint64_t sk = seed_key(SEED_RHS);                                                   \
    int64_t b;                                                                                \
    _Pragma("omp parallel for schedule(static, 4096)")                                        \
    for (b = 0; b < nb; ++b) {                                                                \
        const int m = sizes[b] > 0 ? sizes[b] : 0;                                            \
        const uint64_t g = (uint64_t)(ids ? ids[b] : first + b);                              \
        for (int r = 0; r < m; ++r) out[vec_off[b] + r] = (T)uniform_pm1(hash64(sk, g * 32ULL + (uint64_t)r)); \
    }                                                                                         \
}
RHS_VALUES(bjs_rhs_values_d, double)
RHS_VALUES(bjs_rhs_values_s, float)

/* ---------------------------------------------------------------- FEM grid
 * Mirrors bj_synth.FemGrid (27-point x 3 dofs, skewed hub rows). */
typedef struct { int64_t nx, ny, nz, n, band, W, P; int skew; } grid_t;

static grid_t make_grid(int nx, int ny, int nz, int skew) {
    static const int64_t primes[5] = {1000003, 1000033, 1000037, 1000039, 1000081};
    grid_t g;
    g.nx = nx; g.ny = ny; g.nz = nz;
    g.n = 3LL * nx * ny * nz;
    g.band = 3LL * (1 + nx + (int64_t)nx * ny) + 2;
    g.W = g.n - (2 * g.band + 1);
    g.skew = skew && g.W > 0;
    g.P = 1;
    if (g.W > 0)
        for (int i = 0; i < 5; ++i)
            if (g.W % primes[i] != 0) { g.P = primes[i]; break; }
    return g;
}

static int64_t icbrt(uint64_t v) {
    int64_t x = (int64_t)cbrt((double)v);
    while (x > 0 && (uint64_t)x * x * x > v) --x;
    while ((uint64_t)(x + 1) * (x + 1) * (x + 1) <= v) ++x;
    return x;
}

static int64_t n_extra(const grid_t *g, int64_t r) {
    if (!g->skew) return 0;
    const uint64_t sk = seed_key(SEED_SKEW);
    if ((hash64(sk, 2ULL * r) >> 11) >= HUB_THRESHOLD) return 0;
    const uint64_t uu = 1ULL + (hash64(sk, 2ULL * r + 1ULL) >> 44);
    const uint64_t v = (1000000ULL << 40) / (uu * uu);
    int64_t k = icbrt(v);
    if (k > HUB_CAP) k = HUB_CAP;
    if (k > g->W) k = g->W;
    return k;
}

static int n_stencil(const grid_t *g, int64_t r) {
    const int64_t node = r / 3;
    const int64_t x = node % g->nx, y = (node / g->nx) % g->ny, z = node / (g->nx * g->ny);
    const int cx = 1 + (x > 0) + (x < g->nx - 1);
    const int cy = 1 + (y > 0) + (y < g->ny - 1);
    const int cz = 1 + (z > 0) + (z < g->nz - 1);
    return 3 * cx * cy * cz;
}

/* row_ptr[0..r1-r0] of rows [r0, r1) (local rows). */
EXPORT int bjs_fem_row_ptr(int nx, int ny, int nz, int skew, int64_t r0, int64_t r1, int64_t *row_ptr) {
    const grid_t g = make_grid(nx, ny, nz, skew);
    if (r0 < 0 || r1 < r0 || r1 > g.n) return -1;
    const int64_t n = r1 - r0;
    int64_t i;
    row_ptr[0] = 0;
#pragma omp parallel for schedule(static, 4096)
    for (i = 0; i < n; ++i) row_ptr[i + 1] = n_stencil(&g, r0 + i) + n_extra(&g, r0 + i);
    for (i = 0; i < n; ++i) row_ptr[i + 1] += row_ptr[i];
    return 0;
}

/* columns (global ids, stencil sorted then hub extras) and values of rows [r0, r1). */
#define FEM_FILL(NAME, T)                                                                         \
EXPORT int NAME(int nx, int ny, int nz, int skew, int64_t r0, int64_t r1, const int64_t *row_ptr, \
                int32_t *col_idx, T *values) {                                                    \
    const grid_t g = make_grid(nx, ny, nz, skew);                                                 \
    if (r0 < 0 || r1 < r0 || r1 > g.n) return -1;                                                 \
    const uint64_t skv = seed_key(SEED_VALUES), skc = seed_key(SEED_HUBCOL), skh = seed_key(SEED_HUBVAL); \
    int64_t i;                                                                                    \
    _Pragma("omp parallel for schedule(dynamic, 1024)")                                          \
    for (i = 0; i < r1 - r0; ++i) {                                                               \
        const int64_t r = r0 + i, node = r / 3;                                                   \
        const int64_t x = node % g.nx, y = (node / g.nx) % g.ny, z = node / (g.nx * g.ny);        \
        int64_t p = row_ptr[i], diag = -1;                                                        \
        double off = 0.0;                                                                         \
        for (int dz = -1; dz <= 1; ++dz) {                                                        \
            if (z + dz < 0 || z + dz >= g.nz) continue;                                           \
            for (int dy = -1; dy <= 1; ++dy) {                                                    \
                if (y + dy < 0 || y + dy >= g.ny) continue;                                       \
                for (int dx = -1; dx <= 1; ++dx) {                                                \
                    if (x + dx < 0 || x + dx >= g.nx) continue;                                   \
                    const int64_t nd = (x + dx) + g.nx * ((y + dy) + g.ny * (z + dz));            \
                    for (int d = 0; d < 3; ++d, ++p) {                                            \
                        const int64_t c = 3 * nd + d;                                             \
                        col_idx[p] = (int32_t)c;                                                  \
                        if (c == r) { diag = p; continue; }                                       \
                        const uint64_t h = hash64(skv, ((uint64_t)r << 32) + (uint64_t)c);        \
                        const double v = -((double)(h >> 44) + 1.0) * 0x1p-20;                    \
                        off += -v;                                                                \
                        values[p] = (T)v;                                                         \
                    }                                                                             \
                }                                                                                 \
            }                                                                                     \
        }                                                                                         \
        const int64_t k = n_extra(&g, r);                                                         \
        if (k > 0) {                                                                              \
            const int64_t h0 = (int64_t)(hash64(skc, (uint64_t)r) % (uint64_t)g.W);               \
            for (int64_t j = 0; j < k; ++j, ++p) {                                                \
                const int64_t t = (h0 + j * g.P) % g.W;                                           \
                const int64_t c = (r + g.band + 1 + t) % g.n;                                     \
                const uint64_t eh = hash64(skh, ((uint64_t)r << 32) + (uint64_t)c) >> 40;         \
                const double v = (double)((int64_t)(eh % (uint64_t)(2 * HUB_VAL_K + 1)) - HUB_VAL_K) * 0x1p-30; \
                col_idx[p] = (int32_t)c;                                                          \
                values[p] = (T)v;                                                                 \
                off += fabs(v);                                                                   \
            }                                                                                     \
        }                                                                                         \
        /* every partial sum is exact (all terms on the 2^-30 grid, |sum| < 2^8) */              \
        if (diag >= 0) values[diag] = (T)(1.0 + off);                                             \
    }                                                                                             \
    return 0;                                                                                     \
}
FEM_FILL(bjs_fem_fill_d, double)
FEM_FILL(bjs_fem_fill_s, float)
