// krylov.cu -- NEXT(4) of SURVEY 8(f): the block-Jacobi preconditioned
// Krylov solve that the paper uses the preconditioner for (section IV.D,
// b = ones, x0 = 0, stop at a 10^6 residual reduction, <= 10,000
// iterations; the preconditioner is applied once per step).  The
// paper's solver is IDR(4) from MAGMA-sparse; this build runs BiCGSTAB
// (reading R29).  Every reduction runs in a fixed order (R27 SpMV, R28 dot,
// R30 rank-ordered sum across shards) so the solve is bit-reproducible and
// equal to the oracle (oracle/bj_oracle.c bjo_spmv_d / bjo_dot_d /
// bjo_bicgstab_d).
//
// Kernels (fp64; all HBM/L2 streaming, no tensor cores -- nothing here is a
// dense contraction):
//   k_spmv        persistent, one warp per row, tasks of 32 rows; a row's
//                 entries are read in 128-entry passes (4 independent
//                 col/val loads per lane, then 4 gathers of x, then the fma
//                 chain in R27 order), two rows per pass for memory-level
//                 parallelism; row pointers of a task come from one
//                 coalesced load + uniform SHFLs.  Rows longer than kLongRow
//                 entries are queued for k_spmv_long.
//   k_spmv_long   one 512-thread CTA per queued long row: warps 1..15 stage
//                 (val, x[col]) of 4096-entry slices in shared memory (double
//                 buffer) while warp 0 runs the 32 lane chains of R27 over
//                 the staged slice -- the chains are sequential by definition,
//                 so the slice loads are what must be hidden.
//   k_dot         one 256-thread CTA per 8192-element chunk (R28 exactly),
//                 up to two dots per pass; the xr variant also performs the
//                 x / r updates of the iteration and dots (r, r), (rh, r).
//   k_phase       one warp: chunk sums in chunk order, the scalar recurrences
//                 of R29 (alpha, omega, residual test, beta) in device memory.
//   elementwise   p and s updates (grid-stride, 16-byte loads).
// The preconditioner is bj_apply (GETRS per block, or the GEMV of an inverse
// handle).  The host loop enqueues iterations without waiting; a completion
// flag written by the device is polled two iterations behind.
#include <math.h>
#include <string.h>

#include <vector>

#include "common.cuh"
#include "internal.h"

namespace bj {
namespace krylov {

constexpr int kChunk = 8192;        // R28: elements per chunk
constexpr int kDotThreads = 256;    // R28: partial sums per chunk
constexpr int kSpmvThreads = 256;
constexpr int kLongRow = 2048;      // rows with more entries take k_spmv_long
constexpr int kLongThreads = 512;
constexpr int kSlice = 4096;        // entries staged per k_spmv_long slice

// Device-resident solver state (R29).
struct Scalars {
    double rho, rho_prev, alpha, omega, beta;
    double nb_norm, res, thresh, tol;
    int it;        // current iteration (1-based)
    int done;      // 0 running, 1 converged, 2 maxit reached
    int maxit;
    int iters;     // reported iteration count
};

// ---------------------------------------------------------------- SpMV (R27)

__device__ __forceinline__ double ld_stream(const double *p) { return __ldcs(p); }
__device__ __forceinline__ int ld_stream(const int32_t *p) { return __ldcs(p); }

// R27 with 8 lanes per row: lane lg of a row's group holds the lane
// partials p = lg + 8q (q = 0..3).  Partial p accumulates the row's entries
// p, p + 32, p + 64, ...; numbering the lane's entries lg + 8t (t = 0, 1, ...)
// gives p = lg + 8 (t mod 4), and for a fixed q the slots t = q, q + 4, ...
// come in increasing order -- the lane runs the four chains interleaved, each
// in R27's order.  Butterfly: s_p += s_(p^16) and s_p += s_(p^8) are
// in-lane adds (q^2, q^1); s_p += s_(p^4), (p^2), (p^1) are SHFL-xors inside
// the group; y_i = s_0 = lane lg = 0, q = 0.
constexpr int kGrp = 8;             // lanes per row
constexpr int kSlots = 12;          // entries per lane per pass (96 per row)

__device__ __forceinline__ double group_reduce(const double (&s)[4]) {
    double u = (s[0] + s[2]) + (s[1] + s[3]);           // offsets 16 and 8
    u = u + __shfl_xor_sync(0xffffffffu, u, 4);
    u = u + __shfl_xor_sync(0xffffffffu, u, 2);
    u = u + __shfl_xor_sync(0xffffffffu, u, 1);
    return u;
}

// Rows of more than kLongRow entries (computed by k_spmv_long).
__global__ void k_classify_long(int64_t n, const int64_t *__restrict__ rp, int32_t *long_rows, int32_t *nlong) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        if (rp[i + 1] - rp[i] > kLongRow) long_rows[atomicAdd(nlong, 1)] = (int32_t)i;
}

__global__ void __launch_bounds__(kSpmvThreads, 3) k_spmv(int64_t n, const int64_t *__restrict__ rp,
                                                          const int32_t *__restrict__ ci,
                                                          const double *__restrict__ val, int64_t coff,
                                                          const double *__restrict__ x, double *__restrict__ y,
                                                          const int *done) {
    if (done && *done) return;
    const int lane = threadIdx.x & 31, g = lane >> 3, lg = lane & 7;
    const int64_t warp = (int64_t)blockIdx.x * (kSpmvThreads / 32) + (threadIdx.x >> 5);
    const int64_t nwarps = (int64_t)gridDim.x * (kSpmvThreads / 32);
    const int64_t ntask = (n + 31) / 32;
    const double *xs = x - coff;                         // x indexed by the stored column id
    for (int64_t task = warp; task < ntask; task += nwarps) {
        const int64_t r0 = task * 32;
        const int nr = (int)min((int64_t)32, n - r0);
        const int64_t myp = rp[r0 + min(lane, nr - 1)];  // lane l: rp[r0 + l]
        const int64_t lastp = rp[r0 + nr];
        for (int k = 0; k < nr; k += 4) {
            const int kr = k + g;                        // this group's row of the quad
            const int64_t b = __shfl_sync(0xffffffffu, myp, kr & 31);
            const int64_t e1 = __shfl_sync(0xffffffffu, myp, (kr + 1) & 31);
            const int64_t e = (kr + 1 < nr) ? e1 : lastp;
            int len = kr < nr ? (int)(e - b) : 0;
            const bool skip = len > kLongRow;            // k_spmv_long's row
            if (skip) len = 0;
            const int maxlen = __reduce_max_sync(0xffffffffu, len);
            const int32_t *cp = ci + b + lg;
            const double *vp = val + b + lg;
            const int rem = len - lg;                    // entries of this lane: offsets 8t < rem
            double s[4] = {0.0, 0.0, 0.0, 0.0};
            for (int base = 0; base < maxlen; base += kGrp * kSlots) {
                int c[kSlots];
                double v[kSlots], xv[kSlots];
#pragma unroll
                for (int t = 0; t < kSlots; ++t) {
                    const int o = base + 8 * t;
                    c[t] = 0;
                    v[t] = 0.0;
                    if (o < rem) { c[t] = ld_stream(cp + o); v[t] = ld_stream(vp + o); }
                }
#pragma unroll
                for (int t = 0; t < kSlots; ++t) xv[t] = (base + 8 * t < rem) ? xs[c[t]] : 0.0;
#pragma unroll
                for (int t = 0; t < kSlots; ++t)
                    if (base + 8 * t < rem) s[t & 3] = fma(v[t], xv[t], s[t & 3]);
            }
            const double u = group_reduce(s);
            if (lg == 0 && kr < nr && !skip) y[r0 + kr] = u;
        }
    }
}

// k_spmv over an explicit list of rows (multi-rank solves: interior rows
// while the halo is in flight, then the boundary rows).  Same per-row code
// and order as k_spmv; tasks of 32 listed rows, row pointers per lane.
__global__ void __launch_bounds__(kSpmvThreads, 3) k_spmv_rows(int64_t nlist, const int32_t *__restrict__ list,
                                                               const int64_t *__restrict__ rp,
                                                               const int32_t *__restrict__ ci,
                                                               const double *__restrict__ val,
                                                               const double *__restrict__ x,
                                                               double *__restrict__ y, const int *done) {
    if (done && *done) return;
    const int lane = threadIdx.x & 31, g = lane >> 3, lg = lane & 7;
    const int64_t warp = (int64_t)blockIdx.x * (kSpmvThreads / 32) + (threadIdx.x >> 5);
    const int64_t nwarps = (int64_t)gridDim.x * (kSpmvThreads / 32);
    const int64_t ntask = (nlist + 31) / 32;
    for (int64_t task = warp; task < ntask; task += nwarps) {
        const int64_t t0 = task * 32;
        const int nr = (int)min((int64_t)32, nlist - t0);
        const int myrow = list[t0 + min(lane, nr - 1)];
        const int64_t myb = rp[myrow], mye = rp[myrow + 1];
        for (int k = 0; k < nr; k += 4) {
            const int kr = k + g;
            const int row = __shfl_sync(0xffffffffu, myrow, kr & 31);
            const int64_t b = __shfl_sync(0xffffffffu, myb, kr & 31);
            const int64_t e = __shfl_sync(0xffffffffu, mye, kr & 31);
            int len = kr < nr ? (int)(e - b) : 0;
            const bool skip = len > kLongRow;            // k_spmv_long's row
            if (skip) len = 0;
            const int maxlen = __reduce_max_sync(0xffffffffu, len);
            const int32_t *cp = ci + b + lg;
            const double *vp = val + b + lg;
            const int rem = len - lg;
            double s[4] = {0.0, 0.0, 0.0, 0.0};
            for (int base = 0; base < maxlen; base += kGrp * kSlots) {
                int c[kSlots];
                double v[kSlots], xv[kSlots];
#pragma unroll
                for (int t = 0; t < kSlots; ++t) {
                    const int o = base + 8 * t;
                    c[t] = 0;
                    v[t] = 0.0;
                    if (o < rem) { c[t] = ld_stream(cp + o); v[t] = ld_stream(vp + o); }
                }
#pragma unroll
                for (int t = 0; t < kSlots; ++t) xv[t] = (base + 8 * t < rem) ? x[c[t]] : 0.0;
#pragma unroll
                for (int t = 0; t < kSlots; ++t)
                    if (base + 8 * t < rem) s[t & 3] = fma(v[t], xv[t], s[t & 3]);
            }
            const double u = group_reduce(s);
            if (lg == 0 && kr < nr && !skip) y[row] = u;
        }
    }
}

// Rows with a halo column (local extended id >= n) -> boundary list, the
// others -> interior list (warp per row; append order is irrelevant).
__global__ void k_split_rows(int64_t n, const int64_t *__restrict__ rp, const int32_t *__restrict__ ci,
                             int32_t *interior, int32_t *ninterior, int32_t *boundary, int32_t *nboundary) {
    const int lane = threadIdx.x & 31;
    const int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t i = warp; i < n; i += nwarps) {
        bool remote = false;
        for (int64_t e = rp[i] + lane; e < rp[i + 1]; e += 32) remote = remote || ci[e] >= n;
        remote = __any_sync(0xffffffffu, remote);
        if (lane == 0) {
            if (remote) boundary[atomicAdd(nboundary, 1)] = (int32_t)i;
            else interior[atomicAdd(ninterior, 1)] = (int32_t)i;
        }
    }
}

// Full 32-lane butterfly of R27 (k_spmv_long: warp 0 holds s_l in lane l).
__device__ __forceinline__ double butterfly(double s) {
#pragma unroll
    for (int off = 16; off >= 1; off >>= 1) s = s + __shfl_xor_sync(0xffffffffu, s, off);
    return s;
}

// One CTA per long row (grid-stride over the queue).  Warp 0 owns the 32
// chains; warps 1..15 stage slices of (val, x[col]) into shared memory.
__global__ void __launch_bounds__(kLongThreads) k_spmv_long(const int64_t *__restrict__ rp,
                                                           const int32_t *__restrict__ ci,
                                                           const double *__restrict__ val, int64_t coff,
                                                           const double *__restrict__ x, double *__restrict__ y,
                                                           const int32_t *long_rows, const int32_t *nlong,
                                                           const int *done) {
    if (done && *done) return;
    extern __shared__ double sm[];            // [2][2][kSlice]: val, xval
    const int nq = *nlong;
    const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
    constexpr int kLoaders = kLongThreads - 32;
    for (int q = blockIdx.x; q < nq; q += gridDim.x) {
        const int64_t i = long_rows[q];
        const int64_t beg = rp[i], end = rp[i + 1];
        const int64_t len = end - beg;
        const int nslice = (int)((len + kSlice - 1) / kSlice);
        double s = 0.0;
        auto load = [&](int sl) {
            double *bv = sm + (sl & 1) * 2 * kSlice, *bx = bv + kSlice;
            const int64_t base = beg + (int64_t)sl * kSlice;
            const int cnt = (int)min((int64_t)kSlice, end - base);
            for (int e = tid - 32; e < cnt; e += kLoaders) {
                bv[e] = ld_stream(val + base + e);
                bx[e] = x[ld_stream(ci + base + e) - coff];
            }
        };
        if (w > 0) load(0);
        __syncthreads();
        for (int sl = 0; sl < nslice; ++sl) {
            if (w > 0) {
                if (sl + 1 < nslice) load(sl + 1);
            } else {
                const double *bv = sm + (sl & 1) * 2 * kSlice, *bx = bv + kSlice;
                const int cnt = (int)min((int64_t)kSlice, end - beg - (int64_t)sl * kSlice);
                // entries of lane l in this slice: l, l+32, ... (slice starts are multiples of 32)
                int e = lane;
                for (; e + 96 < cnt; e += 128) {
                    s = fma(bv[e], bx[e], s);
                    s = fma(bv[e + 32], bx[e + 32], s);
                    s = fma(bv[e + 64], bx[e + 64], s);
                    s = fma(bv[e + 96], bx[e + 96], s);
                }
                for (; e < cnt; e += 32) s = fma(bv[e], bx[e], s);
            }
            __syncthreads();
        }
        if (w == 0) {
            s = butterfly(s);
            if (lane == 0) y[i] = s;
        }
        __syncthreads();
    }
}

// ------------------------------------------------------------------ dot (R28)

// Tree of R28 over the 256 partials of a CTA: s_t += s_(t+h), h = 128..1.
// Levels h >= 32 through shared memory, h <= 16 by shuffles (same operands).
template <int ND>
__device__ __forceinline__ void tree256(double (&s)[ND], double (*sh)[kDotThreads], double *out) {
    const int t = threadIdx.x;
#pragma unroll
    for (int d = 0; d < ND; ++d) sh[d][t] = s[d];
    __syncthreads();
#pragma unroll
    for (int h = 128; h >= 32; h >>= 1) {
        if (t < h) {
#pragma unroll
            for (int d = 0; d < ND; ++d) sh[d][t] = sh[d][t] + sh[d][t + h];
        }
        __syncthreads();
    }
    if (t < 32) {
#pragma unroll
        for (int d = 0; d < ND; ++d) {
            double v = sh[d][t];
#pragma unroll
            for (int h = 16; h >= 1; h >>= 1) v = v + __shfl_down_sync(0xffffffffu, v, h);
            if (t == 0) out[d] = v;
        }
    }
}

// Partials of dot(a_d, b_d), d < ND, chunk = blockIdx.x; P[chunk * 4 + d].
template <int ND>
__global__ void __launch_bounds__(kDotThreads) k_dot(int64_t n, const double *__restrict__ a0,
                                                    const double *__restrict__ b0,
                                                    const double *__restrict__ a1,
                                                    const double *__restrict__ b1, double *P,
                                                    const int *done) {
    if (done && *done) return;
    __shared__ double sh[ND][kDotThreads];
    const int64_t base = (int64_t)blockIdx.x * kChunk + threadIdx.x;
    double s[ND];
#pragma unroll
    for (int d = 0; d < ND; ++d) s[d] = 0.0;
    // loads of 8 chain steps ahead of their fmas; chain in R28 order
#pragma unroll
    for (int j0 = 0; j0 < 32; j0 += 8) {
        double va[ND][8], vb[ND][8];
#pragma unroll
        for (int d = 0; d < ND; ++d) {
            const double *a = d == 0 ? a0 : a1, *b = d == 0 ? b0 : b1;
#pragma unroll
            for (int j = 0; j < 8; ++j) {
                const int64_t k = base + 256 * (j0 + j);
                va[d][j] = k < n ? a[k] : 0.0;
                vb[d][j] = k < n ? b[k] : 0.0;
            }
        }
#pragma unroll
        for (int d = 0; d < ND; ++d)
#pragma unroll
            for (int j = 0; j < 8; ++j)
                if (base + 256 * (j0 + j) < n) s[d] = fma(va[d][j], vb[d][j], s[d]);
    }
    tree256<ND>(s, sh, P + (int64_t)blockIdx.x * 4);
}

// The end of an iteration (R29), chunk by chunk: x = fma(omega, sh, fma(alpha,
// ph, x)); r = fma(-omega, t, s); partials of dot(r, r) and dot(rh, r).
__global__ void __launch_bounds__(kDotThreads) k_xr(int64_t n, const Scalars *S, double *__restrict__ x,
                                                   double *__restrict__ r, const double *__restrict__ ph,
                                                   const double *__restrict__ shv, const double *__restrict__ t,
                                                   const double *__restrict__ s, const double *__restrict__ rh,
                                                   double *P) {
    if (S->done) return;
    __shared__ double sh[2][kDotThreads];
    const double alpha = S->alpha, omega = S->omega;
    const int64_t base = (int64_t)blockIdx.x * kChunk + threadIdx.x;
    double acc[2] = {0.0, 0.0};
#pragma unroll 4
    for (int j = 0; j < 32; ++j) {
        const int64_t k = base + 256 * j;
        if (k < n) {
            const double xn = fma(omega, shv[k], fma(alpha, ph[k], x[k]));
            const double rn = fma(-omega, t[k], s[k]);
            x[k] = xn;
            r[k] = rn;
            acc[0] = fma(rn, rn, acc[0]);
            acc[1] = fma(rh[k], rn, acc[1]);
        }
    }
    tree256<2>(acc, sh, P + (int64_t)blockIdx.x * 4);
}

// ------------------------------------------------------- elementwise updates

__global__ void k_pupdate(int64_t n, const Scalars *S, double *__restrict__ p, const double *__restrict__ v,
                          const double *__restrict__ r) {
    if (S->done) return;
    const double beta = S->beta, om = -S->omega;
    for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < n; k += (int64_t)gridDim.x * blockDim.x)
        p[k] = fma(beta, fma(om, v[k], p[k]), r[k]);
}

__global__ void k_supdate(int64_t n, const Scalars *S, double *__restrict__ s, const double *__restrict__ v,
                          const double *__restrict__ r) {
    if (S->done) return;
    const double na = -S->alpha;
    for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < n; k += (int64_t)gridDim.x * blockDim.x)
        s[k] = fma(na, v[k], r[k]);
}

__global__ void k_init(int64_t n, const double *__restrict__ b, double *x, double *r, double *rh, double *p,
                       double *v) {
    for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < n; k += (int64_t)gridDim.x * blockDim.x) {
        const double bk = b[k];
        x[k] = 0.0; r[k] = bk; rh[k] = bk; p[k] = 0.0; v[k] = 0.0;
    }
}

__global__ void k_pack(int64_t m, const int32_t *__restrict__ idx, const double *__restrict__ src,
                       double *__restrict__ dst, const int *done) {
    if (done && *done) return;
    for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < m; k += (int64_t)gridDim.x * blockDim.x)
        dst[k] = src[idx[k]];
}

__global__ void k_unpack(int64_t m, const double *__restrict__ src, double *__restrict__ dst, const int *done) {
    if (done && *done) return;
    for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < m; k += (int64_t)gridDim.x * blockDim.x)
        dst[k] = src[k];
}

// ---------------------------------------------------------- scalar phases

enum Phase { kInit = 0, kAlpha = 1, kOmega = 2, kResid = 3, kDotOut = 4 };

// The scalar recurrences of R29 given the global dot values g[].
__device__ void phase_apply(int phase, const double *g, Scalars *S, double *out) {
    switch (phase) {
    case kInit:                       // g0 = dot(b, b) = dot(rh, r) of iteration 1
        S->nb_norm = sqrt(g[0]);
        S->thresh = S->tol * S->nb_norm;
        S->rho = g[0];
        S->rho_prev = 1.0;
        S->alpha = 1.0;
        S->omega = 1.0;
        S->beta = (S->rho / S->rho_prev) * (S->alpha / S->omega);
        S->res = 1.0;
        S->it = 1;
        S->iters = S->maxit + 1;
        S->done = S->maxit < 1 ? 2 : 0;
        break;
    case kAlpha:                      // g0 = dot(rh, v)
        S->alpha = S->rho / g[0];
        break;
    case kOmega:                      // g0 = dot(t, s), g1 = dot(t, t)
        S->omega = g[0] / g[1];
        break;
    case kResid:                      // g0 = dot(r, r), g1 = dot(rh, r) (next rho)
        S->res = sqrt(g[0]);
        if (S->res <= S->thresh) {
            S->done = 1;
            S->iters = S->it;
        } else {
            S->rho_prev = S->rho;
            S->rho = g[1];
            S->beta = (S->rho / S->rho_prev) * (S->alpha / S->omega);
            if (S->it >= S->maxit) S->done = 2;
            else S->it += 1;
        }
        break;
    case kDotOut:
        *out = g[0];
        break;
    }
}

// Rank-local stage: chunk sums (R28: in chunk order from +0) -- the
// partials are staged in shared memory by all threads (one round trip), then
// one thread adds them in order.  With gather != nullptr the rank values are
// published for the caller's allgather, else the phase completes here.
constexpr int kPhaseThreads = 256;
constexpr int kPhaseStage = 512;    // chunks staged per round
__global__ void __launch_bounds__(kPhaseThreads) k_phase_local(int phase, int nd, const double *P, int64_t nc,
                                                               Scalars *S, double *gather, int rank,
                                                               double *out) {
    if (S && phase != kInit && S->done) return;
    __shared__ double sp[kPhaseStage * 4];
    double g[4] = {0.0, 0.0, 0.0, 0.0};
    for (int64_t c0 = 0; c0 < nc; c0 += kPhaseStage) {
        const int cnt = (int)min((int64_t)kPhaseStage, nc - c0);
        for (int i = threadIdx.x; i < cnt * 4; i += kPhaseThreads) sp[i] = P[c0 * 4 + i];
        __syncthreads();
        if (threadIdx.x == 0) {
            for (int c = 0; c < cnt; ++c) {
#pragma unroll
                for (int d = 0; d < 4; ++d)
                    if (d < nd) g[d] = g[d] + sp[c * 4 + d];
            }
        }
        __syncthreads();
    }
    if (threadIdx.x != 0) return;
    if (gather) {
#pragma unroll
        for (int d = 0; d < 4; ++d)
            if (d < nd) gather[rank * 4 + d] = g[d];
        return;
    }
    phase_apply(phase, g, S, out);
}

// After the allgather: global value = sum over ranks in rank order from +0 (R30).
__global__ void k_phase_global(int phase, int nd, const double *gather, int nranks, Scalars *S) {
    if (threadIdx.x != 0 || blockIdx.x != 0) return;
    if (phase != kInit && S->done) return;
    double g[4] = {0.0, 0.0, 0.0, 0.0};
#pragma unroll
    for (int d = 0; d < 4; ++d) {
        double acc = 0.0;
        if (d < nd)
            for (int r = 0; r < nranks; ++r) acc = acc + gather[r * 4 + d];
        g[d] = acc;
    }
    phase_apply(phase, g, S, nullptr);
}

// ------------------------------------------------------------- host side

int elem_grid() { return sm_count() * 8; }

// Optional side stream for k_spmv_long: the few long rows run concurrently
// with k_spmv (fork / join by events).
struct LongCtx {
    cudaStream_t side = nullptr;
    cudaEvent_t fork = nullptr, join = nullptr;
};
constexpr int kLongGrid = 32;

bj_status launch_spmv(const bj_csr &A, const double *x, double *y, const int32_t *long_rows,
                      const int32_t *nlong, const int *done, cudaStream_t s, const LongCtx *lc) {
    const int64_t n = A.nrows;
    if (n == 0) return BJ_OK;
    static int smem_set[64] = {0};
    int dev = 0;
    cudaGetDevice(&dev);
    if (dev >= 0 && dev < 64 && !smem_set[dev]) {
        BJ_CUDA_TRY(cudaFuncSetAttribute(k_spmv_long, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         (int)(4 * kSlice * sizeof(double))));
        smem_set[dev] = 1;
    }
    const double *vals = (const double *)A.values;
    cudaStream_t ls = s;
    if (lc) {
        BJ_CUDA_TRY(cudaEventRecord(lc->fork, s));
        BJ_CUDA_TRY(cudaStreamWaitEvent(lc->side, lc->fork, 0));
        ls = lc->side;
    }
    k_spmv_long<<<kLongGrid, kLongThreads, 4 * kSlice * sizeof(double), ls>>>(A.row_ptr, A.col_idx, vals,
                                                                              A.col_offset, x, y, long_rows,
                                                                              nlong, done);
    BJ_LAUNCH_CHECK();
    if (lc) BJ_CUDA_TRY(cudaEventRecord(lc->join, ls));
    const int grid = persistent_grid(k_spmv, kSpmvThreads);
    k_spmv<<<grid, kSpmvThreads, 0, s>>>(n, A.row_ptr, A.col_idx, vals, A.col_offset, x, y, done);
    BJ_LAUNCH_CHECK();
    if (lc) BJ_CUDA_TRY(cudaStreamWaitEvent(s, lc->join, 0));
    return BJ_OK;
}

bj_status classify_long(const bj_csr &A, int32_t *long_rows, int32_t *nlong, cudaStream_t s) {
    BJ_CUDA_TRY(cudaMemsetAsync(nlong, 0, sizeof(int32_t), s));
    if (A.nrows == 0) return BJ_OK;
    k_classify_long<<<elem_grid(), 256, 0, s>>>(A.nrows, A.row_ptr, long_rows, nlong);
    BJ_LAUNCH_CHECK();
    return BJ_OK;
}

bj_status check_csr64(const bj_csr *A) {
    if (!A || A->nrows < 0 || A->nnz < 0 || A->dtype != BJ_F64) return BJ_ERR_ARG;
    if (A->nrows >= ((int64_t)1 << 31)) return BJ_ERR_ARG;              // row ids are int32 in the queue
    if (!A->row_ptr || (A->nnz > 0 && (!A->col_idx || !A->values))) return BJ_ERR_ARG;
    return BJ_OK;
}

}  // namespace krylov
}  // namespace bj

using namespace bj;
using namespace bj::krylov;

extern "C" bj_status bj_spmv(const bj_csr *A, const double *x, double *y, bj_stream_t stream) {
    bj_status st = check_csr64(A);
    if (st != BJ_OK) return st;
    if (A->nrows == 0) return BJ_OK;
    if (!x || !y) return BJ_ERR_ARG;
    cudaStream_t s = (cudaStream_t)stream;
    AsyncScratch scr(s);
    const int64_t cap = A->nnz / kLongRow + 2;
    BJ_CUDA_TRY(cudaMallocAsync((void **)&scr.p, (size_t)(cap + 1) * sizeof(int32_t), s));
    int32_t *nlong = (int32_t *)scr.p, *long_rows = nlong + 1;
    if ((st = classify_long(*A, long_rows, nlong, s)) != BJ_OK) return st;
    // per-device side stream + events for the long rows (created once, kept)
    static LongCtx cached[64];
    int dev = 0;
    cudaGetDevice(&dev);
    LongCtx *lc = nullptr;
    if (dev >= 0 && dev < 64) {
        lc = &cached[dev];
        if (!lc->side) {
            BJ_CUDA_TRY(cudaStreamCreateWithFlags(&lc->side, cudaStreamNonBlocking));
            BJ_CUDA_TRY(cudaEventCreateWithFlags(&lc->fork, cudaEventDisableTiming));
            BJ_CUDA_TRY(cudaEventCreateWithFlags(&lc->join, cudaEventDisableTiming));
        }
    }
    return launch_spmv(*A, x, y, long_rows, nlong, nullptr, s, lc);
}

extern "C" bj_status bj_dot(int64_t n, const double *x, const double *y, double *result, bj_stream_t stream) {
    if (n < 0 || !result || (n > 0 && (!x || !y))) return BJ_ERR_ARG;
    cudaStream_t s = (cudaStream_t)stream;
    const int64_t nc = (n + kChunk - 1) / kChunk;
    AsyncScratch scr(s);
    BJ_CUDA_TRY(cudaMallocAsync((void **)&scr.p, (size_t)(nc > 0 ? nc : 1) * 4 * sizeof(double), s));
    double *P = (double *)scr.p;
    if (nc > 0) {
        k_dot<1><<<(unsigned)nc, kDotThreads, 0, s>>>(n, x, y, nullptr, nullptr, P, nullptr);
        BJ_LAUNCH_CHECK();
    }
    k_phase_local<<<1, kPhaseThreads, 0, s>>>(kDotOut, 1, P, nc, nullptr, nullptr, 0, result);
    BJ_LAUNCH_CHECK();
    return BJ_OK;
}

namespace bj {
namespace krylov {
// dot phase: chunk partials already in P; completes the phase (comm or not)
bj_status finish_phase(int phase, int nd, const double *P, int64_t nc, Scalars *S, const bj_comm *comm,
                       cudaStream_t s) {
    k_phase_local<<<1, kPhaseThreads, 0, s>>>(phase, nd, P, nc, S, comm ? comm->gather_buf : nullptr,
                                   comm ? comm->rank : 0, nullptr);
    BJ_LAUNCH_CHECK();
    if (comm) {
        if (comm->allgather(comm->ctx, nd, (bj_stream_t)s) != 0) return BJ_ERR_COMM;
        k_phase_global<<<1, 32, 0, s>>>(phase, nd, comm->gather_buf, comm->nranks, S);
        BJ_LAUNCH_CHECK();
    }
    return BJ_OK;
}

struct RowLists {
    int32_t *interior = nullptr, *boundary = nullptr;
    int64_t ninterior = 0, nboundary = 0;
};

// Multi-rank SpMV (R27 per row, R30 solve): pack the rows peers need, start
// the halo exchange, compute the interior rows while it is in flight (when
// the caller provides halo_wait), complete it, unpack the halo behind the
// own rows of v, compute the boundary rows, then the long rows (which may
// touch the halo).
bj_status spmv_comm(const bj_csr &A, double *v, double *y, const bj_comm *comm, const RowLists &rl,
                    const int32_t *long_rows, const int32_t *nlong, const int *done, cudaStream_t s) {
    const int64_t n = A.nrows;
    const double *vals = (const double *)A.values;
    const int grid = persistent_grid(k_spmv_rows, kSpmvThreads);
    if (comm->nsend > 0) {
        k_pack<<<elem_grid(), 256, 0, s>>>(comm->nsend, comm->send_idx, v, comm->send_buf, done);
        BJ_LAUNCH_CHECK();
    }
    if (comm->halo_exchange(comm->ctx, (bj_stream_t)s) != 0) return BJ_ERR_COMM;
    auto rows = [&](const int32_t *list, int64_t cnt) -> bj_status {
        if (cnt == 0) return BJ_OK;
        k_spmv_rows<<<grid, kSpmvThreads, 0, s>>>(cnt, list, A.row_ptr, A.col_idx, vals, v, y, done);
        BJ_LAUNCH_CHECK();
        return BJ_OK;
    };
    bj_status st;
    const bool overlap = comm->halo_wait != nullptr;
    if (overlap && (st = rows(rl.interior, rl.ninterior)) != BJ_OK) return st;
    if (overlap && comm->halo_wait(comm->ctx, (bj_stream_t)s) != 0) return BJ_ERR_COMM;
    if (comm->nhalo > 0) {
        k_unpack<<<elem_grid(), 256, 0, s>>>(comm->nhalo, comm->recv_buf, v + n, done);
        BJ_LAUNCH_CHECK();
    }
    if (!overlap && (st = rows(rl.interior, rl.ninterior)) != BJ_OK) return st;
    if ((st = rows(rl.boundary, rl.nboundary)) != BJ_OK) return st;
    static int smem_set[64] = {0};
    int dev = 0;
    cudaGetDevice(&dev);
    if (dev >= 0 && dev < 64 && !smem_set[dev]) {
        BJ_CUDA_TRY(cudaFuncSetAttribute(k_spmv_long, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         (int)(4 * kSlice * sizeof(double))));
        smem_set[dev] = 1;
    }
    k_spmv_long<<<kLongGrid, kLongThreads, 4 * kSlice * sizeof(double), s>>>(A.row_ptr, A.col_idx, vals, 0, v, y,
                                                                              long_rows, nlong, done);
    BJ_LAUNCH_CHECK();
    return BJ_OK;
}
}  // namespace krylov
}  // namespace bj

extern "C" bj_status bj_bicgstab(bj_handle *M, const bj_csr *A, const bj_comm *comm, const double *b, double *x,
                                 double tol, int maxit, int *iters_h, double *resid_h, bj_stream_t stream) {
    bj_status st = check_csr64(A);
    if (st != BJ_OK) return st;
    if (!M || !iters_h || !resid_h || (A->nrows > 0 && (!b || !x))) return BJ_ERR_ARG;
    if (comm) {
        if (comm->nranks < 1 || comm->rank < 0 || comm->rank >= comm->nranks || !comm->halo_exchange ||
            !comm->allgather || !comm->gather_buf || comm->nhalo < 0 || comm->nsend < 0 || A->col_offset != 0 ||
            (comm->nsend > 0 && (!comm->send_idx || !comm->send_buf)) || (comm->nhalo > 0 && !comm->recv_buf))
            return BJ_ERR_ARG;
    }
    cudaStream_t s = (cudaStream_t)stream;
    const int64_t n = A->nrows, nh = comm ? comm->nhalo : 0, ne = n + nh;
    const int64_t nc = (n + kChunk - 1) / kChunk;
    const int64_t cap = A->nnz / kLongRow + 2;
    // scratch: 6 vectors of n, 2 of n + halo, chunk partials, scalars, long-row queue
    const size_t vec = (size_t)(n > 0 ? n : 1) * 8, vecx = (size_t)(ne > 0 ? ne : 1) * 8;
    auto up = [](size_t v) { return (v + 255) & ~(size_t)255; };
    const size_t o_r = 0, o_rh = o_r + up(vec), o_p = o_rh + up(vec), o_v = o_p + up(vec), o_s = o_v + up(vec),
                 o_t = o_s + up(vec), o_ph = o_t + up(vec), o_sh = o_ph + up(vecx), o_P = o_sh + up(vecx),
                 o_S = o_P + up((size_t)(nc > 0 ? nc : 1) * 32), o_q = o_S + up(sizeof(Scalars)),
                 o_lists = o_q + up((size_t)(cap + 1) * 4),
                 total = o_lists + (comm ? up((size_t)(2 * (n > 0 ? n : 1) + 2) * 4) : 0);
    AsyncScratch scr(s);
    BJ_CUDA_TRY(cudaMallocAsync((void **)&scr.p, total, s));
    char *base = scr.p;
    double *r = (double *)(base + o_r), *rh = (double *)(base + o_rh), *p = (double *)(base + o_p),
           *v = (double *)(base + o_v), *sv = (double *)(base + o_s), *t = (double *)(base + o_t),
           *ph = (double *)(base + o_ph), *shv = (double *)(base + o_sh), *P = (double *)(base + o_P);
    Scalars *S = (Scalars *)(base + o_S);
    int32_t *nlong = (int32_t *)(base + o_q), *long_rows = nlong + 1;
    RowLists rl{};
    const int *done = &S->done;

    // initial state; x0 = 0 also defines the halo parts of ph / sh (never read before written)
    Scalars init{};
    init.tol = tol;
    init.maxit = maxit;
    BJ_CUDA_TRY(cudaMemcpyAsync(S, &init, sizeof(Scalars), cudaMemcpyHostToDevice, s));
    if ((st = classify_long(*A, long_rows, nlong, s)) != BJ_OK) return st;
    if (comm && n > 0) {   // interior / boundary rows (counts to the host once)
        int32_t *cnt = (int32_t *)(base + o_lists);
        rl.interior = cnt + 2;
        rl.boundary = rl.interior + n;
        BJ_CUDA_TRY(cudaMemsetAsync(cnt, 0, 2 * sizeof(int32_t), s));
        k_split_rows<<<elem_grid(), 256, 0, s>>>(n, A->row_ptr, A->col_idx, rl.interior, cnt, rl.boundary, cnt + 1);
        BJ_LAUNCH_CHECK();
        int32_t hc[2] = {0, 0};
        BJ_CUDA_TRY(cudaMemcpyAsync(hc, cnt, sizeof(hc), cudaMemcpyDeviceToHost, s));
        BJ_CUDA_TRY(cudaStreamSynchronize(s));
        rl.ninterior = hc[0];
        rl.nboundary = hc[1];
    }
    BJ_CUDA_TRY(cudaMemsetAsync(ph, 0, vecx, s));
    BJ_CUDA_TRY(cudaMemsetAsync(shv, 0, vecx, s));
    if (n > 0) {
        k_init<<<elem_grid(), 256, 0, s>>>(n, b, x, r, rh, p, v);
        BJ_LAUNCH_CHECK();
        k_dot<1><<<(unsigned)nc, kDotThreads, 0, s>>>(n, b, b, nullptr, nullptr, P, nullptr);
        BJ_LAUNCH_CHECK();
    }
    if ((st = finish_phase(kInit, 1, P, nc, S, comm, s)) != BJ_OK) return st;

    // pinned ring of completion flags, polled two iterations behind
    constexpr int kRing = 4;
    int *hflag = nullptr;
    BJ_CUDA_TRY(cudaHostAlloc((void **)&hflag, kRing * sizeof(int), cudaHostAllocDefault));
    cudaEvent_t ev[kRing];
    for (int i = 0; i < kRing; ++i) cudaEventCreateWithFlags(&ev[i], cudaEventDisableTiming);
    LongCtx lc;
    cudaStreamCreateWithFlags(&lc.side, cudaStreamNonBlocking);
    cudaEventCreateWithFlags(&lc.fork, cudaEventDisableTiming);
    cudaEventCreateWithFlags(&lc.join, cudaEventDisableTiming);
    auto cleanup = [&]() {
        for (int i = 0; i < kRing; ++i) cudaEventDestroy(ev[i]);
        cudaEventDestroy(lc.fork);
        cudaEventDestroy(lc.join);
        cudaStreamDestroy(lc.side);
        cudaFreeHost(hflag);
    };
    const unsigned eg = (unsigned)elem_grid();
    bj_status err = BJ_OK;
    for (int it = 1; it <= (maxit > 0 ? maxit : 0) && err == BJ_OK; ++it) {
        do {
            if (n > 0) { k_pupdate<<<eg, 256, 0, s>>>(n, S, p, v, r); BJ_LAUNCH_CHECK(); }
            if ((err = bj_apply(M, p, ph, stream)) != BJ_OK) break;
            if ((err = comm ? spmv_comm(*A, ph, v, comm, rl, long_rows, nlong, done, s)
                            : launch_spmv(*A, ph, v, long_rows, nlong, done, s, &lc)) != BJ_OK) break;
            if (n > 0) {
                k_dot<1><<<(unsigned)nc, kDotThreads, 0, s>>>(n, rh, v, nullptr, nullptr, P, done);
                BJ_LAUNCH_CHECK();
            }
            if ((err = finish_phase(kAlpha, 1, P, nc, S, comm, s)) != BJ_OK) break;
            if (n > 0) { k_supdate<<<eg, 256, 0, s>>>(n, S, sv, v, r); BJ_LAUNCH_CHECK(); }
            if ((err = bj_apply(M, sv, shv, stream)) != BJ_OK) break;
            if ((err = comm ? spmv_comm(*A, shv, t, comm, rl, long_rows, nlong, done, s)
                            : launch_spmv(*A, shv, t, long_rows, nlong, done, s, &lc)) != BJ_OK) break;
            if (n > 0) {
                k_dot<2><<<(unsigned)nc, kDotThreads, 0, s>>>(n, t, sv, t, t, P, done);
                BJ_LAUNCH_CHECK();
            }
            if ((err = finish_phase(kOmega, 2, P, nc, S, comm, s)) != BJ_OK) break;
            if (n > 0) {
                k_xr<<<(unsigned)nc, kDotThreads, 0, s>>>(n, S, x, r, ph, shv, t, sv, rh, P);
                BJ_LAUNCH_CHECK();
            }
            if ((err = finish_phase(kResid, 2, P, nc, S, comm, s)) != BJ_OK) break;
        } while (0);
        if (err != BJ_OK) break;
        const int slot = it % kRing;
        if (cudaMemcpyAsync(hflag + slot, done, sizeof(int), cudaMemcpyDeviceToHost, s) != cudaSuccess ||
            cudaEventRecord(ev[slot], s) != cudaSuccess) { err = BJ_ERR_CUDA; break; }
        if (it >= 3) {
            const int old = (it - 2) % kRing;
            if (cudaEventSynchronize(ev[old]) != cudaSuccess) { err = BJ_ERR_CUDA; break; }
            if (hflag[old] != 0) break;
        }
    }
    if (err != BJ_OK) { cudaStreamSynchronize(s); cleanup(); return err; }
    Scalars fin{};
    if (cudaMemcpyAsync(&fin, S, sizeof(Scalars), cudaMemcpyDeviceToHost, s) != cudaSuccess ||
        cudaStreamSynchronize(s) != cudaSuccess) { cleanup(); return BJ_ERR_CUDA; }
    cleanup();
    *iters_h = fin.iters;
    *resid_h = fin.res / fin.nb_norm;
    return BJ_OK;
}

// Halo plan (HOST): bitmap of the remote columns, ascending order = owner
// order because the shards are contiguous row ranges.
extern "C" bj_status bj_halo_plan(int64_t nnz, const int32_t *col_idx_h, int64_t lo, int64_t hi, int G,
                                  const int64_t *row_bounds_h, int32_t *col_local_h, int32_t *halo_cols_h,
                                  int64_t *nhalo_h, int64_t *recv_counts_h) {
    if (nnz < 0 || G < 1 || !row_bounds_h || !nhalo_h || !recv_counts_h || lo < 0 || hi < lo ||
        (nnz > 0 && (!col_idx_h || !col_local_h || !halo_cols_h)))
        return BJ_ERR_ARG;
    const int64_t N = row_bounds_h[G];
    if (row_bounds_h[0] != 0 || hi > N || N >= ((int64_t)1 << 31)) return BJ_ERR_ARG;
    for (int q = 0; q < G; ++q)
        if (row_bounds_h[q + 1] < row_bounds_h[q]) return BJ_ERR_ARG;
    const int64_t nw = (N + 63) / 64;
    std::vector<uint64_t> bits((size_t)(nw > 0 ? nw : 1), 0);
    for (int64_t e = 0; e < nnz; ++e) {
        const int64_t c = col_idx_h[e];
        if (c < 0 || c >= N) return BJ_ERR_ARG;
        if (c < lo || c >= hi) bits[(size_t)(c >> 6)] |= (uint64_t)1 << (c & 63);
    }
    std::vector<int64_t> pre((size_t)nw + 1, 0);
    for (int64_t w = 0; w < nw; ++w) pre[(size_t)w + 1] = pre[(size_t)w] + __builtin_popcountll(bits[(size_t)w]);
    const int64_t nh = pre[(size_t)nw], nown = hi - lo;
    if (nown + nh >= ((int64_t)1 << 31)) return BJ_ERR_ARG;
    for (int64_t e = 0; e < nnz; ++e) {
        const int64_t c = col_idx_h[e];
        if (c >= lo && c < hi) {
            col_local_h[e] = (int32_t)(c - lo);
        } else {
            const uint64_t below = bits[(size_t)(c >> 6)] & ((((uint64_t)1) << (c & 63)) - 1);
            col_local_h[e] = (int32_t)(nown + pre[(size_t)(c >> 6)] + __builtin_popcountll(below));
        }
    }
    int64_t k = 0;
    for (int64_t w = 0; w < nw; ++w)
        for (uint64_t m = bits[(size_t)w]; m; m &= m - 1) halo_cols_h[k++] = (int32_t)(w * 64 + __builtin_ctzll(m));
    for (int q = 0; q < G; ++q) recv_counts_h[q] = 0;
    int q = 0;
    for (int64_t j = 0; j < nh; ++j) {
        while (q < G - 1 && halo_cols_h[j] >= row_bounds_h[q + 1]) ++q;
        recv_counts_h[q] += 1;
    }
    *nhalo_h = nh;
    return BJ_OK;
}
