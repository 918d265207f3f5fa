/*
 * bj.h -- C ABI of the B200-native block-Jacobi hot path.
 *
 * Method: H. Anzt, J. Dongarra, G. Flegar, E. S. Quintana-Orti, "Variable-Size
 * Batched LU for Small Matrices and its Integration into Block-Jacobi
 * Preconditioning", ICPP 2017.  "P:n" cites line n of the paper text
 * with the section / figure it falls in; "R#" cites
 * a reading of a silent or garbled passage, listed in DESIGN.md section 3.
 *
 * Conventions shared by every call
 *  - Pointers are DEVICE pointers (cudaMalloc / torch CUDA tensors) unless the
 *    parameter name ends in _h (HOST pointer).
 *  - Calls are stream-ordered and asynchronous on `stream` (a cudaStream_t,
 *    NULL = legacy default stream); none synchronises the host except those
 *    documented as synchronous (bj_gesv_host).  The caller keeps every buffer
 *    alive until the stream work completes.
 *  - The library never allocates or frees caller data.  Library-owned memory
 *    is limited to plan metadata (bj_plan, bj_handle, bj_workspace) and
 *    stream-ordered scratch (cudaMallocAsync / cudaFreeAsync).
 *  - Dense blocks are column-major, D(i,j) = values[val_off[b] + i + j*m]
 *    (P:520-524), packed back to back; block b starts at element val_off[b],
 *    which must be a multiple of 16/sizeof(element) (16-byte aligned, R18).
 *    Vectors (pivots, right-hand sides, solutions) of block b start at element
 *    vec_off[b].  bj_layout produces exactly this layout.
 *  - Block orders m must lie in 0..32 (R10).  A block of
 *    any other order gets info[b] = -1 and is not touched; there is no CPU or
 *    other fallback path.
 *  - Return value: BJ_OK, or a host-detectable error (bad arguments, launch
 *    failure).  Data errors found on the device are reported per block in
 *    info[] without a host synchronisation.
 *  - Calls are reentrant; one bj_plan / bj_handle / bj_workspace must not be
 *    used from two host threads at once.
 */
#ifndef BJ_H
#define BJ_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct CUstream_st *bj_stream_t;      /* == cudaStream_t */

typedef enum { BJ_F32 = 0, BJ_F64 = 1 } bj_dtype;

typedef enum {
    BJ_OK = 0,
    BJ_ERR_ARG = -1,         /* null pointer, negative count, bad dtype, ...   */
    BJ_ERR_BLOCK_SIZE = -2,  /* reserved: sizes are checked per block (info=-1) */
    BJ_ERR_ALIGN = -3,       /* a base pointer is not 16-byte aligned          */
    BJ_ERR_CUDA = -4,        /* a CUDA runtime call or launch failed           */
    BJ_ERR_NOMEM = -5,       /* library scratch allocation failed              */
    BJ_ERR_STATE = -6,       /* handle used before bj_setup, ...               */
    BJ_ERR_COMM = -7         /* a bj_comm callback reported failure             */
} bj_status;

/* Sparse matrix in CSR (CSR [3]; Fig. 3).  Rows are
 * local (0..nrows-1); col_idx holds GLOBAL column ids; local column =
 * col_idx - col_offset (0 for a whole matrix; the first global row of a row
 * slab when rows are sharded over GPUs).  Columns inside a row may be
 * unsorted; (row, col) pairs must be unique (R14). */
typedef struct {
    int64_t nrows;
    int64_t nnz;
    int64_t col_offset;
    const int64_t *row_ptr;      /* [nrows+1]                                 */
    const int32_t *col_idx;      /* [nnz]                                     */
    const void    *values;       /* [nnz] of dtype                            */
    bj_dtype dtype;
} bj_csr;

/* A packed batch of dense blocks (layout above).  `values` is read and/or
 * written depending on the call; the other arrays are inputs unless a call
 * says it fills them. */
typedef struct {
    int64_t nblocks;
    int32_t *sizes;              /* [nblocks]   block orders m_b              */
    int64_t *vec_off;            /* [nblocks+1] exclusive prefix of m_b        */
    int64_t *val_off;            /* [nblocks+1] element offset of block b      */
    void    *values;             /* [val_off[nblocks]] elements of dtype       */
    bj_dtype dtype;
} bj_batch;

/* Opaque objects (library-owned device metadata). */
typedef struct bj_plan bj_plan;
typedef struct bj_handle bj_handle;
typedef struct bj_workspace bj_workspace;

const char *bj_status_string(bj_status st);
const char *bj_version(void);

/* ---------------------------------------------------------------------------
 * Hot-path row a1 -- batch layout.  n = sum m_b.
 *   vec_off[b] = sum_{c<b} m_c;  val_off[b] = sum_{c<b} roundup(m_c^2, 16/s)
 * with s = sizeof(dtype); both int64[nblocks+1] (last entry = totals).
 * Negative sizes count as 0.  Device scans; asynchronous.
 * ------------------------------------------------------------------------- */
bj_status bj_layout(int64_t nblocks, const int32_t *sizes, bj_dtype dtype,
                    int64_t *vec_off, int64_t *val_off, bj_stream_t stream);

/* Same layout from block boundaries (R15): sizes[b] = block_ptr[b+1] -
 * block_ptr[b] is written to `sizes`, vec_off[b] = block_ptr[b] - block_ptr[0]. */
bj_status bj_layout_from_block_ptr(int64_t nblocks, const int32_t *block_ptr, bj_dtype dtype,
                                   int32_t *sizes, int64_t *vec_off, int64_t *val_off,
                                   bj_stream_t stream);

/* Size-bucket plan: block ids grouped by order m (stable counting sort on the
 * device) and per-bucket task tables for the size-specialised kernels.  Reused
 * by every call that receives it while `sizes` is unchanged.  Asynchronous;
 * `sizes` must stay valid until the plan is destroyed only if the caller
 * wants to reuse it (the plan copies what it needs). */
bj_status bj_plan_create(bj_plan **plan, int64_t nblocks, const int32_t *sizes,
                         bj_stream_t stream);
/* Frees the plan's device memory stream-ordered on the creation stream (no
 * host sync): work already enqueued on that stream may still use it; work on
 * other streams must be ordered before this call by the caller. */
bj_status bj_plan_destroy(bj_plan *plan);

/* ---------------------------------------------------------------------------
 * Hot-path row a2 -- diagonal-block extraction, section III.C,
 * block-Jacobi splitting P:159-171.
 * For block b with rows bs = block_ptr[b] .. be = block_ptr[b+1]-1 (local
 * rows; block columns are bs..be-1 in local column numbering):
 *   D_b(r, c) = A(bs+r, bs+c) for every stored entry of row bs+r whose local
 *   column lies in [bs, be); every other element of D_b is +0.0.
 * Values are copied bit for bit.  `out` must carry the layout of
 * bj_layout_from_block_ptr(block_ptr) (sizes/vec_off/val_off filled by the
 * caller or by that call); out->values receives the blocks (pad elements
 * between blocks are written as +0.0).  Rows with more than a few thousand
 * stored entries are handled cooperatively (load balance for skewed rows).
 * ------------------------------------------------------------------------- */
bj_status bj_extract(const bj_csr *A, const int32_t *block_ptr, bj_batch *out,
                     bj_stream_t stream);

/* ---------------------------------------------------------------------------
 * Hot-path row a3 -- GETRF with implicit (swap-free) partial pivoting,
 * Fig. 1 bottom, section III.A.
 * Per block, for k = 0..m-1: pivot = the unpivoted row with the largest |a_ik|
 * (bits of |a| compared as unsigned, the lowest original row wins ties, R1/R2);
 * tag it; SCAL a_ik /= a_pk (IEEE division, R3) and GER a_ij = fma(-a_ik,
 * a_pj, a_ij) on the unpivoted rows (R5); rows are finally stored in pivot
 * order (combined row swap), giving P*D = L*U with unit-lower L
 * (diagonal not stored) and upper U in place of D.
 *   pivots[vec_off[b] + k] = original (0-based) row chosen at step k (R7).
 *   info[b] = 0, or k+1 for the first step whose candidates are all +-0 (that
 *   step's SCAL/GER are skipped, R4), or -1 if m_b is outside 0..32.
 * `plan` may be NULL (a transient plan is built on `stream`).
 * ------------------------------------------------------------------------- */
bj_status bj_getrf_vbatched(bj_batch *blocks, int32_t *pivots, int32_t *info,
                            const bj_plan *plan, bj_stream_t stream);

/* ---------------------------------------------------------------------------
 * Hot-path row a4 -- GETRS: x_b = D_b^{-1} b_b from the factors
 * steps 2-4, Fig. 2 bottom and the mirrored upper solve (R8):
 *   y = P b; eager unit-lower solve; eager upper solve with
 *   y_k /= U(k,k) (IEEE division); x = y.
 * b and x are packed at lu->vec_off; x may alias b exactly (not partially).
 * Blocks whose order is outside 0..32 are skipped (x untouched).
 * ------------------------------------------------------------------------- */
bj_status bj_getrs_vbatched(const bj_batch *lu, const int32_t *pivots, const void *b, void *x,
                            const bj_plan *plan, bj_stream_t stream);

/* ---------------------------------------------------------------------------
 * Rows a3 + a4 fused -- factor and solve in one pass (LAPACK gesv semantics):
 * exactly bj_getrf_vbatched(blocks, pivots, info) followed by
 * bj_getrs_vbatched(blocks, pivots, b, x) -- same outputs, bit for bit
 * (pivots, info, L\U in blocks->values, x) -- but each block is solved while
 * its factors are still in registers, so the factors are not read back from
 * memory (data kept in registers; the solve of P:218-238 follows
 * the factorization of the same block).  b and x are packed at
 * blocks->vec_off; x may alias b exactly.  Blocks with info != 0 get the
 * IEEE results of the division by the zero pivot (as bj_getrs_vbatched).
 * ------------------------------------------------------------------------- */
bj_status bj_gesv_vbatched(bj_batch *blocks, int32_t *pivots, int32_t *info, const void *b, void *x,
                           const bj_plan *plan, bj_stream_t stream);

/* ---------------------------------------------------------------------------
 * Hot-path row a5 -- block-Jacobi preconditioner, section II.A:
 * setup = extract + factor every diagonal block,
 * apply   y = D^{-1} x, one GETRS per block over the segments
 *         x[block_ptr[b] .. block_ptr[b+1]) ("once per step").
 * bj_setup fills factors->sizes/vec_off/val_off (caller buffers of nblocks /
 * nblocks+1 / nblocks+1 entries; factors->values must hold
 * val_off[nblocks] elements -- size it with bj_layout_from_block_ptr first),
 * extracts into factors->values, factors in place, and keeps references to
 * factors, pivots, block_ptr and a size plan in the handle.  x and y cover
 * the rows the blocks own, relative to the first block: x[i] and y[i] belong
 * to local row block_ptr[0] + i (i < block_ptr[nb] - block_ptr[0]; with the
 * usual block_ptr[0] = 0 they are indexed by local row).  y may alias x.
 * ------------------------------------------------------------------------- */
bj_status bj_create(bj_handle **handle);
bj_status bj_setup(bj_handle *handle, const bj_csr *A, const int32_t *block_ptr,
                   bj_batch *factors, int32_t *pivots, int32_t *info, bj_stream_t stream);
bj_status bj_apply(bj_handle *handle, const void *x, void *y, bj_stream_t stream);
bj_status bj_destroy(bj_handle *handle);

/* ---------------------------------------------------------------------------
 * NEXT(3) -- inversion-based block-Jacobi: "explicitly
 * compute the block-inverse before the iterative solution phase, and apply
 * the preconditioner as a matrix-vector multiplication".
 * bj_getri_vbatched: in place, blocks->values (packed per bj_layout) are
 *   replaced by the inverses, column-major, computed by Gauss-Jordan
 *   elimination with implicit partial pivoting (readings R23-R25 of DESIGN.md:
 *   the GETRF pivot rule on the working matrix, IEEE division, single-rounding
 *   FMA, unscaled pivot rows divided at the end).  pivots[vec_off[b] + k] =
 *   pivot row of step k, info as for GETRF (k+1 for the first zero pivot; the
 *   "inverse" of a singular block holds the IEEE results of the divisions by
 *   zero; -1 for an order outside 0..32, block untouched).
 * bj_gemv_vbatched: y_b = Dinv_b x_b per block (R26: fma chain over the
 *   columns in order, from +0); x, y packed at inv->vec_off; y may alias x.
 * bj_setup_inverse: like bj_setup with bj_getri_vbatched instead of GETRF;
 *   bj_apply on such a handle runs bj_gemv_vbatched.
 * ------------------------------------------------------------------------- */
bj_status bj_getri_vbatched(bj_batch *blocks, int32_t *pivots, int32_t *info,
                            const bj_plan *plan, bj_stream_t stream);
bj_status bj_gemv_vbatched(const bj_batch *inv, const void *x, void *y,
                           const bj_plan *plan, bj_stream_t stream);
bj_status bj_setup_inverse(bj_handle *handle, const bj_csr *A, const int32_t *block_ptr,
                           bj_batch *inverses, int32_t *pivots, int32_t *info, bj_stream_t stream);

/* ---------------------------------------------------------------------------
 * Hot-path row a6 -- contiguous cost-balanced batch partitioner (multi-GPU;
 * not in the paper, which is single-GPU P:648).  HOST function.
 *   cost_b = m_b^2, P(i) = sum_{b<i} cost_b (int64),
 *   bounds[0] = 0, bounds[G] = nblocks,
 *   bounds[r] = min{ i : G*P(i) >= r*P(nblocks) } for 0 < r < G   (R19).
 * Rank r owns blocks [bounds[r], bounds[r+1]).
 * ------------------------------------------------------------------------- */
bj_status bj_partition(int64_t nblocks, const int32_t *sizes_h, int G, int64_t *bounds_h);

/* ---------------------------------------------------------------------------
 * Next row NEXT(2) -- supervariable blocking (section II.A, P:186-193;
 * the experiments vary only the upper bound): the block
 * boundaries that bj_extract takes as input.
 *   A supervariable is a maximal run of consecutive rows whose column index
 *   sequences are identical as stored (R20); a supervariable longer than
 *   `max_block` is cut into max_block-row pieces plus a remainder (R22); the
 *   pieces are clustered greedily in row order into blocks of at most
 *   `max_block` rows (R21).  Only A->row_ptr / A->col_idx are read (values
 *   and dtype are ignored).
 *   block_ptr: DEVICE int32[A->nrows + 1] (capacity); receives nb+1 entries,
 *   block_ptr[0] = 0, block_ptr[nb] = nrows.  nblocks_h: HOST int64, receives
 *   nb.  max_block must lie in 1..32 and nrows in 0..2^31-2, else BJ_ERR_ARG.
 *   SYNCHRONOUS: returns after the stream work completes (nb is read back to
 *   the host; this is a once-per-sparsity-pattern analysis, not on the
 *   setup/apply path).
 * ------------------------------------------------------------------------- */
bj_status bj_supervariable_blocking(const bj_csr *A, int32_t max_block, int32_t *block_ptr,
                                    int64_t *nblocks_h, bj_stream_t stream);

/* ---------------------------------------------------------------------------
 * Test hook (not the hot path), SYNCHRONOUS: checks on the device that the
 * split IEEE divisions the kernels use for every quotient (R3) reproduce the
 * correctly rounded quotient (__ddiv_rn / __fdiv_rn) on n pseudo-random
 * operand pairs covering every exponent and the specials.  counts_h (HOST,
 * 6 entries): [0] full division mismatches, [1] mismatches of the flag-only
 * quotient where it claims validity, [2] its flagged count, [3] / [4] the
 * same for the normal-divisor variant, [5] pairs tested.  sample_h (HOST,
 * 3*nsample elements of dtype) receives (a, b, a/b) of the first pairs.
 * ------------------------------------------------------------------------- */
bj_status bj_selftest_div(bj_dtype dtype, int64_t n, uint64_t seed, uint64_t *counts_h, void *sample_h,
                          int64_t nsample);

/* ---------------------------------------------------------------------------
 * NEXT(4) -- block-Jacobi preconditioned Krylov solve, the paper's end-to-end
 * use of the preconditioner (section IV.D: right-hand side of all
 * ones, initial guess zero, stop once the relative residual norm has dropped
 * by six orders of magnitude, at most 10,000 iterations; the
 * preconditioner is applied "once per step of the iterative solve").  The
 * paper runs IDR(4); this build runs BiCGSTAB (reading R29).  fp64 only
 * (A->dtype must be BJ_F64).  Every reduction has a fixed order, so results
 * are reproducible bit for bit and equal to the oracle's:
 *
 * bj_spmv:  y = A x (R27).  Row i: lane l of a warp accumulates
 *   s_l = fma(val_e, x[col_e - col_offset], s_l) over the row's entries
 *   e = row_ptr[i] + l, + l + 32, ... in order, from +0; then
 *   s_l += s_(l^16), s_l += s_(l^8), ..., s_l += s_(l^1); y_i = s_0.
 *   x has at least max(col_idx) - col_offset + 1 elements; y (A->nrows) must
 *   not overlap x.
 * bj_dot:  *result (a DEVICE double) = dot(x, y) over n elements (R28): chunks
 *   of 8192 consecutive elements; thread t of 256 accumulates
 *   fma(x_k, y_k, s_t) over k = chunk + t + 256 j (j = 0..31) from +0; the
 *   256 partials are added by the tree s_t += s_(t+h), h = 128, ..., 1; the
 *   chunk sums are added in chunk order from +0.
 * bj_bicgstab: solves A x = b with right-preconditioned BiCGSTAB, M^-1 =
 *   bj_apply(M, .) (a handle set up by bj_setup or bj_setup_inverse on the
 *   same rows; the oracle pins the LU handle).  r = rh = b, p = v = 0, x = 0,
 *   rho_prev = alpha = omega = 1; per iteration
 *     rho = dot(rh, r); beta = (rho / rho_prev) * (alpha / omega);
 *     p = fma(beta, fma(-omega, v, p), r); ph = M^-1 p; v = A ph;
 *     alpha = rho / dot(rh, v); s = fma(-alpha, v, r); sh = M^-1 s; t = A sh;
 *     omega = dot(t, s) / dot(t, t); x = fma(omega, sh, fma(alpha, ph, x));
 *     r = fma(-omega, t, s); stop if sqrt(dot(r, r)) <= tol * sqrt(dot(b, b));
 *     rho_prev = rho.
 *   The loop runs on the device (scalars in device memory, no host round
 *   trip per iteration; the host polls a completion flag two iterations
 *   behind).  *iters_h (HOST) = the iteration that converged, or maxit + 1;
 *   *resid_h (HOST) = final ||r|| / ||b||.  x (A->nrows) is overwritten; b
 *   is read only.  Synchronous on return.  Scratch: 9 vectors of A->nrows
 *   (+ halo) doubles (cudaMallocAsync).
 *   comm = NULL: one GPU, A holds every column (col_offset as in bj_csr).
 *   comm != NULL (rows sharded over comm->nranks processes): A's col_idx are
 *   LOCAL EXTENDED ids from bj_halo_plan (own rows 0..nrows-1, then the halo)
 *   and A->col_offset must be 0.  Before each SpMV the library packs
 *   x[send_idx[j]] into comm->send_buf and calls halo_exchange(ctx, stream),
 *   which must deliver every peer's entries into comm->recv_buf in halo order
 *   (stream-ordered).  If halo_wait is not NULL the exchange may complete
 *   asynchronously: the library then computes the INTERIOR rows (no halo
 *   column) while it is in flight, calls halo_wait(ctx, stream) -- after
 *   which recv_buf must be complete in stream order -- and computes the
 *   boundary rows (each row's value is the same R27 result either way).
 *   For each dot the library writes its k <= 4 rank sums
 *   to gather_buf[rank*4 .. rank*4+k) and calls allgather(ctx, k, stream),
 *   which must fill every rank's row; the global value is the sum over ranks
 *   in rank order from +0 (reading R30; one rank reproduces R28 exactly).
 *   A callback returning nonzero aborts with BJ_ERR_COMM.
 * bj_halo_plan (HOST): for rows [lo, hi) of a matrix whose rows are sharded
 *   as row_bounds_h[0..G] (rank q owns [row_bounds_h[q], row_bounds_h[q+1])),
 *   maps the nnz global column ids col_idx_h to col_local_h: c - lo for an
 *   own column, (hi - lo) + j for the j-th distinct remote column in
 *   ascending order.  halo_cols_h (capacity nnz) receives those distinct
 *   remote columns in ascending order, *nhalo_h their count and
 *   recv_counts_h[q] (G entries) how many of them rank q owns (so the halo is
 *   grouped by owner, in rank order).  A column outside [0, row_bounds_h[G])
 *   is BJ_ERR_ARG.
 * ------------------------------------------------------------------------- */
typedef struct {
    void *ctx;
    int nranks;
    int rank;
    int64_t nhalo;              /* halo entries received (x extension length)   */
    int64_t nsend;              /* entries sent to peers                        */
    const int32_t *send_idx;    /* device [nsend]: own rows to send, by peer     */
    double *send_buf;           /* device [nsend], caller-owned                 */
    double *recv_buf;           /* device [nhalo], caller-owned                 */
    double *gather_buf;         /* device [nranks * 4], caller-owned            */
    int (*halo_exchange)(void *ctx, bj_stream_t stream);
    int (*allgather)(void *ctx, int k, bj_stream_t stream);
    int (*halo_wait)(void *ctx, bj_stream_t stream);   /* optional (NULL: exchange is stream-synchronous) */
} bj_comm;

bj_status bj_spmv(const bj_csr *A, const double *x, double *y, bj_stream_t stream);
bj_status bj_dot(int64_t n, const double *x, const double *y, double *result, bj_stream_t stream);
bj_status bj_bicgstab(bj_handle *M, const bj_csr *A, const bj_comm *comm, const double *b, double *x,
                      double tol, int maxit, int *iters_h, double *resid_h, bj_stream_t stream);
bj_status bj_halo_plan(int64_t nnz, const int32_t *col_idx_h, int64_t lo, int64_t hi, int G,
                       const int64_t *row_bounds_h, int32_t *col_local_h, int32_t *halo_cols_h,
                       int64_t *nhalo_h, int64_t *recv_counts_h);

/* ---------------------------------------------------------------------------
 * End-to-end call with HOST buffers (synchronous): copies sizes_h (nblocks),
 * blocks_h (nvalues elements, packed per bj_layout) and b_h (nvec elements)
 * to the device, runs layout + plan + GETRF + GETRS, and copies x_h (nvec),
 * pivots_h (nvec, may be NULL)
 * and info_h (nblocks, may be NULL) back.  nvalues / nvec smaller than the
 * layout of sizes_h requires (sum of round_up(m^2, 16/s) / sum of m) is
 * BJ_ERR_ARG (checked on the host before any copy).
 * Large batches (>= 131,072 blocks) run as up to 4 contiguous chunks in a
 * pipeline: host-to-device copies (one copy stream), compute (`stream`) and
 * device-to-host copies (a second copy stream) of different chunks overlap;
 * results are identical to the unchunked call (the blocks are independent).
 * Device buffers live in `ws` and grow on demand.  Host buffers should be
 * pinned (cudaHostAlloc / torch pin_memory) for full PCIe bandwidth and for
 * the copies to overlap.
 * ------------------------------------------------------------------------- */
bj_status bj_workspace_create(bj_workspace **ws);
bj_status bj_workspace_destroy(bj_workspace *ws);
bj_status bj_gesv_host(bj_workspace *ws, int64_t nblocks, const int32_t *sizes_h,
                       int64_t nvalues, const void *blocks_h, int64_t nvec, const void *b_h,
                       void *x_h, int32_t *pivots_h, int32_t *info_h, bj_dtype dtype,
                       bj_stream_t stream);

/* Kernel launches issued by this library on the calling thread since the
 * last reset (for the bench's gpu_launches count). */
int64_t bj_launch_count(void);
void bj_launch_count_reset(void);

#ifdef __cplusplus
}
#endif
#endif /* BJ_H */
