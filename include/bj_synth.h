/*
 * bj_synth.h -- device-side seeded input generators (bench / test inputs).
 *
 * Not part of the method: these calls only draw random numbers and build
 * input structures.  They implement the same counter-based generator as the
 * host module bj_synth/ (splitmix64: the i-th output of the stream keyed by
 * `seed` is mix64(seedkey(seed) + (i+1)*0x9E3779B97F4A7C15)), so any shard or
 * subset regenerates bit-identical data on host and device.  Recipe and keys:
 * DESIGN.md section 5.  All pointers are device pointers; asynchronous.
 */
#ifndef BJ_SYNTH_H
#define BJ_SYNTH_H

#include "bj.h"

#ifdef __cplusplus
extern "C" {
#endif

/* sizes[i] = lo + ((h(seed, first+i) >> 32) * (hi-lo+1) >> 32) */
bj_status bj_synth_sizes(int64_t nblocks, int64_t first, int lo, int hi, uint64_t seed,
                         int32_t *sizes, bj_stream_t stream);

/* Block b (global id first+b) element (r,c) = U[-1,1) draw of key
 * (first+b)*1024 + c*32 + r (kind 0, seed 2) or U{-3..3} (kind 1, seed 7);
 * fp32 = the fp64 draw rounded to nearest.  Pad elements are set to 0. */
bj_status bj_synth_blocks(const bj_batch *batch, int64_t first, int kind, bj_stream_t stream);

/* b (packed at vec_off) element r of block first+b = U[-1,1) draw of key
 * (first+b)*32 + r, seed 3. */
bj_status bj_synth_rhs(const bj_batch *batch, int64_t first, void *b, bj_stream_t stream);

/* FEM-like 27-point x 3-dof CSR on an nx*ny*nz node grid, rows [r0, r1) of
 * the global matrix (global column ids).  Step 1: row_ptr (r1-r0+1 entries,
 * row_ptr[0] = 0; device scan).  Step 2: col_idx / values (row_ptr[r1-r0]
 * entries).  skew = 0 disables the hub rows. */
bj_status bj_synth_fem_row_ptr(int nx, int ny, int nz, int skew, int64_t r0, int64_t r1,
                               int64_t *row_ptr, bj_stream_t stream);
bj_status bj_synth_fem_fill(int nx, int ny, int nz, int skew, int64_t r0, int64_t r1,
                            const int64_t *row_ptr, int32_t *col_idx, void *values,
                            bj_dtype dtype, bj_stream_t stream);

#ifdef __cplusplus
}
#endif
#endif /* BJ_SYNTH_H */
