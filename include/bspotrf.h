/*
 * bspotrf.h -- B200 (sm_100a) batched single-precision Cholesky factorization
 * (SPOTRF, lower, in place) of very many tiny SPD matrices stored in the
 * interleaved / chunked-interleaved layout of
 *   Gates, Kurzak, Luszczek, Pei, Dongarra, "Autotuning Batch Cholesky
 *   Factorization in CUDA with Interleaved Layout of Matrices", IPDPS-W 2017
 *   (cited below as PAPER.md:<line>, the text of that paper).
 *
 * C ABI: plain pointers and sizes, no C++ or torch types.  Link with
 * libbspotrf.so.  All "device pointers" are CUDA global-memory pointers owned
 * by the caller; "stream" is a cudaStream_t (0 = legacy default stream).
 *
 * ----------------------------------------------------------------------------
 * LAYOUT (Sec. II.B, Figs. 7-8; address formula from Fig. 10,
 * PAPER.md:222-231; readings R6/R7 in DESIGN.md)
 *   Every matrix is stored full n x n, column-major (lda = n); only the lower
 *   triangle (i >= j) is read or written.  With chunk size C (C = batch when
 *   chunk == 0, "simple interleaved", Fig. 7; otherwise C = chunk, a multiple
 *   of 32, "chunked interleaved", Fig. 8), element (i, j) of matrix b is the
 *   float at
 *        A[(b / C) * C * n*n + (i + j*n) * C + (b % C)].
 *   Storage holds ceil(batch/C)*C matrices (batch_interleaved_elems); the pad
 *   lanes of the last chunk are never read as data and never written.
 *
 * ERRORS (LAPACK xerbla style): return 0 on success; -i if argument i is
 * illegal (nothing is enqueued); a positive value is a cudaError_t from the
 * launch.  No exceptions, no exit(), no printing.  Calls only ENQUEUE work on
 * `stream` (except batch_spotrf_interleaved_host, which is blocking); read
 * results after synchronising the stream.  No hidden allocation except in
 * batch_spotrf_interleaved_host, which takes its slab buffers from a
 * library-owned cudaMemPool per device (created on first use, kept for reuse;
 * the process's default pool is not touched).  Thread-safe and reentrant.
 *
 * TENSOR MEMORY.  Variants PTMEM, QTM, RCW and RCW16 (the table's choice for
 * 24 <= n <= 64 at most chunks) allocate Tensor Memory per CTA with
 * tcgen05.alloc and release it before the CTA exits; their shared-memory
 * footprint caps the library's own demand at 512 columns per SM, so any number
 * of concurrent launches of this library (any streams) make progress.
 * tcgen05.alloc WAITS while the columns are held: a kernel from elsewhere that
 * holds Tensor Memory on the same SM for an unbounded time (e.g. a persistent
 * kernel that never relinquishes it) would stall these variants until it
 * exits.  Such a process should select a non-TMEM variant explicitly through
 * batch_spotrf_interleaved_ex (REG, SMEM, PANEL or TILE).
 * ----------------------------------------------------------------------------
 */
#ifndef BSPOTRF_H
#define BSPOTRF_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct CUstream_st *bspotrf_stream_t; /* == cudaStream_t */

#define BSPOTRF_MAX_N 64

/* Kernel variants.  All right-looking-order variants
 * perform the same per-element FP32 operation sequence (sqrt.rn, rcp.rn,
 * mul.rn, fma.rn in k order), so their outputs are bitwise identical. */
enum {
    BSPOTRF_VARIANT_AUTO = 0, /* tuning table                                  */
    BSPOTRF_VARIANT_REG = 1,  /* whole lower triangle in registers, n <= 24    */
    BSPOTRF_VARIANT_SMEM = 2, /* left panel of `param` columns staged in shared
                                 memory (TMA bulk or cp.async), trailing
                                 triangle in registers; 2 <= n <= 32           */
    BSPOTRF_VARIANT_TILE = 3, /* paper's top-looking tile algorithm (Figs. 9-11)
                                 with param x param register tiles, tiles
                                 streamed from global memory; any n <= 64      */
    BSPOTRF_VARIANT_PANEL = 4, /* SMEM split with compact code: the panel of
                                 `param` columns (multiple of 4) factored by a
                                 rolled 4x4-tile loop in shared memory, rolled
                                 SYRK, unrolled register tail; 20 <= n <= 32   */
    BSPOTRF_VARIANT_PTMEM = 5, /* PANEL with the first panel tile columns held in
                                 Tensor Memory (tcgen05.ld/st), 128-thread
                                 CTAs with 256 TMEM columns each (two per SM;
                                 512, one per SM, for n > 32); staging 1 =
                                 TMA (chunk 32), TMEM fill in batches of 5
                                 tiles; 3 = TMA, batches of 12 (n <= 32);
                                 2 = per-thread cp.async; 24 <= n <= 44       */
    BSPOTRF_VARIANT_RTMA = 6, /* REG with TMA bulk copies in and out of a
                                 shared-memory image (chunk 32 only); `param`
                                 warps per CTA (2 or 4); 4 <= n <= 20         */
    BSPOTRF_VARIANT_RTMAP = 7, /* persistent RTMA: each warp loops over chunks,
                                 the next chunk's TMA load overlapping this
                                 chunk's arithmetic; per-thread stores; grid =
                                 resident warps; chunk 32; 4 <= n <= 20       */
    BSPOTRF_VARIANT_QTM = 8,  /* `param` (4 or 8) threads per matrix, each
                                 owning tile rows; the whole matrix on chip
                                 (off-diagonal 4x4 tiles in Tensor Memory and
                                 shared memory), left-looking; staging 1 =
                                 256 TMEM columns per CTA (two CTAs per SM),
                                 0/2 = 512 (one), input streamed by cp.async;
                                 3/4 = the same with the input preloaded;
                                 any chunk; 33 <= n <= 64                     */
    BSPOTRF_VARIANT_REGX = 9, /* REG with the extra sweep axes: `param` (1, 2,
                                 4) matrices per thread; staging 1 = fast-math
                                 sqrt/rcp (sqrt.approx, rcp.approx, ftz;
                                 tolerance-checked, not bitwise reproducible,
                                 never chosen by the default table), 0 = IEEE;
                                 <= 128 threads per block; 1 <= n <= 16       */
    BSPOTRF_VARIANT_RCW = 10, /* row-cyclic warps: 8 warps share 32 matrices
                                 (lane = matrix), warp h owns rows 8r+h, the
                                 factor in Tensor Memory, left-looking over
                                 8-wide column blocks; `param` = CTAs per SM
                                 (1: 512 TMEM columns, any n; 2: 256 each,
                                 n <= 48); any chunk; 33 <= n <= 64           */
    BSPOTRF_VARIANT_REGV = 11, /* REG with 128-bit accesses: each thread owns 4
                                 adjacent matrices (one float4 per element);
                                 needs C % 4 == 0 (C = chunk, or batch when
                                 chunk == 0), else runs REG (same bits);
                                 <= 128 threads per block; 1 <= n <= 8        */
    BSPOTRF_VARIANT_RCW16 = 12,/* RCW with 16 warps per 32 matrices (rows
                                 16r+h), one CTA per SM; faster than RCW where
                                 the input comes by per-thread copies (chunk
                                 != 32), slower with chunk 32 (TMA path);
                                 any chunk; 49 <= n <= 64                     */
    BSPOTRF_VARIANT_RCWD = 13, /* RCW plus a ninth warp that factors each 8x8
                                 diagonal block while the row warps run the
                                 GEMM of their other rows (two passes over the
                                 row buffer); one CTA per SM; any chunk;
                                 49 <= n <= 64                                */
    BSPOTRF_VARIANT_RCWP = 14  /* "paged" RCW: the factor in 8-column TMEM
                                 pages recycled as row slots die (at most 128
                                 columns per warp), one row buffer + stage set
                                 in shared memory, TWO CTAs per SM (256 TMEM
                                 columns each); `param` 1 = the 8x8 diagonal
                                 block factored by one warp (0: by all eight,
                                 as RCW); any chunk; 33 <= n <= 64            */
};

/* Launch tuning (a row of the autotuning table). */
typedef struct {
    int variant;           /* BSPOTRF_VARIANT_*                                */
    int threads_per_block; /* multiple of 32, 32..1024; 0 = variant default.
                              SMEM variant with TMA staging uses one chunk per
                              block and ignores this.                         */
    int param;             /* SMEM/PANEL: panel width s; TILE: tile size nb;
                              REG: min resident warps per SM requested from
                              the compiler (0 = none; 12, 16 for some n;
                              forces 128 threads per block)                  */
    int staging;           /* SMEM/PANEL: 0 = auto, 1 = TMA bulk copy
                              (cp.async.bulk, needs chunk in {32,64,128}),
                              2 = per-thread cp.async                         */
    int carveout;          /* preferred shared-memory carveout of the SM's
                              unified L1/shared capacity, in percent (1..100;
                              0 = driver default) -- Table I's "L1 or shared"
                              parameter.  Applied to the
                              kernel on every launch; the driver rounds it to a
                              supported split and never grants less shared
                              memory than the launch needs (a small carveout
                              can lower the resident CTAs per SM).  Values
                              outside 0..100 are rejected (-7).               */
} bspotrf_tuning;

/* 1 if the library holds a kernel instance for this explicit tuning at (n,
 * chunk) -- i.e. batch_spotrf_interleaved_ex would not return -7 for want of
 * an instance -- else 0; -1 n, -2 chunk invalid, -3 tune null.  The default
 * build holds every instance the tuning table reaches plus a representative
 * subset of the sweep space; BSPOTRF_SWEEP=1 at build time holds all of it
 * (scripts/gen_instances.py).  No GPU work. */
int bspotrf_tuning_available(int n, int chunk, const bspotrf_tuning *tune);

/* Library version (major*10000 + minor*100 + patch). */
int bspotrf_version(void);

/* Number of floats the interleaved storage of `batch` n x n matrices with
 * chunk size `chunk` occupies: ceil(batch/C)*C*n*n (C = batch if chunk == 0).
 * Returns 0 if n == 0 or batch == 0, -1 on illegal arguments. */
int64_t batch_interleaved_elems(int n, int64_t batch, int chunk);

/* Batched SPOTRF, lower, in place (Alg. 1; Fig. 9 op order).
 *   n      1..64 (0 -> quick return)                                  arg 1
 *   batch  >= 0 (0 -> quick return)                                   arg 2
 *   chunk  0 (simple interleaved) or a positive multiple of 32        arg 3
 *   A      device, batch_interleaved_elems(n,batch,chunk) floats,
 *          16-byte aligned; on return the lower triangle of every
 *          matrix holds L with A = L L^T; the strict upper triangle
 *          and pad lanes are untouched                                arg 4
 *   info   device int32[batch]: 0 = success, k > 0 = the leading
 *          minor of order k is not positive definite (pivot !(>0),
 *          NaN included; LAPACK convention, reading R1).  Columns
 *          j < k-1 of a failed matrix are final; the rest is
 *          unspecified (R2)                                           arg 5
 *   stream                                                            arg 6
 * Errors: -1 n, -2 batch, -3 chunk, -4 A null/misaligned, -5 info null. */
int batch_spotrf_interleaved(int n, int64_t batch, int chunk, float *A,
                             int32_t *info, bspotrf_stream_t stream);

/* Runtime chunks (any chunk but 32, including 0) whose stride is a multiple of
 * 16 B stage some kernels' column runs by 2-D tensor TMA (RCWP n <= 51, PTMEM
 * n = 32..38); the environment variable BSPOTRF_TMA2D=0, read per
 * call, selects the per-thread cp.async staging instead (an A/B probe; the
 * results are bitwise the same, tested). */

/* As above, plus:
 *   nfailed  device int32* or NULL: atomically INCREMENTED by the number of
 *            matrices with info != 0 (the caller zeroes it) -- fused into the
 *            factorization kernel (warp ballot + popc + one atomic per warp)
 *   tune     NULL = tuning table; otherwise an explicit launch tuning
 *            (-7 if the requested variant/param/staging is not available
 *            for this n and chunk). */
int batch_spotrf_interleaved_ex(int n, int64_t batch, int chunk, float *A,
                                int32_t *info, int32_t *nfailed,
                                const bspotrf_tuning *tune,
                                bspotrf_stream_t stream);

/* The tuning the table selects for (n, chunk) (chunk as in the factor call).
 * Returns 0 and fills *out, or -1/-3 on an illegal n/chunk. */
int bspotrf_get_tuning(int n, int chunk, bspotrf_tuning *out);

/* Layout conversion, out of place, bit-exact (a pure permutation):
 * canonical = batch consecutive n x n column-major matrices,
 * batch*n*n floats; interleaved as above.  src and dst must not overlap.
 * Pad lanes of the interleaved side are never read or written.  The kernel
 * is chosen per direction and n class (v1 / v2 / v3 / v4); the
 * environment variable BSPOTRF_CONVERT_PATH=v2|v3|v4, read per call, forces
 * one where it applies (an A/B probe for the benchmarks; every path produces
 * the same bits, tested).
 * Errors: -1 n, -2 batch, -3 chunk, -4 src null, -5 dst null or overlapping. */
int batch_canonical_to_interleaved(int n, int64_t batch, int chunk,
                                   const float *src_canonical,
                                   float *dst_interleaved,
                                   bspotrf_stream_t stream);
int batch_interleaved_to_canonical(int n, int64_t batch, int chunk,
                                   const float *src_interleaved,
                                   float *dst_canonical,
                                   bspotrf_stream_t stream);

/* ---- Canonical storage, conversion fused (round 2) -----
 * The factorization on CANONICAL storage: A = batch consecutive n x n
 * column-major matrices (lda = n), factored in place, lower,
 * with the layout conversion fused into the kernel's loads and stores instead
 * of canonical -> interleaved -> factor -> canonical (3 launches, 2 x 8n^2
 * extra bytes per matrix).  A warp owns 32 consecutive matrices: each lane
 * cp.asyncs its own lower triangle into a shared image (the 32 sectors of an
 * instruction are re-hit in L1 by the next copies of the same column), the
 * factorization is REG's (same per-element FP32 op sequence as every
 * interleaved variant: bitwise the same L and info), and each final column is
 * stored with a flat mapping (a warp store = 32 consecutive run elements).
 *   n        1..BSPOTRF_CANON_MAX_N (20); n = 0 or batch = 0: quick return 0
 *   A        device float*, batch*n*n floats, 4-B aligned; only lower-triangle
 *            elements are read and written
 *   info     device int32[batch], LAPACK convention (as the interleaved call)
 *   nfailed  device int32* or NULL, incremented by the failure count
 * Errors: -1 n, -2 batch, -3 A null/misaligned, -4 info null; positive =
 * CUDA error.  Larger n: batch_canonical_to_interleaved + the interleaved
 * call + batch_interleaved_to_canonical. */
#define BSPOTRF_CANON_MAX_N 20
int batch_spotrf_canonical(int n, int64_t batch, float *A, int32_t *info,
                           int32_t *nfailed, bspotrf_stream_t stream);

/* End-to-end call on HOST buffers (blocking).  hA is the interleaved storage
 * in host memory, hinfo host int32[batch], nfailed_out host int32* or NULL
 * (set, not incremented).  Only the lower triangles cross PCIe.
 *   slab == 0 and hA, hinfo pinned (page-locked and mapped, e.g.
 *     cudaHostAlloc / torch pin_memory): ZERO-COPY -- the factorization kernel
 *     reads and writes the host storage directly over PCIe, one 128-B line per
 *     warp access, both directions at once;
 *   otherwise: COPY PIPELINE -- slabs of `slab` matrices (rounded to whole
 *     chunks; 0 = auto, ~32 MB) flow over three streams (H2D / factor / D2H)
 *     through device workspace from the stream-ordered allocator; per slab,
 *     one cudaMemcpy2DAsync per column moves that column's lower runs of every
 *     chunk (pitch n*n*C); a partial last chunk is copied lane-exactly.
 * `stream` orders the call after prior work.
 * Errors as batch_spotrf_interleaved, plus -6 slab < 0; positive = CUDA error. */
int batch_spotrf_interleaved_host(int n, int64_t batch, int chunk, float *hA,
                                  int32_t *hinfo, int32_t *nfailed_out,
                                  int64_t slab, bspotrf_stream_t stream);

/* ---- Solves -------------------------------------------
 * "A symmetric positive definite system of linear equations Ax = b can be
 * solved by computing the Cholesky factorization A = LL^T, and then applying
 * forward substitution and backward substitution to the vector b using the
 * factors L and L^T".  Right-hand sides B are n x nrhs per
 * matrix, column-major, interleaved with the SAME chunk as the matrices:
 * element (i, r) of matrix b's block at (b/C)*C*n*nrhs + (i + r*n)*C + b%C.
 * One thread per matrix; FP32 with fma accumulation and reciprocal scaling
 * (the factorization's conventions). */

/* Floats of the interleaved right-hand-side storage: ceil(batch/C)*C*n*nrhs
 * (0 for an empty problem, -1 on illegal arguments). */
int64_t batch_interleaved_rhs_elems(int n, int nrhs, int64_t batch, int chunk);

/* Batched SPOTRS: B := A^-1 B using the factor L written by
 * batch_spotrf_interleaved (device, read only).  B device, overwritten by X.
 * Matrices must have factored successfully (info == 0); others produce
 * undefined X.  Right-hand sides are processed 4/2/1 at a time (L is re-read
 * per group).  Errors: -1 n, -2 nrhs, -3 batch, -4 chunk, -5 L, -6 B;
 * -7 no kernel instance (n * group > 128 for every group size). */
int batch_spotrs_interleaved(int n, int nrhs, int64_t batch, int chunk,
                             const float *L, float *B, bspotrf_stream_t stream);

/* Batched SPOSV: factor A in place (as batch_spotrf_interleaved_ex) and solve
 * A X = B.  Fused (one kernel, L never re-read) for n <= 20 and nrhs <= 4 (L in
 * registers) and for 24 <= n <= 44 with nrhs == 1 (L in registers + shared
 * memory + Tensor Memory, the PTMEM structure); otherwise factor then
 * SPOTRS.  X is bitwise identical either way.  LAPACK
 * semantics: a matrix with info > 0 keeps its right-hand sides unchanged.
 * nfailed as in _ex.  Errors: -1 n, -2 nrhs, -3 batch, -4 chunk, -5 A,
 * -6 B, -7 info. */
int batch_sposv_interleaved(int n, int nrhs, int64_t batch, int chunk,
                            float *A, float *B, int32_t *info, int32_t *nfailed,
                            bspotrf_stream_t stream);

/* Bytes of A the host call moves each way (lower triangles only). */
int64_t batch_spotrf_host_bytes(int n, int64_t batch, int chunk);

#ifdef __cplusplus
}
#endif
#endif /* BSPOTRF_H */
