/*
 * bspotrf_synth.h -- on-device seeded synthetic SPD batches (bench and test
 * utility; not part of the factorization).
 *
 * Implements, independently of the host module synth/__init__.py, the same
 * counter-based generator: splitmix64 finaliser
 *   mix64(z), h(seed, b, e) = mix64(mix64(seed*G + b) ^ (e*K1 + K2)),
 * b = GLOBAL matrix index, so every partition of a batch over GPUs produces
 * the same matrices, and the host can regenerate any matrix bit for bit.
 * Kinds: 0 = dd (diagonally dominant), 1 = als (regularised Gram, the ALS
 * workload of PAPER.md:22-24), 2 = l0 (A = L0 L0^T, integer L0).
 * Failure injection: matrices with h(fail_seed, b, E_FAIL) % fail_period == 0
 * get one pivot forced negative (fail_period 0 = none).
 */
#ifndef BSPOTRF_SYNTH_H
#define BSPOTRF_SYNTH_H

#include <stdint.h>
#include "bspotrf.h"

#ifdef __cplusplus
extern "C" {
#endif

enum { BSPOTRF_SYNTH_DD = 0, BSPOTRF_SYNTH_ALS = 1, BSPOTRF_SYNTH_L0 = 2 };
enum {
    BSPOTRF_UPPER_MIRROR = 0, /* write a_ji = a_ij                          */
    BSPOTRF_UPPER_NAN = 1,    /* write the sentinel NaN 0x7FC0FFEE          */
    BSPOTRF_UPPER_KEEP = 2    /* do not write the strict upper triangle     */
};

/* Fill the interleaved storage A (device; layout as bspotrf.h) with matrices
 * b0 .. b0+batch-1 of the global sequence.  Pad lanes are not written.
 * Errors: -1 n, -2 batch, -3 chunk, -4 A, -5 kind, -6 upper; >0 CUDA error. */
int bspotrf_synth_generate(int n, int64_t batch, int chunk, int64_t b0,
                           int kind, uint64_t seed, int upper_mode,
                           uint64_t fail_seed, int64_t fail_period, float *A,
                           bspotrf_stream_t stream);

/* Write `value_bits` into every float of A[0..elems) (sentinel fills). */
int bspotrf_fill_u32(float *A, int64_t elems, uint32_t value_bits,
                     bspotrf_stream_t stream);

/* Diagnostic "null factorization" (chunk 32 layout only): every thread loads
 * its matrix's lower triangle exactly as the REG kernel does and stores it
 * back unchanged, writing info = 0 -- the factorization's memory traffic with
 * no arithmetic.  n in {4, 8, 16, 20}; tpb multiple of 32 in 32..256.
 * Errors: -1 n, -2 batch, -3 A/info null, -5 tpb; >0 CUDA error. */
int bspotrf_probe_copy_lower(int n, int64_t batch, float *A, int32_t *info,
                             int tpb, bspotrf_stream_t stream);

#ifdef __cplusplus
}
#endif
#endif /* BSPOTRF_SYNTH_H */
