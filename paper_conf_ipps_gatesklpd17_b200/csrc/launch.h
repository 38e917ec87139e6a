// launch.h -- host-side launcher declarations shared by the C ABI (api.cu)
// and the per-instance compilation units (gen/inst_*.cu).
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

namespace bsp {

struct FactorArgs {
    float *A;
    int32_t *info;
    int32_t *nfailed;    // may be null
    int64_t batch;
    int64_t cstride;     // effective chunk C (== batch for simple interleaved)
    int tpb;             // threads per block (multiple of 32)
    cudaStream_t stream;
    int carveout = 0;    // preferred shared-memory carveout, percent (0 = driver default)
};

// Table I's "L1 or shared" axis (Sec. II.D): the
// preferred split of the SM's unified L1 / shared-memory capacity, in percent
// of the maximum shared memory, set on every launch (the attribute is per
// function and persists, so a default launch must undo a tuned one).  0 is the
// driver default (-1 to CUDA); the driver rounds to a supported configuration
// and always grants at least what the launch needs.
template <typename K>
inline cudaError_t apply_carveout(K kern, int pct) {
    return cudaFuncSetAttribute(reinterpret_cast<const void *>(kern),
                                cudaFuncAttributePreferredSharedMemoryCarveout,
                                pct <= 0 ? -1 : (pct > 100 ? 100 : pct));
}

using LaunchFn = cudaError_t (*)(const FactorArgs &);

// Variant REG: lower triangle in registers (csrc/potrf_reg.cuh); MINW = the
// minimum resident warps per SM requested from ptxas (0 = no register cap).
template <int N, int CT, int MINW>
cudaError_t launch_reg(const FactorArgs &a);

// Variant SMEM: left panel of S columns in shared memory, trailing triangle in
// registers (csrc/potrf_smem.cuh).  TMA: stage with cp.async.bulk (one chunk of
// CT matrices per block); otherwise per-thread cp.async, per-warp staging.
template <int N, int CT, int S, bool TMA>
cudaError_t launch_smem(const FactorArgs &a);

// Variant PANEL: SMEM split with a rolled tile loop for the panel
// (csrc/potrf_panel.cuh).
template <int N, int CT, int S, bool TMA>
cudaError_t launch_panel(const FactorArgs &a);

// Variant PTMEM: PANEL with the first panel tile columns in Tensor Memory
// (csrc/potrf_tmem.cuh); 4-warp CTAs, 256 TMEM columns each.
template <int N, int CT, int S, bool TMA, int FILL = 0>
cudaError_t launch_ptmem(const FactorArgs &a);

// Variant RTMA: REG with TMA bulk staging in and out (chunk 32 only), W warps
// per CTA (csrc/potrf_regtma.cuh).
template <int N, int W>
cudaError_t launch_regtma(const FactorArgs &a);

// Variant RTMAP: persistent RTMA, next chunk's TMA load overlapping this
// chunk's arithmetic (csrc/potrf_regtma.cuh).
template <int N, int W>
cudaError_t launch_rtmap(const FactorArgs &a);

// Variant REGX: REG with M matrices per thread and optional fast-math sqrt/rcp
// (csrc/potrf_reg.cuh).
template <int N, int M, bool FAST>
cudaError_t launch_regx(const FactorArgs &a);

// Variant QTM: P threads per matrix, the whole matrix on chip (TMEM + shared
// memory), COLS TMEM columns per 128-thread CTA, input streamed (PRE = false)
// or preloaded (csrc/potrf_qtm.cuh).
template <int N, int CT, int P, int COLS, bool PRE>
cudaError_t launch_qtm(const FactorArgs &a);

// Variant RCW: 8 warps share 32 matrices (lane = matrix, warp h owns rows
// 8r+h), factor in TMEM, NCTA CTAs per SM (csrc/potrf_rcw.cuh).
template <int N, int CT, int NCTA>
cudaError_t launch_rcw(const FactorArgs &a);

// Variant REGV: REG with four adjacent matrices per thread and 128-bit
// accesses (csrc/potrf_regv.cuh); falls back to REG when C % 4 != 0.
template <int N>
cudaError_t launch_regv(const FactorArgs &a);

// Variant RCW16: RCW with 16 warps per 32 matrices (rows 16r+h), one CTA per SM
// (csrc/potrf_rcw16.cuh).
template <int N, int CT>
cudaError_t launch_rcw16(const FactorArgs &a);

// Variant RCWD: RCW with a diagonal-factorization warp (csrc/potrf_rcwd.cuh).
template <int N, int CT>
cudaError_t launch_rcwd(const FactorArgs &a);

// Variant RCWP: RCW with the factor in recycled TMEM pages, two CTAs per SM
// (csrc/potrf_rcwp.cuh); D1: the diagonal block factored by one warp.
template <int N, int CT, int P>
cudaError_t launch_rcwp(const FactorArgs &a);

// Variant TILE: the paper's top-looking tile algorithm, NB x NB register
// tiles streamed from global memory, runtime chunk stride (csrc/potrf_tile.cuh).
template <int N, int NB>
cudaError_t launch_tile(const FactorArgs &a);

// Solves (csrc/potrs.cuh).
struct SolveArgs {
    float *A;       // factor L (spotrs, read) or matrix A (sposv, factored in place)
    float *B;       // right-hand sides -> solutions
    int32_t *info;  // sposv only (potrs: nullable "skip failed matrices" mask)
    int32_t *nfailed;
    int64_t batch;
    int64_t cstride;
    int nrhs;
    cudaStream_t stream;
};
using PotrsFn = cudaError_t (*)(const SolveArgs &, int rhs0);
using SposvFn = cudaError_t (*)(const SolveArgs &);
template <int N, int NR, int CT>
cudaError_t launch_potrs(const SolveArgs &a, int rhs0);
template <int N, int NR, int CT>
cudaError_t launch_sposv(const SolveArgs &a);
template <int N, int CT, int S, bool TMA>
cudaError_t launch_sposv_ptmem(const SolveArgs &a);

// Grid size for one-thread-per-matrix kernels.
inline unsigned grid_for(int64_t batch, int tpb) {
    return (unsigned)((batch + tpb - 1) / tpb);
}

}  // namespace bsp
