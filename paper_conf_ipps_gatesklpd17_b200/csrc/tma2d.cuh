// tma2d.cuh -- 2-D tensor TMA over the (chunked-)interleaved array (round 2).
// The array is viewed as rows x C floats: row = element (i, j) of one chunk of
// C consecutive matrices, C*4 bytes apart (C = batch for simple interleaved).
// A box of 32 matrices x H rows lands in shared memory as [H][32] -- the stage
// layout of the kernels that otherwise use one cp.async.bulk per column run at
// chunk 32 (RCWP, PTMEM).  One tensor map per box height; maps travel as
// __grid_constant__ kernel parameters.
#pragma once

#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdlib.h>

#include "ptx.cuh"

namespace bsp {

__device__ __forceinline__ void tma_load_2d(void *dst, const CUtensorMap *map, int x, int y, uint64_t *bar) {
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];" ::"r"(
            smem_u32(dst)),
        "l"(reinterpret_cast<uint64_t>(map)), "r"(x), "r"(y), "r"(smem_u32(bar))
        : "memory");
}

// cuTensorMapEncodeTiled through the runtime's driver entry point (no libcuda
// link dependency); resolved once.
inline PFN_cuTensorMapEncodeTiled_v12000 tma2d_encode_fn() {
    static PFN_cuTensorMapEncodeTiled_v12000 fn = []() -> PFN_cuTensorMapEncodeTiled_v12000 {
        void *p = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) != cudaSuccess ||
            q != cudaDriverEntryPointSuccess)
            return nullptr;
        return reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(p);
    }();
    return fn;
}

// Map of the interleaved array of n x n matrices (E = n*n rows per chunk) with
// chunk stride C and box 32 x H.  False if the layout does not qualify for TMA
// (C % 4 != 0: row stride not a multiple of 16 B; C < 32: box wider than the
// row; coordinates beyond int32) -- callers fall back to per-thread copies.
inline bool tma2d_make_map(CUtensorMap *m, const float *A, int64_t batch, int64_t C, int E, int H) {
    if (C % 4 != 0 || C < 32 || H < 1 || H > 256) return false;
    if (const char *ev = getenv("BSPOTRF_TMA2D"); ev && ev[0] == '0') return false;   // A/B probes
    const int64_t rows = (batch + C - 1) / C * (int64_t)E;
    if (rows >= ((int64_t)1 << 31) || C >= ((int64_t)1 << 31)) return false;
    auto enc = tma2d_encode_fn();
    if (enc == nullptr) return false;
    const cuuint64_t dims[2] = {(cuuint64_t)C, (cuuint64_t)rows};
    const cuuint64_t strides[1] = {(cuuint64_t)C * 4};
    const cuuint32_t box[2] = {32u, (cuuint32_t)H};
    const cuuint32_t estr[2] = {1u, 1u};
    return enc(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, const_cast<float *>(A), dims, strides, box, estr,
               CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
               CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

}  // namespace bsp
