// canon.cu -- batch_spotrf_canonical: the factorization on canonical storage
// with the layout conversion fused into its loads and stores (variant CANON,
// potrf_canon.cuh), n = 1..BSPOTRF_CANON_MAX_N.
#include "bspotrf.h"
#include "potrf_canon.cuh"

namespace bsp {

static cudaError_t launch_canon_n(int n, float *A, int32_t *info, int32_t *nfailed, int64_t batch,
                                  cudaStream_t s) {
    switch (n) {
#define BSP_CANON(NN) \
    case NN:          \
        return launch_canon<NN>(A, info, nfailed, batch, s);
        BSP_CANON(1) BSP_CANON(2) BSP_CANON(3) BSP_CANON(4) BSP_CANON(5) BSP_CANON(6) BSP_CANON(7)
        BSP_CANON(8) BSP_CANON(9) BSP_CANON(10) BSP_CANON(11) BSP_CANON(12) BSP_CANON(13) BSP_CANON(14)
        BSP_CANON(15) BSP_CANON(16) BSP_CANON(17) BSP_CANON(18) BSP_CANON(19) BSP_CANON(20)
#undef BSP_CANON
    default:
        return cudaErrorInvalidValue;
    }
}

}  // namespace bsp

extern "C" int batch_spotrf_canonical(int n, int64_t batch, float *A, int32_t *info, int32_t *nfailed,
                                      bspotrf_stream_t stream) {
    if (n < 0 || n > BSPOTRF_CANON_MAX_N) return -1;
    if (batch < 0) return -2;
    if (n == 0 || batch == 0) return 0;
    if (A == nullptr || (reinterpret_cast<uintptr_t>(A) & 3u) != 0) return -3;
    if (info == nullptr) return -4;
    const cudaError_t e = bsp::launch_canon_n(n, A, info, nfailed, batch, (cudaStream_t)stream);
    return e == cudaSuccess ? 0 : (int)e;
}
