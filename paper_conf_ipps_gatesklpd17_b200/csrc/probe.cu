// probe.cu -- diagnostic "null factorization": the exact memory traffic of the
// REG variant (each thread loads its matrix's lower triangle with the same
// one-line-per-warp-access pattern and stores it back unchanged, plus info)
// with no arithmetic.  Its bandwidth is the practical ceiling of the access
// pattern, reported beside the factorization's roofline fraction.
#include <cuda_runtime.h>
#include <stdint.h>

#include "../../include/bspotrf_synth.h"
#include "common.cuh"

namespace bsp {

template <int N>
__global__ void __launch_bounds__(256)
probe_copy_lower_kernel(float *__restrict__ A, int32_t *__restrict__ info, int64_t batch, int64_t cs) {
    constexpr int T = N * (N + 1) / 2;
    const int64_t gid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const bool active = gid < batch;
    const int64_t g = active ? gid : batch - 1;
    const Addr<N, 32> ad(A, g, cs);
    float a[T];
#pragma unroll
    for (int j = 0; j < N; ++j)
#pragma unroll
        for (int i = j; i < N; ++i) a[tri<N>(i, j)] = ld_stream(ad.at(i, j));
    if (active) {
#pragma unroll
        for (int j = 0; j < N; ++j)
#pragma unroll
            for (int i = j; i < N; ++i) st_stream(ad.at(i, j), a[tri<N>(i, j)]);
        info[gid] = 0;
    }
}

}  // namespace bsp

extern "C" int bspotrf_probe_copy_lower(int n, int64_t batch, float *A, int32_t *info, int tpb,
                                        bspotrf_stream_t stream) {
    if (batch <= 0) return batch == 0 ? 0 : -2;
    if (A == nullptr || info == nullptr) return -3;
    if (tpb <= 0 || tpb > 256 || tpb % 32) return -5;
    const unsigned grid = (unsigned)((batch + tpb - 1) / tpb);
    cudaStream_t s = (cudaStream_t)stream;
    switch (n) {
    case 4: bsp::probe_copy_lower_kernel<4><<<grid, tpb, 0, s>>>(A, info, batch, 32); break;
    case 8: bsp::probe_copy_lower_kernel<8><<<grid, tpb, 0, s>>>(A, info, batch, 32); break;
    case 16: bsp::probe_copy_lower_kernel<16><<<grid, tpb, 0, s>>>(A, info, batch, 32); break;
    case 20: bsp::probe_copy_lower_kernel<20><<<grid, tpb, 0, s>>>(A, info, batch, 32); break;
    default: return -1;
    }
    return (int)cudaGetLastError();
}
