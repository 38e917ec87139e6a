// potrf_regv.cuh -- variant REGV: REG with 128-bit accesses.  Each thread owns
// FOUR adjacent matrices b..b+3 (b % 4 == 0) of the interleaved layout, so the
// same element (i, j) of its four matrices is one aligned float4: every load
// and store is a 128-bit access and a warp access covers 512 contiguous bytes
// (the north star's "fully coalesced 128-bit accesses", reading R9: with one
// matrix per thread a 128-bit access would have to span four threads' data).
// The four factorizations are independent instruction streams (4-way ILP) with
// the exact Fig. 9 op sequence of REG, so the output is bitwise identical to
// every other variant (pin P8).  For tiny n (n <= 8), where a launch is a few
// microseconds and the kernel is bound by the rate of memory instructions and
// their latency, a quarter of the instructions and 4x the bytes per request is
// what moves it towards the copy ceiling (REG at n = 4 runs exactly at the
// null-factorization ceiling of its own access pattern,
// profiles/r01/probe_ceiling.json).
//
// Needs C % 4 == 0 (C = chunk, or batch for chunk 0); otherwise the launcher
// falls back to REG (same bits).  A group that straddles the end of the batch
// loads its pad lanes (chunked storage is padded) but stores only real lanes.
#pragma once

#include "common.cuh"
#include "launch.h"
#include "potrf_reg.cuh"

namespace bsp {

template <int N>
__global__ void __launch_bounds__(128)
potrf_regv_kernel(float *__restrict__ A, int32_t *__restrict__ info, int32_t *__restrict__ nfailed,
                  int64_t batch, int64_t cs) {
    constexpr int T = N * (N + 1) / 2;
    const int64_t b0 = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) * 4;
    const bool any = b0 < batch;
    const bool full = b0 + 3 < batch;
    const int64_t g = any ? b0 : ((batch - 1) & ~(int64_t)3);
    const Addr<N, 0> ad(A, g, cs);                       // base of matrix g, 16-B aligned

    float a[T][4];
#pragma unroll
    for (int j = 0; j < N; ++j)
#pragma unroll
        for (int i = j; i < N; ++i) {
            const float4 v = __ldcs(reinterpret_cast<const float4 *>(ad.at(i, j)));
            a[tri<N>(i, j)][0] = v.x, a[tri<N>(i, j)][1] = v.y, a[tri<N>(i, j)][2] = v.z, a[tri<N>(i, j)][3] = v.w;
        }

    int inf[4] = {0, 0, 0, 0};
    sfor<0, N>([&](auto k_) {
        constexpr int k = BSP_CI(k_);
#pragma unroll
        for (int u = 0; u < 4; ++u) {
            const float d = a[tri<N>(k, k)][u];
            pivot_check(d, k, inf[u]);
            const float s = f_sqrt(d);
            a[tri<N>(k, k)][u] = s;
            const float inv = f_rcp(s);
#pragma unroll
            for (int m = k + 1; m < N; ++m) a[tri<N>(m, k)][u] = f_mul(a[tri<N>(m, k)][u], inv);
        }
#pragma unroll
        for (int n = k + 1; n < N; ++n)
#pragma unroll
            for (int m = n; m < N; ++m)
#pragma unroll
                for (int u = 0; u < 4; ++u)
                    a[tri<N>(m, n)][u] = f_upd(a[tri<N>(m, n)][u], a[tri<N>(m, k)][u], a[tri<N>(n, k)][u]);
        if (full) {
#pragma unroll
            for (int m = k; m < N; ++m)
                __stcs(reinterpret_cast<float4 *>(ad.at(m, k)),
                       make_float4(a[tri<N>(m, k)][0], a[tri<N>(m, k)][1], a[tri<N>(m, k)][2], a[tri<N>(m, k)][3]));
        } else if (any) {
#pragma unroll
            for (int m = k; m < N; ++m)
#pragma unroll
                for (int u = 0; u < 4; ++u)
                    if (b0 + u < batch) st_stream(ad.at(m, k) + u, a[tri<N>(m, k)][u]);
        }
    });
#pragma unroll
    for (int u = 0; u < 4; ++u) {
        const bool real = b0 + u < batch;
        if (real) info[b0 + u] = inf[u];
        count_failures(real && inf[u] != 0, nfailed);
    }
}

template <int N>
cudaError_t launch_regv(const FactorArgs &a) {
    if (a.cstride % 4 != 0) return launch_reg<N, 0, 0>(a);   // no 16-B groups: REG, same bits
    const int tpb = a.tpb > 0 ? a.tpb : 128;
    if (tpb > 128) return cudaErrorInvalidConfiguration;
    const int64_t groups = (a.batch + 3) / 4;
    {
        auto kern = potrf_regv_kernel<N>;
        if (const cudaError_t ce = apply_carveout(kern, a.carveout); ce != cudaSuccess) return ce;
    }
    potrf_regv_kernel<N><<<grid_for(groups, tpb), tpb, 0, a.stream>>>(a.A, a.info, a.nfailed, a.batch,
                                                                       a.cstride);
    return cudaGetLastError();
}

}  // namespace bsp
