// potrf_reg.cuh -- variant REG: one thread per matrix, whole lower triangle in
// registers, fully unrolled right-looking factorization.
//
// This is the paper's fastest kernel shape for n < 20 ("the
// system is able to preserve data in registers throughout the factorization",
// PAPER.md:358 "full unrolling pays off up to the size of 20"): Fig. 10's
// load_lower / store_lower around Fig. 9's spotrf_tile
// with NB = N.  B200 specifics:
//  * the unroll is a C++ template on N instead of pyexpander;
//  * every warp access is one 128-B line (32 lanes x 4 B of 32 consecutive
//    matrices), issued with streaming cache hints (ld.global.cs / st.global.cs)
//    because every byte is touched exactly once per launch;
//  * all N(N+1)/2 loads are issued before the first use (up to 210 independent
//    LDGs in flight per thread at N = 20), which is what keeps HBM busy;
//  * column k is stored as soon as it is final, so its registers die early;
//  * info (LAPACK convention, reading R1) and the fused per-rank failure count
//    (warp ballot + popc + one atomic per warp) come out of the same kernel.
#pragma once

#include "common.cuh"
#include "launch.h"

namespace bsp {

// MINW > 0: ask ptxas for at least MINW resident warps per SM (blocks of 128
// threads), i.e. cap registers at 65536 / (32 * MINW) -- an occupancy axis of
// the sweep.  MINW == 0: no cap (up to 255 registers).
template <int N, int CT, int MINW = 0>
__global__ void __launch_bounds__(MINW ? 128 : 256, MINW ? MINW / 4 : 1)
potrf_reg_kernel(float *__restrict__ A, int32_t *__restrict__ info,
                 int32_t *__restrict__ nfailed, int64_t batch, int64_t cs) {
    constexpr int T = N * (N + 1) / 2;
    const int64_t gid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const bool active = gid < batch;
    // Lanes past the end factor a copy of the last matrix (same cache lines,
    // no extra traffic) and store nothing: no divergence, no pad-lane access.
    const int64_t g = active ? gid : batch - 1;
    const Addr<N, CT> ad(A, g, cs);

    float a[T];
#pragma unroll
    for (int j = 0; j < N; ++j)
#pragma unroll
        for (int i = j; i < N; ++i) a[tri<N>(i, j)] = ld_stream(ad.at(i, j));

    int inf = 0;
    const Addr<N, CT> ads = ad.opaque();           // store addresses (see Addr::opaque)
    sfor<0, N>([&](auto k_) {
        constexpr int k = BSP_CI(k_);
        const float d = a[tri<N>(k, k)];
        pivot_check(d, k, inf);
        const float s = f_sqrt(d);
        a[tri<N>(k, k)] = s;
        const float inv = f_rcp(s);
#pragma unroll
        for (int m = k + 1; m < N; ++m) a[tri<N>(m, k)] = f_mul(a[tri<N>(m, k)], inv);
#pragma unroll
        for (int n = k + 1; n < N; ++n)
#pragma unroll
            for (int m = n; m < N; ++m)
                a[tri<N>(m, n)] = f_upd(a[tri<N>(m, n)], a[tri<N>(m, k)], a[tri<N>(n, k)]);
        if (active) {
#pragma unroll
            for (int m = k; m < N; ++m) st_stream(ads.at(m, k), a[tri<N>(m, k)]);
        }
    });
    if (active) info[gid] = inf;
    count_failures(active && inf != 0, nfailed);
}

template <int N, int CT, int MINW>
cudaError_t launch_reg(const FactorArgs &a) {
    const int tpb = MINW ? 128 : (a.tpb > 0 ? a.tpb : 128);
    if (tpb > 256) return cudaErrorInvalidConfiguration;
    {
        auto kern = potrf_reg_kernel<N, CT, MINW>;
        if (const cudaError_t ce = apply_carveout(kern, a.carveout); ce != cudaSuccess) return ce;
    }
    potrf_reg_kernel<N, CT, MINW><<<grid_for(a.batch, tpb), tpb, 0, a.stream>>>(
        a.A, a.info, a.nfailed, a.batch, a.cstride);
    return cudaGetLastError();
}

}  // namespace bsp

namespace bsp {

// ---- variant REGX: REG with the extra sweep axes of SURVEY §8(f) f3 -------------
// M matrices per thread (thread t of a CTA owns matrices base + t + u*blockDim,
// u < M, so every warp access is still one 128-B line of 32 consecutive
// matrices; the M factorizations are independent instruction streams -> ILP
// and M x the loads in flight per thread), and FAST = the --use_fast_math
// reading of PAPER.md:271,318 (sqrt.approx / rcp.approx, flush-to-zero) --
// reading R4: tolerance-checked (O1-O3), exempt from the bitwise pins, never
// chosen by the default table.
__device__ __forceinline__ float fx_sqrt(float x) {
    float r;
    asm("sqrt.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(x));
    return r;
}
__device__ __forceinline__ float fx_rcp(float x) {
    float r;
    asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(x));
    return r;
}

template <int N, int M, bool FAST>
__global__ void __launch_bounds__(128)
potrf_regx_kernel(float *__restrict__ A, int32_t *__restrict__ info, int32_t *__restrict__ nfailed,
                  int64_t batch, int64_t cs) {
    constexpr int T = N * (N + 1) / 2;
    const int64_t base = (int64_t)blockIdx.x * blockDim.x * M + threadIdx.x;
    float a[M][T];
    bool act[M];
    float *bp[M];
#pragma unroll
    for (int u = 0; u < M; ++u) {
        const int64_t gid = base + (int64_t)u * blockDim.x;
        act[u] = gid < batch;
        const Addr<N, 0> ad(A, act[u] ? gid : batch - 1, cs);
        bp[u] = ad.base;
    }
#pragma unroll
    for (int j = 0; j < N; ++j)
#pragma unroll
        for (int i = j; i < N; ++i)
#pragma unroll
            for (int u = 0; u < M; ++u) a[u][tri<N>(i, j)] = ld_stream(bp[u] + (int64_t)(i + j * N) * cs);
    int inf[M];
#pragma unroll
    for (int u = 0; u < M; ++u) inf[u] = 0;
    sfor<0, N>([&](auto k_) {
        constexpr int k = BSP_CI(k_);
#pragma unroll
        for (int u = 0; u < M; ++u) {
            const float d = a[u][tri<N>(k, k)];
            pivot_check(d, k, inf[u]);
            const float s = FAST ? fx_sqrt(d) : f_sqrt(d);
            a[u][tri<N>(k, k)] = s;
            const float inv = FAST ? fx_rcp(s) : f_rcp(s);
#pragma unroll
            for (int m = k + 1; m < N; ++m) a[u][tri<N>(m, k)] = f_mul(a[u][tri<N>(m, k)], inv);
        }
#pragma unroll
        for (int n = k + 1; n < N; ++n)
#pragma unroll
            for (int m = n; m < N; ++m)
#pragma unroll
                for (int u = 0; u < M; ++u)
                    a[u][tri<N>(m, n)] = f_upd(a[u][tri<N>(m, n)], a[u][tri<N>(m, k)], a[u][tri<N>(n, k)]);
#pragma unroll
        for (int u = 0; u < M; ++u)
            if (act[u]) {
#pragma unroll
                for (int m = k; m < N; ++m) st_stream(bp[u] + (int64_t)(m + k * N) * cs, a[u][tri<N>(m, k)]);
            }
    });
#pragma unroll
    for (int u = 0; u < M; ++u) {
        if (act[u]) info[base + (int64_t)u * blockDim.x] = inf[u];
        count_failures(act[u] && inf[u] != 0, nfailed);
    }
}

template <int N, int M, bool FAST>
cudaError_t launch_regx(const FactorArgs &a) {
    const int tpb = a.tpb > 0 ? a.tpb : 128;
    if (tpb > 128) return cudaErrorInvalidConfiguration;
    const int64_t per = (int64_t)tpb * M;
    {
        auto kern = potrf_regx_kernel<N, M, FAST>;
        if (const cudaError_t ce = apply_carveout(kern, a.carveout); ce != cudaSuccess) return ce;
    }
    potrf_regx_kernel<N, M, FAST><<<(unsigned)((a.batch + per - 1) / per), tpb, 0, a.stream>>>(
        a.A, a.info, a.nfailed, a.batch, a.cstride);
    return cudaGetLastError();
}

}  // namespace bsp
