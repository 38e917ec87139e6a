// potrf_regtma.cuh -- variant RTMA: the REG variant (whole lower triangle in
// registers, fully unrolled Fig. 9 order) with its global traffic moved by the
// Tensor Memory Accelerator instead of per-thread loads/stores.
//
// Why: ncu on REG at n = 16 shows the warps stalled on their own LDG
// instructions ("lg_throttle" + "misc" ~4 per issued instruction): 12 warps x
// 136 one-line loads per SM overflow the load/store unit's queues.  In the
// chunked layout (chunk 32 = one warp) column j's lower part is ONE contiguous
// run of (n-j)*128 bytes, so a warp's whole triangle is n cp.async.bulk copies
// issued by one lane into a [slot][lane] shared-memory image (conflict-free:
// bank = lane), read with LDS; final columns are written back to the image and
// stored by cp.async.bulk (global <- shared) column by column, overlapping the
// remaining arithmetic.  A partial last chunk (pad lanes, reading R7) is
// stored per thread instead, so pad lanes are never written.
#pragma once

#include "common.cuh"
#include "launch.h"
#include "ptx.cuh"

namespace bsp {

__device__ __forceinline__ void bulk_s2g(void *dst, const void *src, uint32_t bytes) {
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst),
                 "r"(smem_u32(src)), "r"(bytes)
                 : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
__device__ __forceinline__ void bulk_wait_all() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }

// Resident CTAs per SM to ask ptxas for: as many as shared memory allows, but
// never so many that fewer than T + 40 registers per thread would remain.
template <int N, int W>
struct RtmaOcc {
    static constexpr int T = N * (N + 1) / 2;
    static constexpr int by_smem = (227 * 1024) / (W * T * 32 * 4);
    static constexpr int by_regs = 65536 / (W * 32 * (T + 40));
    static constexpr int v = by_smem < by_regs ? by_smem : by_regs;
    static constexpr int minb = v < 1 ? 1 : v;
};

template <int N, int W>
__global__ void __launch_bounds__(W * 32, RtmaOcc<N, W>::minb)
potrf_regtma_kernel(float *__restrict__ A, int32_t *__restrict__ info,
                    int32_t *__restrict__ nfailed, int64_t batch) {
    constexpr int T = N * (N + 1) / 2;
    extern __shared__ __align__(128) float smem[];
    __shared__ __align__(8) uint64_t bars[W];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int64_t gid = (int64_t)blockIdx.x * (W * 32) + threadIdx.x;
    const bool active = gid < batch;
    int64_t q = ((int64_t)blockIdx.x * (W * 32) + warp * 32) / 32;   // this warp's chunk
    const int64_t qmax = (batch - 1) / 32;
    const bool warp_live = q <= qmax;
    if (!warp_live) q = qmax;                    // idle warp past the end: reread a valid chunk
    const bool full = (q + 1) * 32 <= batch;     // every lane of the chunk is a real matrix
    float *chunk = A + q * 32 * (N * N);
    float *img = smem + (size_t)warp * T * 32;   // [slot][32]
    uint64_t *bar = &bars[warp];

    if (lane == 0) {
        mbar_init(bar, 1);
        mbar_fence_init();
        mbar_arrive_expect_tx(bar, (uint32_t)(T * 32 * 4));
#pragma unroll 1
        for (int j = 0; j < N; ++j)
            bulk_g2s(img + tri<N>(j, j) * 32, chunk + (j + j * N) * 32, (uint32_t)((N - j) * 128), bar);
    }
    __syncwarp();                                // barrier initialised before any lane polls it
    mbar_wait(bar, 0);

    float a[T];
#pragma unroll
    for (int s = 0; s < T; ++s) a[s] = img[s * 32 + lane];

    int inf = 0;
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
        // column k is final
        if (full) {
#pragma unroll
            for (int m = k; m < N; ++m) img[tri<N>(m, k) * 32 + lane] = a[tri<N>(m, k)];
            fence_proxy_async_smem();
            __syncwarp();
            if (lane == 0 && warp_live)
                bulk_s2g(chunk + (k + k * N) * 32, img + tri<N>(k, k) * 32, (uint32_t)((N - k) * 128));
        } else if (active) {
#pragma unroll
            for (int m = k; m < N; ++m) st_stream(chunk + (m + k * N) * 32 + lane, a[tri<N>(m, k)]);
        }
    });
    if (lane == 0) {
        bulk_commit();
        bulk_wait_all();
    }
    if (active) info[gid] = inf;
    count_failures(active && inf != 0, nfailed);
}

template <int N, int W>
cudaError_t launch_regtma(const FactorArgs &a) {
    constexpr int T = N * (N + 1) / 2;
    const size_t sm = (size_t)W * T * 32 * 4;
    auto kern = potrf_regtma_kernel<N, W>;
    if (sm > 48 * 1024) {   // opt in to exactly what this launch needs (static smem counts too)
        const cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
        if (e != cudaSuccess) return e;
    }
    if (const cudaError_t ce = apply_carveout(kern, a.carveout); ce != cudaSuccess) return ce;
    kern<<<grid_for(a.batch, W * 32), W * 32, sm, a.stream>>>(a.A, a.info, a.nfailed, a.batch);
    return cudaGetLastError();
}

}  // namespace bsp

namespace bsp {

// ---- variant RTMAP: persistent RTMA with the next chunk's TMA load in flight
// during the current chunk's arithmetic ---------------------------------------
// Each warp loops over chunks (warp-strided).  Its single [slot][lane] image is
// free as soon as the chunk has been read into registers, so the bulk copies
// for the NEXT chunk are issued right then and land while this chunk is
// factored; results leave through per-thread streaming stores (the image is
// busy with the prefetch).  The grid is exactly the resident warps, so there
// is no wave tail.
template <int N, int W>
__global__ void __launch_bounds__(W * 32, RtmaOcc<N, W>::minb)
potrf_rtmap_kernel(float *__restrict__ A, int32_t *__restrict__ info,
                   int32_t *__restrict__ nfailed, int64_t batch) {
    constexpr int T = N * (N + 1) / 2;
    extern __shared__ __align__(128) float smem[];
    __shared__ __align__(8) uint64_t bars[W];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int64_t nchunks = (batch + 31) / 32;
    const int64_t wstride = (int64_t)gridDim.x * W;
    int64_t q = (int64_t)blockIdx.x * W + warp;
    float *img = smem + (size_t)warp * T * 32;
    uint64_t *bar = &bars[warp];
    auto issue = [&](int64_t qq) {
        if (lane == 0) {
            mbar_arrive_expect_tx(bar, (uint32_t)(T * 32 * 4));
            const float *chunk = A + qq * 32 * (N * N);
#pragma unroll 1
            for (int j = 0; j < N; ++j)
                bulk_g2s(img + tri<N>(j, j) * 32, chunk + (j + j * N) * 32, (uint32_t)((N - j) * 128), bar);
        }
    };
    if (lane == 0) {
        mbar_init(bar, 1);
        mbar_fence_init();
    }
    __syncwarp();
    if (q < nchunks) issue(q);
    uint32_t phase = 0;
    for (; q < nchunks; q += wstride) {
        mbar_wait(bar, phase);
        phase ^= 1;
        float a[T];
#pragma unroll
        for (int s = 0; s < T; ++s) a[s] = img[s * 32 + lane];
        // every lane's shared-memory reads must be done before the async proxy
        // overwrites the image with the next chunk
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        __syncwarp();
        if (q + wstride < nchunks) issue(q + wstride);
        const int64_t gid = q * 32 + lane;
        const bool active = gid < batch;
        float *cbase = A + q * 32 * (N * N) + lane;
        int inf = 0;
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
                for (int m = k; m < N; ++m) st_stream(cbase + (m + k * N) * 32, a[tri<N>(m, k)]);
            }
        });
        if (active) info[gid] = inf;
        count_failures(active && inf != 0, nfailed);
    }
}

template <int N, int W>
cudaError_t launch_rtmap(const FactorArgs &a) {
    constexpr int T = N * (N + 1) / 2;
    const size_t sm = (size_t)W * T * 32 * 4;
    auto kern = potrf_rtmap_kernel<N, W>;
    if (sm > 48 * 1024) {
        const cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
        if (e != cudaSuccess) return e;
    }
    int dev = 0, sms = 148, per_sm = 1;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, W * 32, sm);
    if (per_sm < 1) per_sm = 1;
    const int64_t nchunks = (a.batch + 31) / 32;
    int64_t grid = (int64_t)sms * per_sm;
    const int64_t need = (nchunks + W - 1) / W;
    if (grid > need) grid = need;
    if (const cudaError_t ce = apply_carveout(kern, a.carveout); ce != cudaSuccess) return ce;
    kern<<<(unsigned)grid, W * 32, sm, a.stream>>>(a.A, a.info, a.nfailed, a.batch);
    return cudaGetLastError();
}

}  // namespace bsp
