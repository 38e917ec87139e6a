// potrf_smem.cuh -- variant SMEM: one thread per matrix for n where the lower
// triangle no longer fits in registers (n(n+1)/2 > ~200 floats, i.e. n > ~19;
// the paper hits the same wall at ~20).
//
// Split at column S:
//   * the left panel -- columns 0..S-1, rows j..N-1 -- is staged in shared
//     memory, laid out [slot][lane] so that every thread reads only its own
//     lane (bank = lane: conflict-free, no barriers between threads);
//   * the trailing triangle -- rows/cols S..N-1 -- lives in registers.
// With chunk C in {32, 64, 128} a block owns one chunk and the panel arrives by
// S TMA bulk copies (cp.async.bulk, one per panel column: in the chunked layout
// column c's lower part is ONE contiguous run of (N-c)*C floats in global
// memory, and the same run in the [slot][lane] shared layout).  Otherwise each
// thread stages its own panel with 4-byte cp.async (LDGSTS).
//
// Arithmetic, in the order that keeps every element's op sequence identical to
// right-looking Alg. 1 / Fig. 9 (pin P8):
//   1. panel, left-looking by column c = 0..S-1 (Fig. 4 order):
//      col := A[c:N, c]; for k < c: col[m] = fma(-L[m][k], L[c][k], col[m]);
//      pivot / sqrt / reciprocal / scale; store col (global + shared);
//   2. SYRK of the panel into the register triangle, k = 0..S-1 ascending;
//   3. right-looking Alg. 1 on the register triangle for k = S..N-1.
#pragma once

#include "common.cuh"
#include "launch.h"
#include "ptx.cuh"

namespace bsp {

template <int N, int S>
struct SmemShape {
    static constexpr int PS = S * N - S * (S - 1) / 2;  // panel slots
    static constexpr int NT = N - S;                    // trailing order
    static constexpr int T = NT * (NT + 1) / 2;         // trailing floats
};

template <int N, int CT, int S, bool TMA>
__global__ void __launch_bounds__(TMA ? CT : 256)
potrf_smem_kernel(float *__restrict__ A, int32_t *__restrict__ info,
                  int32_t *__restrict__ nfailed, int64_t batch, int64_t cs) {
    using SH = SmemShape<N, S>;
    constexpr int PS = SH::PS;
    constexpr int NT = SH::NT;
    constexpr int T = SH::T;
    constexpr int BL = TMA ? CT : 32;  // lanes per staging group
    static_assert(S >= 1 && S < N, "panel width");
    static_assert(!TMA || (CT == 32 || CT == 64 || CT == 128), "TMA staging needs C in {32,64,128}");

    extern __shared__ __align__(128) float smem[];
    const int64_t gid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const bool active = gid < batch;
    const int64_t g = active ? gid : batch - 1;
    const Addr<N, CT> ad(A, g, cs);

    const int t = TMA ? (int)threadIdx.x : (int)(threadIdx.x & 31);
    float *P = TMA ? smem : smem + (size_t)(threadIdx.x >> 5) * PS * 32;
#define BSP_P(m, c) P[tri<N>((m), (c)) * BL + t]

    // ---- stage the panel ----------------------------------------------------
    uint64_t *bar = reinterpret_cast<uint64_t *>(smem + (size_t)PS * BL);
    if constexpr (TMA) {
        if (threadIdx.x == 0) {
            mbar_init(bar, 1);
            mbar_fence_init();
        }
        __syncthreads();
        if (threadIdx.x == 0) {
            mbar_arrive_expect_tx(bar, (uint32_t)(PS * CT * 4));
            const float *chunk = A + (int64_t)blockIdx.x * CT * (N * N);
#pragma unroll
            for (int c = 0; c < S; ++c)
                bulk_g2s(smem + tri<N>(c, c) * CT, chunk + (c + c * N) * CT,
                         (uint32_t)((N - c) * CT * 4), bar);
        }
    } else {
#pragma unroll
        for (int c = 0; c < S; ++c)
#pragma unroll
            for (int m = c; m < N; ++m) cp_async4(&BSP_P(m, c), ad.at(m, c));
    }

    // ---- trailing triangle into registers (in flight during staging) -------
    float r[T];
#pragma unroll
    for (int n = S; n < N; ++n)
#pragma unroll
        for (int m = n; m < N; ++m) r[tri<NT>(m - S, n - S)] = ld_stream(ad.at(m, n));
    const Addr<N, CT> ads = ad.opaque();           // store addresses (see Addr::opaque)

    if constexpr (TMA) {
        mbar_wait(bar, 0);
    } else {
        cp_async_wait_all();
    }

    int inf = 0;
    // ---- 1. panel, left-looking by column ------------------------------------
    sfor<0, S>([&](auto c_) {
        constexpr int c = BSP_CI(c_);
        float col[N];
#pragma unroll
        for (int m = c; m < N; ++m) col[m] = BSP_P(m, c);
        sfor<0, c>([&](auto k_) {
            constexpr int k = BSP_CI(k_);
            const float lck = BSP_P(c, k);
#pragma unroll
            for (int m = c; m < N; ++m) col[m] = f_upd(col[m], BSP_P(m, k), lck);
            sched_fence();
        });
        const float d = col[c];
        pivot_check(d, c, inf);
        const float s = f_sqrt(d);
        col[c] = s;
        const float inv = f_rcp(s);
#pragma unroll
        for (int m = c + 1; m < N; ++m) col[m] = f_mul(col[m], inv);
        if (active) {
#pragma unroll
            for (int m = c; m < N; ++m) st_stream(ads.at(m, c), col[m]);
        }
#pragma unroll
        for (int m = c + 1; m < N; ++m) BSP_P(m, c) = col[m];
    });

    // ---- 2. SYRK: trailing -= panel rows S..N-1 times their transpose -------
    sfor<0, S>([&](auto k_) {
        constexpr int k = BSP_CI(k_);
        float v[NT];
#pragma unroll
        for (int m = S; m < N; ++m) v[m - S] = BSP_P(m, k);
#pragma unroll
        for (int n = 0; n < NT; ++n)
#pragma unroll
            for (int m = n; m < NT; ++m) r[tri<NT>(m, n)] = f_upd(r[tri<NT>(m, n)], v[m], v[n]);
        sched_fence();
    });
#undef BSP_P

    // ---- 3. right-looking on the register triangle -----------------------------
    sfor<0, NT>([&](auto k_) {
        constexpr int k = BSP_CI(k_);
        const float d = r[tri<NT>(k, k)];
        pivot_check(d, k + S, inf);
        const float s = f_sqrt(d);
        r[tri<NT>(k, k)] = s;
        const float inv = f_rcp(s);
#pragma unroll
        for (int m = k + 1; m < NT; ++m) r[tri<NT>(m, k)] = f_mul(r[tri<NT>(m, k)], inv);
#pragma unroll
        for (int n = k + 1; n < NT; ++n)
#pragma unroll
            for (int m = n; m < NT; ++m)
                r[tri<NT>(m, n)] = f_upd(r[tri<NT>(m, n)], r[tri<NT>(m, k)], r[tri<NT>(n, k)]);
        if (active) {
#pragma unroll
            for (int m = k; m < NT; ++m) st_stream(ads.at(m + S, k + S), r[tri<NT>(m, k)]);
        }
    });
    if (active) info[gid] = inf;
    count_failures(active && inf != 0, nfailed);
}

template <int N, int CT, int S, bool TMA>
size_t smem_bytes(int tpb) {
    using SH = SmemShape<N, S>;
    if (TMA) return (size_t)SH::PS * CT * 4 + 16;
    return (size_t)(tpb / 32) * SH::PS * 32 * 4;
}

template <int N, int CT, int S, bool TMA>
cudaError_t launch_smem(const FactorArgs &a) {
    int tpb = TMA ? CT : (a.tpb > 0 ? a.tpb : 32);
    if (tpb > 256) return cudaErrorInvalidConfiguration;
    const size_t sm = smem_bytes<N, CT, S, TMA>(tpb);
    auto kern = potrf_smem_kernel<N, CT, S, TMA>;
    if (sm > 48 * 1024) {
        const cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
        if (e != cudaSuccess) return e;
    }
    if (const cudaError_t ce = apply_carveout(kern, a.carveout); ce != cudaSuccess) return ce;
    kern<<<grid_for(a.batch, tpb), tpb, sm, a.stream>>>(a.A, a.info, a.nfailed, a.batch, a.cstride);
    return cudaGetLastError();
}

}  // namespace bsp
