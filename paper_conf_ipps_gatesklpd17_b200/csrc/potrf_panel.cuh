// potrf_panel.cuh -- variant PANEL: the SMEM split (left panel of S columns in
// shared memory, trailing (N-S) triangle in registers) with COMPACT code.
//
// Why: a fully unrolled n = 32 factorization is ~12K SASS instructions
// (~200 KB), far beyond the instruction caches; ncu shows the SMEM variant at
// n >= 29 stalled on instruction fetch ("no_instruction" ~4x the issue rate).
// The paper saw the same wall: "Full unrolling pays off up to the size of 20
// ... either the number of instructions overwhelm the compiler, or
// instruction fetching and caching becomes a problem", and its
// answer for larger n was partial unrolling with tile operations
// (Fig. 11).  Here:
//   1. the panel (N x S, in shared memory) is factored by a ROLLED left-looking
//      tile loop over NB x NB register tiles -- Fig. 9's spotrf/strsm/ssyrk/
//      sgemm tile microkernels, only the tile bodies unrolled;
//   2. the SYRK of the panel into the register triangle is a rolled loop over
//      the S panel columns whose unrolled body is one rank-1 update;
//   3. the (N-S) trailing triangle is factored fully unrolled in registers.
// Per-element op order is still Fig. 9's right-looking sequence (updates in
// ascending k, one fma each, scaling by rcp.rn), so results are bitwise equal
// to every other variant (pin P8).
#pragma once

#include "common.cuh"
#include "launch.h"
#include "ptx.cuh"

namespace bsp {

template <int N, int S, int NB>
struct PanelShape {
    static_assert(S % NB == 0, "panel width must be a multiple of the tile size");
    static constexpr int PS = S * N - S * (S - 1) / 2;  // panel slots (lower-packed columns)
    static constexpr int NT = N - S;
    static constexpr int T = NT * (NT + 1) / 2;
    static constexpr int TR = (N + NB - 1) / NB;        // tile rows of the panel
    static constexpr int TC = S / NB;                   // tile columns of the panel
};

// slot of (m, c), c < S, in the lower-packed panel (runtime indices)
template <int N>
__device__ __forceinline__ int pslot(int m, int c) {
    return c * N - (c * (c - 1)) / 2 + (m - c);
}

template <int N, int CT, int S, bool TMA, int NB = 4>
__global__ void __launch_bounds__(TMA ? CT : 256)
potrf_panel_kernel(float *__restrict__ A, int32_t *__restrict__ info,
                   int32_t *__restrict__ nfailed, int64_t batch, int64_t cs) {
    using SH = PanelShape<N, S, NB>;
    constexpr int PS = SH::PS, NT = SH::NT, T = SH::T, TR = SH::TR, TC = SH::TC;
    constexpr int BL = TMA ? CT : 32;
    static_assert(!TMA || (CT == 32 || CT == 64 || CT == 128), "TMA staging needs C in {32,64,128}");

    extern __shared__ __align__(128) float smem[];
    const int64_t gid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const bool active = gid < batch;
    const int64_t g = active ? gid : batch - 1;
    const Addr<N, CT> ad(A, g, cs);
    const int t = TMA ? (int)threadIdx.x : (int)(threadIdx.x & 31);
    float *P = (TMA ? smem : smem + (size_t)(threadIdx.x >> 5) * PS * 32) + t;  // lane-private view

    // ---- stage the panel (TMA bulk copies or per-thread cp.async) -----------
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
#pragma unroll 1
            for (int c = 0; c < S; ++c)
                bulk_g2s(smem + pslot<N>(c, c) * CT, chunk + (c + c * N) * CT,
                         (uint32_t)((N - c) * CT * 4), bar);
        }
    } else {
#pragma unroll 1
        for (int c = 0; c < S; ++c)
#pragma unroll 4
            for (int m = c; m < N; ++m) cp_async4(P + pslot<N>(m, c) * BL, ad.at(m, c));
    }

    // ---- trailing triangle -> registers (in flight during the panel) -------
    float r[T];
#pragma unroll
    for (int n = S; n < N; ++n)
#pragma unroll
        for (int m = n; m < N; ++m) r[tri<NT>(m - S, n - S)] = ld_stream(ad.at(m, n));
    const Addr<N, CT> ads = ad.opaque();           // store addresses (see Addr::opaque)

    if constexpr (TMA) mbar_wait(bar, 0);
    else cp_async_wait_all();

    int inf = 0;
    // ---- 1. panel: rolled left-looking over NB x NB tiles --------------------
    // tile (rb, cb) element (i, j) = panel (rb*NB + i, cb*NB + j)
    auto tile_col_base = [&](int cb, int j) { return pslot<N>(0, cb * NB + j); };  // slot of row 0
#pragma unroll 1
    for (int cb = 0; cb < TC; ++cb) {
        int cbase[NB];
#pragma unroll
        for (int j = 0; j < NB; ++j) cbase[j] = tile_col_base(cb, j);
#pragma unroll 1
        for (int rb = cb; rb < TR; ++rb) {
            const int r0 = rb * NB;
            const bool diag = rb == cb;
            float acc[NB * NB];
#pragma unroll
            for (int j = 0; j < NB; ++j)
#pragma unroll
                for (int i = 0; i < NB; ++i) {
                    const int m = r0 + i;
                    const bool ok = m < N && (!diag || i >= j);
                    acc[i + j * NB] = ok ? P[(cbase[j] + m) * BL] : (i == j ? 1.0f : 0.0f);
                }
            // updates from panel tile columns pb < cb, ascending k
#pragma unroll 1
            for (int pb = 0; pb < cb; ++pb) {
                float a[NB * NB], b[NB * NB];
#pragma unroll
                for (int k = 0; k < NB; ++k) {
                    const int pc = tile_col_base(pb, k);
#pragma unroll
                    for (int i = 0; i < NB; ++i) {
                        const int m = r0 + i;
                        a[i + k * NB] = m < N ? P[(pc + m) * BL] : 0.0f;
                        b[i + k * NB] = P[(pc + cb * NB + i) * BL];  // rows of the diagonal block
                    }
                }
#pragma unroll
                for (int k = 0; k < NB; ++k)
#pragma unroll
                    for (int j = 0; j < NB; ++j)
#pragma unroll
                        for (int i = 0; i < NB; ++i)
                            if (!diag || i >= j)
                                acc[i + j * NB] = f_upd(acc[i + j * NB], a[i + k * NB], b[j + k * NB]);
            }
            if (diag) {
                // spotrf_tile (Fig. 9) on the diagonal block; pivot rule R1
#pragma unroll
                for (int k = 0; k < NB; ++k) {
                    const float d = acc[k + k * NB];
                    pivot_check(d, cb * NB + k, inf);
                    const float s = f_sqrt_pos(d);
                    acc[k + k * NB] = s;
                    const float inv = f_rcp_pos(s);
#pragma unroll
                    for (int i = k + 1; i < NB; ++i) acc[i + k * NB] = f_mul(acc[i + k * NB], inv);
#pragma unroll
                    for (int j = k + 1; j < NB; ++j)
#pragma unroll
                        for (int i = j; i < NB; ++i)
                            acc[i + j * NB] = f_upd(acc[i + j * NB], acc[i + k * NB], acc[j + k * NB]);
                }
            } else {
                // strsm_tile (Fig. 9): acc := acc * L_diag^-T, L_diag from shared memory
                float l[NB * NB];
#pragma unroll
                for (int j = 0; j < NB; ++j)
#pragma unroll
                    for (int i = j; i < NB; ++i) l[i + j * NB] = P[(cbase[j] + cb * NB + i) * BL];
#pragma unroll
                for (int k = 0; k < NB; ++k) {
                    const float inv = f_rcp_pos(l[k + k * NB]);
#pragma unroll
                    for (int i = 0; i < NB; ++i) acc[i + k * NB] = f_mul(acc[i + k * NB], inv);
#pragma unroll
                    for (int j = k + 1; j < NB; ++j)
#pragma unroll
                        for (int i = 0; i < NB; ++i)
                            acc[i + j * NB] = f_upd(acc[i + j * NB], acc[i + k * NB], l[j + k * NB]);
                }
            }
            // final: to shared memory (later tiles read it) and to global memory
#pragma unroll
            for (int j = 0; j < NB; ++j)
#pragma unroll
                for (int i = 0; i < NB; ++i) {
                    const int m = r0 + i;
                    if (m < N && (!diag || i >= j)) {
                        P[(cbase[j] + m) * BL] = acc[i + j * NB];
                        if (active) st_stream(ads.at(m, cb * NB + j), acc[i + j * NB]);
                    }
                }
        }
    }

    // ---- 2. SYRK into the register triangle: rolled over panel columns ------
#pragma unroll 1
    for (int k = 0; k < S; ++k) {
        const int kb = pslot<N>(S, k);
        float v[NT];
#pragma unroll
        for (int m = 0; m < NT; ++m) v[m] = P[(kb + m) * BL];
#pragma unroll
        for (int n = 0; n < NT; ++n)
#pragma unroll
            for (int m = n; m < NT; ++m) r[tri<NT>(m, n)] = f_upd(r[tri<NT>(m, n)], v[m], v[n]);
    }

    // ---- 3. right-looking on the register triangle (fully unrolled) ----------
    sfor<0, NT>([&](auto k_) {
        constexpr int k = BSP_CI(k_);
        const float d = r[tri<NT>(k, k)];
        pivot_check(d, k + S, inf);
        const float s = f_sqrt_pos(d);
        r[tri<NT>(k, k)] = s;
        const float inv = f_rcp_pos(s);
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
cudaError_t launch_panel(const FactorArgs &a) {
    using SH = PanelShape<N, S, 4>;
    const int tpb = TMA ? CT : (a.tpb > 0 ? a.tpb : 32);
    if (tpb > 256) return cudaErrorInvalidConfiguration;
    const size_t sm = TMA ? (size_t)SH::PS * CT * 4 + 16 : (size_t)(tpb / 32) * SH::PS * 32 * 4;
    auto kern = potrf_panel_kernel<N, CT, S, TMA>;
    if (sm > 48 * 1024) {
        const cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
        if (e != cudaSuccess) return e;
    }
    if (const cudaError_t ce = apply_carveout(kern, a.carveout); ce != cudaSuccess) return ce;
    kern<<<grid_for(a.batch, tpb), tpb, sm, a.stream>>>(a.A, a.info, a.nfailed, a.batch, a.cstride);
    return cudaGetLastError();
}

}  // namespace bsp
