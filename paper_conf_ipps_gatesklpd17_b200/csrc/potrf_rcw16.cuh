// potrf_rcw16.cuh -- variant RCW16: RCW (potrf_rcw.cuh) with SIXTEEN warps per
// 32 matrices.  Warp h owns rows i = 16r + h (slots r = 0..RS-1); the column
// blocks stay 8 wide, so a block's 8 diagonal rows belong to half of the warps
// (h / 8 == c % 2, slot c / 2) and each warp's slot c / 2 is, depending on its
// half, diagonal, below the block, or finished -- a warp-uniform runtime test on
// a compile-time slot.  Row i keeps L(i, 0..8*floor(i/8)-1) in TMEM: at n = 64
// 128 columns per warp, i.e. four warps per lane quarter in one 512-column
// allocation.  Why: TMEM admits one 32-matrix CTA per SM for n > 48, and with 8
// warps (2 per scheduler) the block loop is latency-bound (profiles/r01/
// ncu_rcw.md); 16 warps put 4 per scheduler on the same data, at the price of
// twice the row-buffer reads (each warp reads the 8 b rows) and of the
// diagonal block factored by 16 warps.  Op order per element is RCW's, so the
// output is bitwise identical to every other variant (pin P8).
#pragma once

#include "common.cuh"
#include "launch.h"
#include "ptx.cuh"
#include "potrf_tmem.cuh"
#include "potrf_rcw.cuh"

namespace bsp {

template <int N>
struct Rcw16Shape {
    static constexpr int P = 16;                         // warps = row classes
    static constexpr int R = (N + 7) / 8;                // 8-wide column blocks
    static constexpr int RS = (N + P - 1) / P;           // row slots per warp
    static constexpr int UNIT = 8 * 8 * 32;              // floats per 8 KB unit
    static constexpr int WCOLS = 128;                    // TMEM columns per warp (4 per lane quarter)
    __host__ __device__ static constexpr int dt(int m, int k) { return m * (m + 1) / 2 + k; }
    __host__ __device__ static constexpr int rs(int c) { return N - 8 * c; }
    __host__ __device__ static constexpr uint32_t bytes(int c) {
        uint32_t b = 0;
        for (int w = 0; w < 8; ++w)
            if (8 * c + w < N) b += (uint32_t)(N - 8 * c - w) * 128u;
        return b;
    }
    __host__ __device__ static constexpr int cols(int h) {   // TMEM columns warp h addresses
        int s = 0;
        for (int r = 0; r < RS; ++r) s += 8 * ((P * r + h) / 8);
        return s;
    }
    static constexpr size_t SMEM = (size_t)(2 * R * UNIT + 36 * 32) * sizeof(float);
    static_assert(cols(P - 1) <= WCOLS && cols(7) <= WCOLS, "slots exceed the TMEM column budget");
};

template <int N, int CT>
__global__ void __launch_bounds__(512, 1)
potrf_rcw16_kernel(float *__restrict__ A, int32_t *__restrict__ info, int32_t *__restrict__ nfailed,
                   int64_t batch, int64_t cs) {
    using SH = Rcw16Shape<N>;
    constexpr int R = SH::R, RS = SH::RS, UNIT = SH::UNIT, P = SH::P;
    constexpr bool TMA = CT == 32;
    extern __shared__ __align__(16) float smf[];
    __shared__ uint32_t tmem_base_sh;
    __shared__ __align__(8) uint64_t mbar[2];

    const int h = threadIdx.x >> 5, q = threadIdx.x & 31;
    const int64_t ngroups = (batch + 31) / 32;
    float *DB = smf + 2 * R * UNIT;
    auto unit = [&](int half, int u) { return smf + (size_t)(half * R + u) * UNIT; };

    if (h == 0) {
        tmem_alloc(&tmem_base_sh, 512);
        tmem_relinquish();
    }
    if (TMA && threadIdx.x == 0) {
        mbar_init(&mbar[0], 1);
        mbar_init(&mbar[1], 1);
        mbar_fence_init();
    }
    tmem_fence_before();
    __syncthreads();
    tmem_fence_after();
    const uint32_t tb = tmem_base_sh + ((uint32_t)(32 * (h & 3)) << 16) + (uint32_t)((h >> 2) * SH::WCOLS);
    int offs[RS];                                        // TMEM column of slot r (warp-uniform)
    {
        int o = 0;
#pragma unroll
        for (int r = 0; r < RS; ++r) {
            offs[r] = o;
            o += 8 * ((P * r + h) / 8);
        }
    }

    auto prefetch = [&](auto c_, int64_t g, int half) {
        constexpr int c = BSP_CI(c_);
        float *stg = unit(half, c);
        if constexpr (TMA) {
            if (threadIdx.x == 0) {
                fence_proxy_async_smem();        // generic RB stores -> async-proxy writes (see RCW)
                const float *chunk = A + g * (int64_t)(32 * N * N);
                mbar_arrive_expect_tx(&mbar[half], SH::bytes(c));
#pragma unroll
                for (int w = 0; w < 8; ++w) {
                    const int j = 8 * c + w;
                    if (j < N)
                        bulk_g2s(stg + (w * SH::rs(c) + w) * 32, chunk + (j + j * N) * 32,
                                 (uint32_t)((N - j) * 128), &mbar[half]);
                }
            }
        } else if (g * 32 + 31 < batch && cs % 4 == 0) {
            // full group: 16-B copies, 8 lanes per 128-B line (as RCW)
            const float *gb = A + ((g * 32) / cs) * cs * (int64_t)(N * N) + (g * 32) % cs;
            const int l8 = q & 7, sub = q >> 3;
#pragma unroll
            for (int tt = 0; tt < 2 * RS; ++tt) {
                const int idx = 4 * tt + sub, r = idx >> 3, w = idx & 7;
                const int i = P * r + h;
                if (i >= 8 * c && i < N && 8 * c + w < N && 8 * c + w <= i)
                    cp_async16(stg + (w * SH::rs(c) + i - 8 * c) * 32 + 4 * l8,
                               gb + (int64_t)(i + (8 * c + w) * N) * cs + 4 * l8);
            }
            cp_async_commit();
        } else {
            const int64_t gm = g * 32 + q;
            const Addr<N, CT> ad(A, gm < batch ? gm : batch - 1, cs);
            sfor<0, RS>([&](auto r_) {
                constexpr int r = BSP_CI(r_);
                const int i = P * r + h;
                if (i >= 8 * c && i < N) {
#pragma unroll
                    for (int w = 0; w < 8; ++w)
                        if (8 * c + w < N && 8 * c + w <= i)
                            cp_async4(stg + (w * SH::rs(c) + i - 8 * c) * 32 + q, ad.at(i, 8 * c + w));
                }
            });
            cp_async_commit();
        }
    };
    int64_t g = blockIdx.x;
    int ph = 0;
    uint32_t par = 0;
    if (g < ngroups) prefetch(std::integral_constant<int, 0>{}, g, ph);

    float acc[RS][8];
    for (; g < ngroups; g += gridDim.x) {
        const int64_t gm = g * 32 + q;
        const bool active = gm < batch;
        const Addr<N, CT> ad(A, active ? gm : batch - 1, cs);
        int inf = 0;
        sfor<0, R>([&](auto c_) {
            constexpr int c = BSP_CI(c_);
            const int half = (c + ph) & 1;
            if constexpr (TMA) {
                mbar_wait(&mbar[half], (par >> half) & 1);
                par ^= 1u << half;
            } else {
                cp_async_wait<0>();
            }
            __syncthreads();
            if constexpr (c + 1 < R) prefetch(std::integral_constant<int, c + 1>{}, g, half ^ 1);
            else if (g + gridDim.x < ngroups) prefetch(std::integral_constant<int, 0>{}, g + gridDim.x, half ^ 1);
            const float *stg = unit(half, c) + q;
            // slot r of this warp relative to block c: row P*r + h = 8c + o,
            // o < 0 finished, 0 <= o < 8 diagonal, o >= 8 below the block
            constexpr int rlo = (8 * c) / P;             // first slot that can be live

            // (a) accumulators of my live rows
            sfor<rlo, RS>([&](auto r_) {
                constexpr int r = BSP_CI(r_);
                const int o = P * r + h - 8 * c;
                if (o >= 0 && P * r + h < N) {
                    const float *src = stg + o * 32;
#pragma unroll
                    for (int w = 0; w < 8; ++w)
                        acc[r][w] = (o >= 8 || w <= o) && 8 * c + w < N ? src[w * SH::rs(c) * 32] : 0.0f;
                }
            });

            // (b) GEMM over k < 8c; the rows of block c+1 are published on the way
            if constexpr (c > 0) {
                const float4 *rb = reinterpret_cast<const float4 *>(unit(half, 0)) + q;
                float4 *rbn = reinterpret_cast<float4 *>(unit(half ^ 1, 0)) + q;
#pragma unroll 1
                for (int kq = 0; kq < 2 * c; ++kq) {
                    float b[8][4];
#pragma unroll
                    for (int w = 0; w < 8; ++w) {
                        const float4 x = rb[(kq * 8 + w) * 32];
                        b[w][0] = x.x, b[w][1] = x.y, b[w][2] = x.z, b[w][3] = x.w;
                    }
                    float a[RS][4];
                    sfor<rlo, RS>([&](auto r_) {
                        constexpr int r = BSP_CI(r_);
                        tmem_ld4(tb + (uint32_t)(offs[r] + 4 * kq), a[r]);
                    });
                    tmem_wait_ld();
                    sfor<rlo, RS>([&](auto r_) {
                        constexpr int r = BSP_CI(r_);
                        const int o1 = P * r + h - 8 * (c + 1);
                        if (c + 1 < R && o1 >= 0 && o1 < 8)
                            rbn[(kq * 8 + o1) * 32] = make_float4(a[r][0], a[r][1], a[r][2], a[r][3]);
                    });
                    sfor<rlo, RS>([&](auto r_) {
                        constexpr int r = BSP_CI(r_);
                        if (P * r + h >= 8 * c) {
#pragma unroll
                            for (int kk = 0; kk < 4; ++kk)
#pragma unroll
                                for (int w = 0; w < 8; ++w) acc[r][w] = f_upd(acc[r][w], a[r][kk], b[w][kk]);
                        }
                    });
                }
            }

            // (c) diagonal block: gather (rows owned by half of the warps), factor everywhere
            sfor<rlo, RS>([&](auto r_) {
                constexpr int r = BSP_CI(r_);
                const int o = P * r + h - 8 * c;
                if (o >= 0 && o < 8 && 8 * c + o < N) {
#pragma unroll
                    for (int w = 0; w < 8; ++w)
                        if (w <= o) DB[(o * (o + 1) / 2 + w) * 32 + q] = acc[r][w];
                }
            });
            __syncthreads();
            float d[36], inv[8];
#pragma unroll
            for (int t = 0; t < 36; ++t) d[t] = DB[t * 32 + q];
#pragma unroll
            for (int k = 0; k < 8; ++k) {
                if (8 * c + k >= N) break;
                const float p = d[SH::dt(k, k)];
                pivot_check(p, 8 * c + k, inf);
                const float s = f_sqrt(p);
                d[SH::dt(k, k)] = s;
                inv[k] = f_rcp(s);
#pragma unroll
                for (int m = k + 1; m < 8; ++m) d[SH::dt(m, k)] = f_mul(d[SH::dt(m, k)], inv[k]);
#pragma unroll
                for (int j = k + 1; j < 8; ++j)
#pragma unroll
                    for (int m = j; m < 8; ++m) d[SH::dt(m, j)] = f_upd(d[SH::dt(m, j)], d[SH::dt(m, k)], d[SH::dt(j, k)]);
            }
            {
                const int od = h - 8 * (c % 2);              // my diagonal row, if h / 8 == c % 2
                if (active && od >= 0 && od < 8 && 8 * c + od < N) {
#pragma unroll
                    for (int m = 0; m < 8; ++m)
                        if (m == od) {
#pragma unroll
                            for (int w = 0; w <= m; ++w) st_stream(ad.at(8 * c + m, 8 * c + w), d[SH::dt(m, w)]);
                        }
                }
            }

            // (d) triangular solve of my rows below the block; out, TMEM, RB(c+1)
            sfor<rlo, RS>([&](auto r_) {
                constexpr int r = BSP_CI(r_);
                const int o = P * r + h - 8 * c;
                if (c + 1 < R && o >= 8) {
#pragma unroll
                    for (int k = 0; k < 8; ++k) {
                        acc[r][k] = f_mul(acc[r][k], inv[k]);
#pragma unroll
                        for (int j = k + 1; j < 8; ++j) acc[r][j] = f_upd(acc[r][j], acc[r][k], d[SH::dt(j, k)]);
                    }
                    const int i = P * r + h;
                    if (active && i < N) {
#pragma unroll
                        for (int w = 0; w < 8; ++w) st_stream(ad.at(i, 8 * c + w), acc[r][w]);
                    }
                    tmem_st8(tb + (uint32_t)(offs[r] + 8 * c), acc[r]);
                    if (o < 16) {                                // a row of block c+1
                        float4 *rbn = reinterpret_cast<float4 *>(unit(half ^ 1, 0)) + q;
                        rbn[((2 * c) * 8 + o - 8) * 32] = make_float4(acc[r][0], acc[r][1], acc[r][2], acc[r][3]);
                        rbn[((2 * c + 1) * 8 + o - 8) * 32] = make_float4(acc[r][4], acc[r][5], acc[r][6], acc[r][7]);
                    }
                }
            });
            tmem_wait_st();
        });
        if (active && h == 0) info[gm] = inf;
        if (h == 0) count_failures(active && inf != 0, nfailed);
        ph = (ph + R) & 1;
    }

    tmem_fence_before();
    __syncthreads();
    if (h == 0) {
        tmem_fence_after();
        tmem_dealloc(tmem_base_sh, 512);
    }
}

template <int N, int CT>
cudaError_t launch_rcw16(const FactorArgs &a) {
    using SH = Rcw16Shape<N>;
    auto kern = potrf_rcw16_kernel<N, CT>;
    size_t sm = SH::SMEM;
    if (sm < (size_t)116 * 1024) sm = (size_t)116 * 1024;   // one CTA per SM (all 512 TMEM columns)
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    if (e != cudaSuccess) return e;
    int dev = 0, nsm = 0;
    e = cudaGetDevice(&dev);
    if (e == cudaSuccess) e = cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
    if (e != cudaSuccess) return e;
    const int64_t groups = (a.batch + 31) / 32;
    const int64_t grid = groups < (int64_t)nsm ? groups : (int64_t)nsm;
    if (const cudaError_t ce = apply_carveout(kern, a.carveout); ce != cudaSuccess) return ce;
    kern<<<(unsigned)grid, 512, sm, a.stream>>>(a.A, a.info, a.nfailed, a.batch, a.cstride);
    return cudaGetLastError();
}

}  // namespace bsp
