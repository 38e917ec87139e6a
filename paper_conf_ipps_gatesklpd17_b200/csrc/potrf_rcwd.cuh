// potrf_rcwd.cuh -- variant RCWD: RCW (potrf_rcw.cuh) plus a ninth "diagonal"
// warp that factors each 8x8 diagonal block while the eight row warps run the
// GEMM of their other row slots (round 2, n = 49..64, one CTA per SM).
//
// Why.  In RCW every warp factors the 8x8 diagonal block of column block c
// redundantly, right after the GEMM: the sqrt.rn -> rcp.rn -> scale -> update
// chain (~700 cycles) runs with no independent work beside it, eight blocks
// per 32-matrix group (profiles/r02/ncu_rcw64_r02.md).  Here the GEMM of block
// c is split in two passes over the row buffer RB(c):
//   pass 1: slot c only (the diagonal rows 8c+h) -> published to DB, named
//           barrier 1 (arrive);
//   pass 2: slots c+1..R-1 (and RB(c+1) rows on the way), overlapping the
//           diagonal warp, which waits on barrier 1, factors DB (its own
//           registers; pivot test and info are its job), writes L and the
//           reciprocals to DR and the diagonal block to global memory, and
//           arrives on named barrier 2;
//   the row warps wait on barrier 2, read DR and run the triangular solve.
// The b operand is read twice per block (once per pass).  Op order per
// element is RCW's (k ascending: GEMM then the block's triangular update,
// multiply by rcp.rn), so the output is bitwise identical (pin P8).
#pragma once

#include "common.cuh"
#include "launch.h"
#include "ptx.cuh"
#include "potrf_rcw.cuh"
#include "potrf_tmem.cuh"

namespace bsp {

__device__ __forceinline__ void named_bar_sync(int id, int count) {
    asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(count) : "memory");
}
__device__ __forceinline__ void named_bar_arrive(int id, int count) {
    asm volatile("bar.arrive %0, %1;" ::"r"(id), "r"(count) : "memory");
}

template <int N, int CT>
__global__ void __launch_bounds__(288, 1)
potrf_rcwd_kernel(float *__restrict__ A, int32_t *__restrict__ info, int32_t *__restrict__ nfailed,
                  int64_t batch, int64_t cs) {
    using SH = RcwShape<N, 1>;
    constexpr int R = SH::R, UNIT = SH::UNIT;
    constexpr bool TMA = CT == 32;
    constexpr int NT = 288;                              // barrier 1 / 2 participants
    extern __shared__ __align__(16) float smf[];
    __shared__ uint32_t tmem_base_sh;
    __shared__ __align__(8) uint64_t mbar[2];

    const int h = threadIdx.x >> 5, q = threadIdx.x & 31;
    const bool diag = h == 8;
    const int64_t ngroups = (batch + 31) / 32;
    float *DB = smf + 2 * R * UNIT;                      // diagonal rows gather [36][32]
    float *DR = DB + 36 * 32;                            // factored block + reciprocals [44][32]
    auto unit = [&](int half, int u) { return smf + (size_t)(half * R + u) * UNIT; };

    if (h == 0) {
        tmem_alloc(&tmem_base_sh, SH::COLS);
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
    const uint32_t tb = tmem_base_sh + ((uint32_t)(32 * (h & 3)) << 16) + (uint32_t)(((h >> 2) & 1) * SH::HALF);

    auto prefetch = [&](auto c_, int64_t g, int half) {
        constexpr int c = BSP_CI(c_);
        float *stg = unit(half, c);
        if constexpr (TMA) {
            if (threadIdx.x == 0) {
                fence_proxy_async_smem();
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
        } else if (!diag) {
            if (g * 32 + 31 < batch && cs % 4 == 0) {
                const float *gb = A + ((g * 32) / cs) * cs * (int64_t)(N * N) + (g * 32) % cs;
                const int l8 = q & 7, sub = q >> 3;
#pragma unroll
                for (int tt = 0; tt < 2 * (R - c); ++tt) {
                    const int idx = 4 * tt + sub, r = c + (idx >> 3), w = idx & 7;
                    const int i = 8 * r + h;
                    if (i < N && 8 * c + w < N && (r > c || w <= h))
                        cp_async16(stg + (w * SH::rs(c) + i - 8 * c) * 32 + 4 * l8,
                                   gb + (int64_t)(i + (8 * c + w) * N) * cs + 4 * l8);
                }
            } else {
                const int64_t gm = g * 32 + q;
                const Addr<N, CT> ad(A, gm < batch ? gm : batch - 1, cs);
                sfor<c, R>([&](auto r_) {
                    constexpr int r = BSP_CI(r_);
                    const int i = 8 * r + h;
                    if (i < N) {
#pragma unroll
                        for (int w = 0; w < 8; ++w)
                            if (8 * c + w < N && (r > c || w <= h))
                                cp_async4(stg + (w * SH::rs(c) + i - 8 * c) * 32 + q, ad.at(i, 8 * c + w));
                    }
                });
            }
            cp_async_commit();
        }
    };
    int64_t g = blockIdx.x;
    int ph = 0;
    uint32_t par = 0;
    if (g < ngroups) prefetch(std::integral_constant<int, 0>{}, g, ph);

    float acc[R][8];
    for (; g < ngroups; g += gridDim.x) {
        const int64_t gm = g * 32 + q;
        const bool active = gm < batch;
        const Addr<N, CT> ad(A, active ? gm : batch - 1, cs);
        int inf = 0;                                     // the diagonal warp's
        sfor<0, R>([&](auto c_) {
            constexpr int c = BSP_CI(c_);
            const int half = (c + ph) & 1;
            if constexpr (TMA) {
                mbar_wait(&mbar[half], (par >> half) & 1);
                par ^= 1u << half;
            } else {
                cp_async_wait<0>();
            }
            __syncthreads();                             // RB(c) published; old units free
            if constexpr (c + 1 < R) prefetch(std::integral_constant<int, c + 1>{}, g, half ^ 1);
            else if (g + gridDim.x < ngroups) prefetch(std::integral_constant<int, 0>{}, g + gridDim.x, half ^ 1);

            if (diag) {
                // ---- the diagonal warp: factor block c while the row warps run pass 2
                named_bar_sync(1, NT);
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
                        for (int m = j; m < 8; ++m)
                            d[SH::dt(m, j)] = f_upd(d[SH::dt(m, j)], d[SH::dt(m, k)], d[SH::dt(j, k)]);
                }
#pragma unroll
                for (int t = 0; t < 36; ++t) DR[t * 32 + q] = d[t];
#pragma unroll
                for (int k = 0; k < 8; ++k) DR[(36 + k) * 32 + q] = inv[k];
                named_bar_arrive(2, NT);
                if (active) {
#pragma unroll
                    for (int m = 0; m < 8; ++m)
                        if (8 * c + m < N) {
#pragma unroll
                            for (int w = 0; w <= m; ++w) st_stream(ad.at(8 * c + m, 8 * c + w), d[SH::dt(m, w)]);
                        }
                }
                return;
            }

            // ---- row warps
            const float *stg = unit(half, c) + q;
            sfor<c, R>([&](auto r_) {                    // (a) A(8r+h, 8c..8c+7)
                constexpr int r = BSP_CI(r_);
                const float *src = stg + (8 * (r - c) + h) * 32;
#pragma unroll
                for (int w = 0; w < 8; ++w)
                    acc[r][w] = (r > c || w <= h) && 8 * c + w < N ? src[w * SH::rs(c) * 32] : 0.0f;
            });
            const float4 *rb = reinterpret_cast<const float4 *>(unit(half, 0)) + q;
            float *rbn = unit(half ^ 1, 0);
            auto ldb = [&](float4 (&x)[4][2], int kq) {
#pragma unroll
                for (int wp = 0; wp < 4; ++wp)
#pragma unroll
                    for (int j = 0; j < 2; ++j) x[wp][j] = rb[((kq * 4 + wp) * 2 + j) * 32];
            };
            auto fma_row = [&](float (&ac)[8], const float (&a)[4], const float4 (&x)[4][2]) {
#pragma unroll
                for (int wp = 0; wp < 4; ++wp) {
                    f_upd2(ac[2 * wp], ac[2 * wp + 1], a[0], x[wp][0].x, x[wp][0].y);
                    f_upd2(ac[2 * wp], ac[2 * wp + 1], a[1], x[wp][0].z, x[wp][0].w);
                    f_upd2(ac[2 * wp], ac[2 * wp + 1], a[2], x[wp][1].x, x[wp][1].y);
                    f_upd2(ac[2 * wp], ac[2 * wp + 1], a[3], x[wp][1].z, x[wp][1].w);
                }
            };
            // pass 1: the diagonal row (slot c)
            if constexpr (c > 0) {
#pragma unroll 1
                for (int kq = 0; kq < 2 * c; ++kq) {
                    float4 x[4][2];
                    ldb(x, kq);
                    float a[4];
                    tmem_ld4(tb + (uint32_t)(SH::off(c) + 4 * kq), a);
                    tmem_wait_ld();
                    fma_row(acc[c], a, x);
                }
            }
#pragma unroll
            for (int m = 0; m < 8; ++m)
                if (m == h && 8 * c + m < N) {
#pragma unroll
                    for (int w = 0; w <= m; ++w) DB[SH::dt(m, w) * 32 + q] = acc[c][w];
                }
            named_bar_arrive(1, NT);
            // pass 2: slots c+1..R-1, RB(c+1) rows on the way
            if constexpr (c > 0 && c + 1 < R) {
#pragma unroll 1
                for (int kq = 0; kq < 2 * c; ++kq) {
                    float4 x[4][2];
                    ldb(x, kq);
                    float a[R][4];
                    sfor<c + 1, R>([&](auto r_) {
                        constexpr int r = BSP_CI(r_);
                        tmem_ld4(tb + (uint32_t)(SH::off(r) + 4 * kq), a[r]);
                    });
                    tmem_wait_ld();
                    rb_put(rbn, kq, h, q, a[c + 1]);
                    sfor<c + 1, R>([&](auto r_) {
                        constexpr int r = BSP_CI(r_);
                        fma_row(acc[r], a[r], x);
                    });
                }
            }
            named_bar_sync(2, NT);
            float d[36], inv[8];
#pragma unroll
            for (int t = 0; t < 36; ++t) d[t] = DR[t * 32 + q];
#pragma unroll
            for (int k = 0; k < 8; ++k) inv[k] = DR[(36 + k) * 32 + q];
            // (d) triangular solve of my rows below the block; out, TMEM, RB(c+1)
            sfor<c + 1, R>([&](auto r_) {
                constexpr int r = BSP_CI(r_);
#pragma unroll
                for (int k = 0; k < 8; ++k) {
                    if (8 * c + k >= N) break;
                    acc[r][k] = f_mul(acc[r][k], inv[k]);
#pragma unroll
                    for (int j = k + 1; j < 8; ++j) acc[r][j] = f_upd(acc[r][j], acc[r][k], d[SH::dt(j, k)]);
                }
                const int i = 8 * r + h;
                if (active && i < N) {
#pragma unroll
                    for (int w = 0; w < 8; ++w)
                        if (8 * c + w < N) st_stream(ad.at(i, 8 * c + w), acc[r][w]);
                }
                tmem_st8(tb + (uint32_t)(SH::off(r) + 8 * c), acc[r]);
                if constexpr (r == c + 1) {
                    rb_put(rbn, 2 * c, h, q, &acc[r][0]);
                    rb_put(rbn, 2 * c + 1, h, q, &acc[r][4]);
                }
            });
            tmem_wait_st();
        });
        if (diag) {
            if (active) info[gm] = inf;
            count_failures(active && inf != 0, nfailed);
        }
        ph = (ph + R) & 1;
    }

    tmem_fence_before();
    __syncthreads();
    if (h == 0) {
        tmem_fence_after();
        tmem_dealloc(tmem_base_sh, SH::COLS);
    }
}

template <int N, int CT>
cudaError_t launch_rcwd(const FactorArgs &a) {
    using SH = RcwShape<N, 1>;
    auto kern = potrf_rcwd_kernel<N, CT>;
    size_t sm = SH::SMEM + (size_t)44 * 32 * sizeof(float);   // + DR
    if (sm < (size_t)116 * 1024) sm = (size_t)116 * 1024;     // one CTA per SM (all 512 TMEM columns)
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    if (e != cudaSuccess) return e;
    if (const cudaError_t ce = apply_carveout(kern, a.carveout); ce != cudaSuccess) return ce;
    int dev = 0, nsm = 0;
    e = cudaGetDevice(&dev);
    if (e == cudaSuccess) e = cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
    if (e != cudaSuccess) return e;
    const int64_t groups = (a.batch + 31) / 32;
    const int64_t grid = groups < (int64_t)nsm ? groups : (int64_t)nsm;
    kern<<<(unsigned)grid, 288, sm, a.stream>>>(a.A, a.info, a.nfailed, a.batch, a.cstride);
    return cudaGetLastError();
}

}  // namespace bsp
