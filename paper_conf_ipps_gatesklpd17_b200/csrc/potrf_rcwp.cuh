// potrf_rcwp.cuh -- variant RCWP ("paged RCW"): RCW's row-cyclic warps
// (potrf_rcw.cuh: 8 warps share 32 matrices, lane = matrix, warp h owns rows
// 8r + h) with the factor kept in Tensor Memory PAGES that are recycled as row
// slots die, so that TWO 32-matrix groups -- two CTAs, 16 warps -- fit per SM
// at n = 49..64, where RCW fits one (round 2).
//
// Why.  RCW at n = 64 is latency-bound at one CTA per SM (8 warps, 2 per
// scheduler: profiles/r02/ncu_rcw64_r02.md).  Its TMEM layout is static: slot r
// of warp h holds L(8r+h, 0..8r-1) at columns 4r(r-1).., 224 columns per warp
// at n = 64, so one group needs all 512 columns of every lane quarter.  But in
// the left-looking order a slot is dead after its own column block: the GEMM of
// block c reads slots r >= c, columns < 8c; slot c is published and then never
// read again.  Live 8-column pages after block t are (r, c) with c <= t < r:
// (t+1)(R-1-t) of them, at most 16 (128 columns) at n = 64 -- half of RCW's.
// A compile-time greedy colouring (RcwpPages) assigns page (r, c) -- L(8r+h,
// 8c..8c+7) -- a column slot that no simultaneously live page uses; each CTA
// allocates 256 columns (warp h: lane quarter h % 4, columns (h / 4) * 128).
// Shared memory shrinks to ONE set of R units of 8 KB (RCW: two): RB(c), the
// rows 8c..8c+7 of L (the GEMM's b operand), in units 0..c-1 and the input
// stage of block c in units c..R-1 (64 KB + the diagonal gather at n = 64), so
// two CTAs fit; registers are capped at 128 per thread.
//
// Per column block c (RCW's op order per element, so the bits are RCW's and
// every other variant's, pin P8):
//   1. wait for stage(c);  (a) acc[r] = A(8r+h, 8c..8c+7), r >= c;
//   B1 (stage(c) consumed, RB(c) visible) -> stage(c+1) issued into units
//      c+1..R-1 (TMA bulk copies for chunk 32, per-thread cp.async otherwise);
//   (b) acc[r] -= L(8r+h, 0..8c-1) RB(c)^T, k ascending (FFMA2 pairs);
//   (c) diagonal rows gathered (B2) and the 8x8 block factored by every warp;
//   (d) rows below: triangular solve, streaming stores, page (r, c) written;
//   B3 (all warps are done with RB(c)) -> RB(c+1) published into units 0..c
//      from pages (c+1, 0..c-1) and the registers of slot c+1; after the last
//      block the next group's stage(0) is issued instead.
// With one stage buffer the next group's first block is not prefetched during
// the current group's last block; the second CTA on the SM covers that gap.
#pragma once

#include "common.cuh"
#include "launch.h"
#include "ptx.cuh"
#include "potrf_rcw.cuh"
#include "potrf_tmem.cuh"
#include "tma2d.cuh"

namespace bsp {

// Runtime-chunk staging by 2-D TMA (round 2): the interleaved array viewed as
// rows (one row = element (i, j) of C consecutive matrices, C*4 bytes apart)
// x C columns; block c's stage of column j = 8c+w is ONE box of 32 matrices x
// (N - 8c) rows (rows 8c..N-1 of the column; the rows above the diagonal land in
// stage slots the kernel never reads).  One tensor map per block c (its box
// height), passed by value as a __grid_constant__ parameter.
struct RcwpMaps {
    CUtensorMap m[8];
};

__device__ __forceinline__ void tmem_ld8(uint32_t taddr, float *v) {
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                 : "=f"(v[0]), "=f"(v[1]), "=f"(v[2]), "=f"(v[3]), "=f"(v[4]), "=f"(v[5]), "=f"(v[6]),
                   "=f"(v[7])
                 : "r"(taddr)
                 : "memory");
}

// Page colouring of the live set: page (r, c), c < r, is written in block c
// (step d) and read for the last time in block r (step b of block r reads slot
// r; step 3 of block r - 1 publishes it).  Greedy over blocks t: the pages of
// slot t are freed, then (r, t), r = t+1..R-1, take the lowest free pages.
// The number of pages equals the interval-graph bound max_t (t+1)(R-1-t);
// valid() re-checks at compile time that no two pages live at the same block
// boundary share a slot (static_assert in RcwpShape).
template <int R>
struct RcwpPages {
    int pg[8][8];
    int npages;
    __host__ __device__ constexpr RcwpPages() : pg{}, npages(0) {
        int fr[64] = {};
        int nf = 0;
        for (int t = 0; t + 1 < R; ++t) {
            for (int c = 0; c < t; ++c) fr[nf++] = pg[t][c];
            for (int i = 1; i < nf; ++i)                 // ascending
                for (int j = i; j > 0 && fr[j - 1] > fr[j]; --j) {
                    const int s = fr[j];
                    fr[j] = fr[j - 1];
                    fr[j - 1] = s;
                }
            for (int r = t + 1; r < R; ++r) {
                if (nf > 0) {
                    pg[r][t] = fr[0];
                    for (int i = 1; i < nf; ++i) fr[i - 1] = fr[i];
                    --nf;
                } else {
                    pg[r][t] = npages++;
                }
            }
        }
    }
    __host__ __device__ constexpr bool valid() const {
        for (int t = 0; t + 1 < R; ++t)
            for (int c1 = 0; c1 <= t; ++c1)
                for (int r1 = t + 1; r1 < R; ++r1) {
                    if (pg[r1][c1] < 0 || pg[r1][c1] >= npages) return false;
                    for (int c2 = 0; c2 <= t; ++c2)
                        for (int r2 = t + 1; r2 < R; ++r2)
                            if ((r1 != r2 || c1 != c2) && pg[r1][c1] == pg[r2][c2]) return false;
                }
        int bound = 0;
        for (int t = 0; t + 1 < R; ++t) bound = (t + 1) * (R - 1 - t) > bound ? (t + 1) * (R - 1 - t) : bound;
        return npages == bound;
    }
    // the pages of slot r, 4 bits each (c = 0..r-1), for the GEMM's runtime k loop
    __host__ __device__ constexpr uint32_t packed(int r) const {
        uint32_t v = 0;
        for (int c = 0; c < r; ++c) v |= (uint32_t)pg[r][c] << (4 * c);
        return v;
    }
};

template <int N, int NC = 2>
struct RcwpShape {
    static constexpr int R = (N + 7) / 8;
    static constexpr int UNIT = 8 * 8 * 32;              // floats per 8 KB unit
    static constexpr RcwpPages<R> PG{};
    static constexpr int COLS = NC == 3 ? 128 : 256;     // TMEM columns per CTA (NC CTAs per SM)
    static constexpr int WCOLS = COLS / 2;               // per warp (warps h, h+4 share a lane quarter)
    static constexpr size_t SMEM = (size_t)(R * UNIT + 44 * 32) * sizeof(float);
    static_assert(PG.valid(), "page colouring: live pages collide or exceed the bound");
    static_assert(PG.npages * 8 <= WCOLS, "live pages exceed the warp's TMEM columns");
    __host__ __device__ static constexpr int page(int r, int c) { return PG.pg[r][c]; }
    __host__ __device__ static constexpr uint32_t packed(int r) { return PG.packed(r); }
};

// D1: the 8x8 diagonal block is factored by warp 0 alone (results and
// reciprocals through shared memory, one more block barrier) instead of
// redundantly by all eight warps -- ~250 instructions per warp and block fewer;
// the idle warps' issue slots go to the SM's other CTA.
template <int N, int CT, bool D1, bool TM, int NC>
__global__ void __launch_bounds__(256, NC)
potrf_rcwp_kernel(float *__restrict__ A, int32_t *__restrict__ info, int32_t *__restrict__ nfailed,
                  int64_t batch, int64_t cs, const __grid_constant__ RcwpMaps maps) {
    using SH = RcwpShape<N, NC>;
    using RS = RcwShape<N, 1>;                           // stage geometry (rs, bytes, dt)
    constexpr int R = SH::R, UNIT = SH::UNIT;
    constexpr bool TMA = CT == 32;                       // one chunk == one group of 32
    constexpr bool MB = TMA || TM;                       // staged by the copy engine, mbarrier-completed
    extern __shared__ __align__(128) float smf[];         // 128 B: tensor-TMA destinations
    __shared__ uint32_t tmem_base_sh;
    __shared__ __align__(8) uint64_t mbar;

    const int h = threadIdx.x >> 5, q = threadIdx.x & 31;
    const int64_t ngroups = (batch + 31) / 32;
    float *DB = smf + R * UNIT;                          // diagonal block gather [36][32], + inv [8][32]

    if (h == 0) {
        tmem_alloc(&tmem_base_sh, SH::COLS);
        tmem_relinquish();
    }
    if (MB && threadIdx.x == 0) {
        mbar_init(&mbar, 1);
        mbar_fence_init();
    }
    tmem_fence_before();
    __syncthreads();
    tmem_fence_after();
    const uint32_t tb = tmem_base_sh + ((uint32_t)(32 * (h & 3)) << 16) + (uint32_t)((h >> 2) * SH::WCOLS);

    // input of column block c of group g -> units c..R-1: element (i, 8c+w) at
    // [w][i - 8c][q] (RCW's stage layout); lower part only
    auto prefetch = [&](auto c_, int64_t g, const float *gb) {
        constexpr int c = BSP_CI(c_);
        float *stg = smf + (size_t)c * UNIT;
        if constexpr (TMA) {
            if (threadIdx.x == 0) {
                // the units were last written by the generic proxy (RB stores,
                // ordered before this thread by the preceding __syncthreads)
                fence_proxy_async_smem();
                const float *chunk = A + g * (int64_t)(32 * N * N);
                mbar_arrive_expect_tx(&mbar, RS::bytes(c));
#pragma unroll
                for (int w = 0; w < 8; ++w) {
                    const int j = 8 * c + w;
                    if (j < N)
                        bulk_g2s(stg + (w * RS::rs(c) + w) * 32, chunk + (j + j * N) * 32,
                                 (uint32_t)((N - j) * 128), &mbar);
                }
            }
        } else if constexpr (TM) {
            if (threadIdx.x == 0) {
                fence_proxy_async_smem();                // as above: generic RB stores -> async-proxy writes
                const int64_t m0 = g * 32;
                const int x = (int)(m0 % cs), y = (int)((m0 / cs) * (int64_t)(N * N)) + 8 * c;
                constexpr int NW = N - 8 * c < 8 ? N - 8 * c : 8;
                mbar_arrive_expect_tx(&mbar, (uint32_t)(NW * RS::rs(c) * 128));
#pragma unroll
                for (int w = 0; w < NW; ++w)
                    tma_load_2d(stg + w * RS::rs(c) * 32, &maps.m[c], x, y + (8 * c + w) * N, &mbar);
            }
        } else {
            if (g * 32 + 31 < batch && cs % 4 == 0) {
                // full group: element (i, j) of the 32 matrices is one 128-B line;
                // 8 lanes x 16 B per line, 4 lines per warp instruction (RCW's form).
                // Step tt covers r = c + tt/2, w = sub + 4 (tt & 1): two running
                // pointers (w = sub, sub + 4) advanced by 8 rows per r -- no 64-bit
                // products or divisions per copy (the runtime-chunk instances
                // spilled 36-232 B at 128 registers with the per-copy form)
                const int l8 = q & 7, sub = q >> 3;
                const int64_t rstep = 8 * cs;
                const float *pa = gb + (int64_t)(8 * c + h + (8 * c + sub) * N) * cs + 4 * l8;
                const float *pb = pa + (int64_t)(4 * N) * cs;
                float *sa = stg + (sub * RS::rs(c) + h) * 32 + 4 * l8;
                float *sb = sa + 4 * RS::rs(c) * 32;
#pragma unroll
                for (int rr = 0; rr < R - c; ++rr) {
                    const int r = c + rr, i = 8 * r + h;
                    if (i < N) {
                        if (8 * c + sub < N && (r > c || sub <= h)) cp_async16(sa + 8 * rr * 32, pa);
                        if (8 * c + sub + 4 < N && (r > c || sub + 4 <= h)) cp_async16(sb + 8 * rr * 32, pb);
                    }
                    pa += rstep;
                    pb += rstep;
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
                                cp_async4(stg + (w * RS::rs(c) + i - 8 * c) * 32 + q, ad.at(i, 8 * c + w));
                    }
                });
            }
            cp_async_commit();
        }
    };

    int64_t g = blockIdx.x;
    uint32_t par = 0;
    // interleaved base of group g's lane 0 (runtime-chunk form)
    auto gbase = [&](int64_t gg) { return A + ((gg * 32) / cs) * cs * (int64_t)(N * N) + (gg * 32) % cs; };
    if (g < ngroups) prefetch(std::integral_constant<int, 0>{}, g, TMA ? A : gbase(g));

    float acc[R][8];
    for (; g < ngroups; g += gridDim.x) {
        const int64_t gm = g * 32 + q;
        const bool active = gm < batch;
        const Addr<N, CT> ad(A, active ? gm : batch - 1, cs);
        const float *gb = TMA ? A : gbase(g);
        int inf = 0;
        sfor<0, R>([&](auto c_) {
            constexpr int c = BSP_CI(c_);
            // 1. stage(c) has landed (the stage rows of warp h are its own copies
            //    in the cp.async form: a warp-level sync publishes them)
            if constexpr (MB) {
                mbar_wait(&mbar, par);
                par ^= 1u;
            } else {
                cp_async_wait<0>();
                __syncwarp();
            }
            {
                const float *stg = smf + (size_t)c * UNIT + q;
                sfor<c, R>([&](auto r_) {                // (a) A(8r+h, 8c..8c+7)
                    constexpr int r = BSP_CI(r_);
                    const float *src = stg + (8 * (r - c) + h) * 32;
#pragma unroll
                    for (int w = 0; w < 8; ++w)
                        acc[r][w] = (r > c || w <= h) && 8 * c + w < N ? src[w * RS::rs(c) * 32] : 0.0f;
                });
            }
            __syncthreads();                             // B1
            if constexpr (c + 1 < R) prefetch(std::integral_constant<int, c + 1>{}, g, gb);

            // (b) acc(r) -= L(8r+h, 0..8c-1) L(8c..8c+7, 0..8c-1)^T, k ascending.
            //     a operand: 4 columns of page (r, kq / 2) of TMEM; b operand: RB(c)
            //     in pair order (rb_put), one LDS.128 = FFMA2 operand pairs.
            if constexpr (c > 0) {
                const float4 *rb = reinterpret_cast<const float4 *>(smf) + q;
#pragma unroll 1
                for (int kp = 0; kp < c; ++kp) {
                    uint32_t pc[R];
                    sfor<c, R>([&](auto r_) {
                        constexpr int r = BSP_CI(r_);
                        constexpr uint32_t PK = SH::packed(r);
                        pc[r] = tb + ((PK >> (4 * kp)) & 15u) * 8u;
                    });
#pragma unroll
                    for (int hh = 0; hh < 2; ++hh) {
                        const int kq = 2 * kp + hh;
                        float a[R][4];
                        sfor<c, R>([&](auto r_) {
                            constexpr int r = BSP_CI(r_);
                            tmem_ld4(pc[r] + 4u * hh, a[r]);
                        });
                        tmem_wait_ld();
#pragma unroll
                        for (int half = 0; half < 2; ++half) {
                            float4 x[2][2];
#pragma unroll
                            for (int wq = 0; wq < 2; ++wq)
#pragma unroll
                                for (int j = 0; j < 2; ++j) x[wq][j] = rb[((kq * 4 + 2 * half + wq) * 2 + j) * 32];
                            sfor<c, R>([&](auto r_) {
                                constexpr int r = BSP_CI(r_);
#pragma unroll
                                for (int wq = 0; wq < 2; ++wq) {
                                    const int wp = 2 * half + wq;
                                    f_upd2(acc[r][2 * wp], acc[r][2 * wp + 1], a[r][0], x[wq][0].x, x[wq][0].y);
                                    f_upd2(acc[r][2 * wp], acc[r][2 * wp + 1], a[r][1], x[wq][0].z, x[wq][0].w);
                                    f_upd2(acc[r][2 * wp], acc[r][2 * wp + 1], a[r][2], x[wq][1].x, x[wq][1].y);
                                    f_upd2(acc[r][2 * wp], acc[r][2 * wp + 1], a[r][3], x[wq][1].z, x[wq][1].w);
                                }
                            });
                        }
                    }
                }
            }

            // (c) diagonal block: gather rows 8c..8c+7, factor it in every warp
#pragma unroll
            for (int m = 0; m < 8; ++m)
                if (m == h && 8 * c + m < N) {
#pragma unroll
                    for (int w = 0; w <= m; ++w) DB[RS::dt(m, w) * 32 + q] = acc[c][w];
                }
            __syncthreads();                             // B2
            float d[36], inv[8];
            auto factor_diag = [&]() { rcw_factor_diag<N, c>(DB, q, d, inv, inf); };
            if constexpr (D1) {
                if (h == 0) {                            // warp 0 alone; info is warp 0's
                    factor_diag();
#pragma unroll
                    for (int t = 0; t < 36; ++t) DB[t * 32 + q] = d[t];
#pragma unroll
                    for (int k = 0; k < 8; ++k) DB[(36 + k) * 32 + q] = inv[k];
                }
                __syncthreads();                         // B2'
#pragma unroll
                for (int t = 0; t < 36; ++t) d[t] = DB[t * 32 + q];
#pragma unroll
                for (int k = 0; k < 8; ++k) inv[k] = DB[(36 + k) * 32 + q];
            } else {
                factor_diag();
            }
#pragma unroll
            for (int m = 0; m < 8; ++m)
                if (m == h && 8 * c + m < N) {
#pragma unroll
                    for (int w = 0; w <= m; ++w)
                        if (active) st_stream(ad.at(8 * c + m, 8 * c + w), d[RS::dt(m, w)]);
                }

            // (d) triangular solve of my rows below the block; out, page (r, c)
            sfor<c + 1, R>([&](auto r_) {
                constexpr int r = BSP_CI(r_);
#pragma unroll
                for (int k = 0; k < 8; ++k) {
                    if (8 * c + k >= N) break;
                    acc[r][k] = f_mul(acc[r][k], inv[k]);
#pragma unroll
                    for (int j = k + 1; j < 8; ++j) acc[r][j] = f_upd(acc[r][j], acc[r][k], d[RS::dt(j, k)]);
                }
                const int i = 8 * r + h;
                if (active && i < N) {
#pragma unroll
                    for (int w = 0; w < 8; ++w)
                        if (8 * c + w < N) st_stream(ad.at(i, 8 * c + w), acc[r][w]);
                }
                constexpr int pg = SH::page(r, c);
                tmem_st8(tb + (uint32_t)(8 * pg), acc[r]);
            });
            tmem_wait_st();

            __syncthreads();                             // B3: RB(c) no longer read
            if constexpr (c + 1 < R) {
                // publish RB(c+1) = L(8(c+1)+h, 0..8c+7) into units 0..c
                float v[c > 0 ? c : 1][8];
                sfor<0, c>([&](auto kp_) {
                    constexpr int kp = BSP_CI(kp_);
                    constexpr int pg = SH::page(c + 1, kp);
                    tmem_ld8(tb + (uint32_t)(8 * pg), v[kp]);
                });
                if constexpr (c > 0) tmem_wait_ld();
                sfor<0, c>([&](auto kp_) {
                    constexpr int kp = BSP_CI(kp_);
                    rb_put(smf, 2 * kp, h, q, &v[kp][0]);
                    rb_put(smf, 2 * kp + 1, h, q, &v[kp][4]);
                });
                rb_put(smf, 2 * c, h, q, &acc[c + 1][0]);
                rb_put(smf, 2 * c + 1, h, q, &acc[c + 1][4]);
            } else if (g + gridDim.x < ngroups) {
                prefetch(std::integral_constant<int, 0>{}, g + gridDim.x, TMA ? A : gbase(g + gridDim.x));
            }
        });
        if (active && h == 0) info[gm] = inf;
        if (h == 0) count_failures(active && inf != 0, nfailed);
    }

    tmem_fence_before();
    __syncthreads();
    if (h == 0) {
        tmem_fence_after();
        tmem_dealloc(tmem_base_sh, SH::COLS);
    }
}

// One map per column block c: the array as [rows][C] floats (rows = chunks * N^2,
// row stride C*4 B), box 32 x (N - 8c).  False if the layout does not qualify
// (C % 4 != 0 or C < 32: TMA needs 16-B strides and a box within the inner
// dimension) -- the per-thread cp.async staging is used then.
template <int N>
inline bool rcwp_make_maps(const FactorArgs &a, RcwpMaps *mp) {
    constexpr int R = (N + 7) / 8;
    for (int c = 0; c < R; ++c)
        if (!tma2d_make_map(&mp->m[c], a.A, a.batch, a.cstride, N * N, N - 8 * c)) return false;
    return true;
}

template <int N, int CT, bool D1, bool TM, int NC>
cudaError_t launch_rcwp_k(const FactorArgs &a, const RcwpMaps &maps) {
    using SH = RcwpShape<N, NC>;
    auto kern = potrf_rcwp_kernel<N, CT, D1, TM, NC>;
    // NC CTAs per SM own NC * COLS <= 512 TMEM columns: ask for enough shared
    // memory that CTA NC+1 never becomes resident (it would spin in
    // tcgen05.alloc until another exits): 80 KB for two, 57 KB for three
    size_t sm = SH::SMEM;
    const size_t floor_sm = NC == 3 ? (size_t)57 * 1024 : (size_t)80 * 1024;
    if (sm < floor_sm) sm = floor_sm;
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    if (e != cudaSuccess) return e;
    if (const cudaError_t ce = apply_carveout(kern, a.carveout); ce != cudaSuccess) return ce;
    int dev = 0, nsm = 0;
    e = cudaGetDevice(&dev);
    if (e == cudaSuccess) e = cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
    if (e != cudaSuccess) return e;
    const int64_t groups = (a.batch + 31) / 32;
    const int64_t grid = groups < (int64_t)nsm * NC ? groups : (int64_t)nsm * NC;
    kern<<<(unsigned)grid, 256, sm, a.stream>>>(a.A, a.info, a.nfailed, a.batch, a.cstride, maps);
    return cudaGetLastError();
}

// P (the tuning param): bit 0 = D1, bit 1 = three CTAs per SM (128 TMEM columns
// and <= 80 registers each; n <= 40, where a warp's live pages fit 64 columns).
template <int N, int CT, int P>
cudaError_t launch_rcwp(const FactorArgs &a) {
    constexpr bool D1 = (P & 1) != 0;
    constexpr int NC = (P & 2) ? 3 : 2;
    RcwpMaps maps{};
    // 2-D TMA staging where it measured faster than the per-thread cp.async form:
    // n <= 51 (+5-20% at runtime chunks, j24b); at n >= 52 the boxes of up to 64
    // rows of 128 B at a large stride are 2-15% slower.
    if constexpr (CT == 0 && N <= 51) {
        if (rcwp_make_maps<N>(a, &maps)) return launch_rcwp_k<N, CT, D1, true, NC>(a, maps);
    }
    return launch_rcwp_k<N, CT, D1, false, NC>(a, maps);
}

}  // namespace bsp
