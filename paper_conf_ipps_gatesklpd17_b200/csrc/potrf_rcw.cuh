// potrf_rcw.cuh -- variant RCW ("row-cyclic warps"): eight warps share 32
// matrices, lane = matrix, warp h owns the rows i = 8r + h (r = 0..R-1) of all
// 32; the factor stays on chip in Tensor Memory.  For 33 <= n <= 64 (SURVEY
// §8(f) f2), where one thread per matrix no longer fits on chip.
//
// Why this shape.  At n = 64 the lower triangle is 2080 floats; 32 matrices
// need 266 KB, which only TMEM (256 KB) + shared memory can hold -- one CTA
// per SM.  QTM (P = 4 threads per matrix inside one warp) gets there with 4
// warps per SM, rows of different length in one warp instruction (dead lanes:
// 28% of its FFMAs) and a per-column publish through TMEM round trips.  Here:
//   * a warp instruction touches the SAME element (i, j) of 32 consecutive
//     matrices: every global access is one 128-B line, and every lane of a
//     warp does the same work (no dead lanes, uniform branches only);
//   * 8 warps per CTA (2 per scheduler) instead of 4;
//   * warp h's rows live in TMEM (lane quarter h % 4, column half h / 4):
//     slot r holds L(8r+h, 0..8r-1) at columns 4r(r-1) .. -- 224 columns at
//     n = 64, so the whole factor fits in one 512-column allocation;
//   * left-looking over 8-wide column blocks c: the rows 8c..8c+7 of L (the
//     "b" operand every warp needs) are published to a row buffer RB(c) in
//     shared memory by their owners while those owners stream them out of TMEM
//     for their own GEMM in block c-1 (no extra TMEM reads);
//   * the input streams in one block ahead.  Shared memory is two halves of R
//     units of 8 KB; block t (counted over all groups a persistent CTA
//     processes) uses half t % 2: RB(c) in units 0..c-1 and the input stage of
//     block c in units c..R-1, while the other half receives RB(c+1) and
//     stage(c+1) -- 16 units at any time (RB grows as the stage shrinks).  The
//     stage is column-run ordered, [w][i - 8c][lane], so for chunk 32 (one
//     chunk = one group) each column j of the block is ONE contiguous run of
//     (n - j) * 128 B: one TMA bulk copy per column (one mbarrier per half);
//     other chunks use per-thread cp.async; results go out as coalesced
//     per-thread streaming stores (one 128-B line per warp instruction);
//   * persistent CTAs: the last block of a group prefetches block 0 of the
//     CTA's next group, so loads never drain between groups.
// Op order per element (i, j): fma with k = 0, 1, ..., j-1 ascending (GEMM over
// k < 8c, then the in-block triangular updates), then mul by rcp.rn(L_jj) --
// the Fig. 9 sequence of every other variant, so the output is bitwise
// identical to REG/PTMEM/QTM (pin P8).
#pragma once

#include "common.cuh"
#include "launch.h"
#include "ptx.cuh"
#include "potrf_tmem.cuh"

namespace bsp {

__device__ __forceinline__ void tmem_st8(uint32_t taddr, const float *v) {
    asm volatile("tcgen05.st.sync.aligned.32x32b.x8.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"r"(taddr),
                 "f"(v[0]), "f"(v[1]), "f"(v[2]), "f"(v[3]), "f"(v[4]), "f"(v[5]), "f"(v[6]), "f"(v[7])
                 : "memory");
}

// Row buffer, pair order: the four values v[kk] = L(8c+w, 4kq+kk) of row w are
// stored so that float4 ((kq*4 + w/2)*2 + kk/2) of lane q holds
// (L(w even, 2j), L(w odd, 2j), L(w even, 2j+1), L(w odd, 2j+1)), j = kk/2:
// the reader's LDS.128 gives FFMA2 operand pairs over adjacent rows w, w+1.
__device__ __forceinline__ void rb_put(float *rb, int kq, int w, int q, const float *v) {
#pragma unroll
    for (int kk = 0; kk < 4; ++kk)
        rb[4 * (((kq * 4 + (w >> 1)) * 2 + (kk >> 1)) * 32 + q) + (kk & 1) * 2 + (w & 1)] = v[kk];
}

template <int N, int NCTA>
struct RcwShape {
    static constexpr int W = 8;                          // column-block width = warps per CTA
    static constexpr int R = (N + W - 1) / W;            // row slots per warp (= column blocks)
    static constexpr int COLS = NCTA == 1 ? 512 : 256;   // TMEM columns per CTA
    static constexpr int HALF = COLS / 2;                // per warp (warps h and h+4 share lanes)
    static constexpr int UNIT = W * W * 32;              // floats per 8 KB unit
    __host__ __device__ static constexpr int off(int r) { return 4 * r * (r - 1); }
    __host__ __device__ static constexpr int dt(int m, int k) { return m * (m + 1) / 2 + k; }
    __host__ __device__ static constexpr int rs(int c) { return N - W * c; }   // stage row stride
    __host__ __device__ static constexpr uint32_t bytes(int c) {                // TMA bytes of block c
        uint32_t b = 0;
        for (int w = 0; w < W; ++w)
            if (W * c + w < N) b += (uint32_t)(N - W * c - w) * 128u;
        return b;
    }
    static constexpr size_t SMEM = (size_t)(2 * R * UNIT + 36 * 32) * sizeof(float);
    static_assert(off(R) <= HALF, "slots exceed the TMEM column budget");
};

// The 8x8 diagonal block of column block c, factored in registers from its
// shared-memory gather DB ([36][32], lane q): d (packed lower, dt order) and
// inv = 1 / diag.  Fig. 9's op order; the sqrt / reciprocal use the branch-free
// fast forms (common.cuh: bitwise equal to the intrinsics wherever their `ok`
// holds, checked exhaustively over all 2^32 inputs), so the block is one basic
// block; a lane outside their range (a failed pivot, extreme exponents) redoes
// the block with the intrinsics -- same bits, info decided by the exact pass.
// (+1-5% for RCWP at n = 49..64, where the redundant diagonal work of every
// warp sits on the critical path, j29.)
template <int N, int C>
__device__ __forceinline__ void rcw_factor_diag(const float *DB, int q, float *d, float *inv, int &inf) {
    using SH = RcwShape<N, 1>;
    auto pass = [&](auto fast_) -> bool {
        constexpr bool FAST = decltype(fast_)::value;
        bool ok = true;
#pragma unroll
        for (int t = 0; t < 36; ++t) d[t] = DB[t * 32 + q];
#pragma unroll
        for (int k = 0; k < 8; ++k) {
            if (8 * C + k >= N) break;
            const float p = d[SH::dt(k, k)];
            pivot_check(p, 8 * C + k, inf);
            const float s = FAST ? f_sqrt_fast(p, ok) : f_sqrt(p);
            d[SH::dt(k, k)] = s;
            inv[k] = FAST ? f_rcp_fast(s, ok) : f_rcp(s);
#pragma unroll
            for (int m = k + 1; m < 8; ++m) d[SH::dt(m, k)] = f_mul(d[SH::dt(m, k)], inv[k]);
#pragma unroll
            for (int j = k + 1; j < 8; ++j)
#pragma unroll
                for (int m = j; m < 8; ++m) d[SH::dt(m, j)] = f_upd(d[SH::dt(m, j)], d[SH::dt(m, k)], d[SH::dt(j, k)]);
        }
        return ok;
    };
    const int inf0 = inf;
    if (!pass(std::true_type{})) {
        inf = inf0;
        pass(std::false_type{});
    }
}


template <int N, int CT, int NCTA>
__global__ void __launch_bounds__(256, NCTA)
potrf_rcw_kernel(float *__restrict__ A, int32_t *__restrict__ info, int32_t *__restrict__ nfailed,
                 int64_t batch, int64_t cs) {
    using SH = RcwShape<N, NCTA>;
    constexpr int R = SH::R, UNIT = SH::UNIT;
    constexpr bool TMA = CT == 32;                       // one chunk == one group of 32
    extern __shared__ __align__(16) float smf[];
    __shared__ uint32_t tmem_base_sh;
    __shared__ __align__(8) uint64_t mbar[2];

    const int h = threadIdx.x >> 5, q = threadIdx.x & 31;
    const int64_t ngroups = (batch + 31) / 32;
    float *DB = smf + 2 * R * UNIT;                      // diagonal block gather [36][32]
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
    const uint32_t tb = tmem_base_sh + ((uint32_t)(32 * (h & 3)) << 16) + (uint32_t)((h >> 2) * SH::HALF);

    // input of column block c of group g -> stage units c..R-1 of `half`:
    // element (i, 8c+w) at [w][i - 8c][q]; lower part only
    auto prefetch = [&](auto c_, int64_t g, int half) {
        constexpr int c = BSP_CI(c_);
        float *stg = unit(half, c);
        if constexpr (TMA) {
            if (threadIdx.x == 0) {
                // the stage units were last written by the generic proxy (row
                // buffer stores); the preceding __syncthreads orders the other
                // threads' writes before this thread, the fence orders them
                // before the async-proxy writes of the bulk copies
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
        } else if (g * 32 + 31 < batch && cs % 4 == 0) {
            // full group, 16-B aligned lines: element (i, j) of the 32 matrices is
            // one 128-B line (a group never straddles a chunk); 8 lanes x 16 B per
            // line, 4 lines per warp instruction -- 8x fewer copy instructions and
            // addresses than one 4-byte copy per element (round 2)
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
            cp_async_commit();
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
            cp_async_commit();
        }
    };
    int64_t g = blockIdx.x;
    int ph = 0;                                          // half of the group's block 0
    uint32_t par = 0;                                    // mbarrier phase bits, one per half
    if (g < ngroups) prefetch(std::integral_constant<int, 0>{}, g, ph);

    float acc[R][8];
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
                cp_async_wait<0>();                      // my stage(c) copies landed
            }
            __syncthreads();                             // RB(c) published; old units free
            if constexpr (c + 1 < R) prefetch(std::integral_constant<int, c + 1>{}, g, half ^ 1);
            else if (g + gridDim.x < ngroups) prefetch(std::integral_constant<int, 0>{}, g + gridDim.x, half ^ 1);
            const float *stg = unit(half, c) + q;

            // (a) accumulators of my live rows = A(8r+h, 8c..8c+7)
            sfor<c, R>([&](auto r_) {
                constexpr int r = BSP_CI(r_);
                const float *src = stg + (8 * (r - c) + h) * 32;
#pragma unroll
                for (int w = 0; w < 8; ++w)
                    acc[r][w] = (r > c || w <= h) && 8 * c + w < N ? src[w * SH::rs(c) * 32] : 0.0f;
            });

            // (b) acc(r) -= L(8r+h, 0..8c-1) L(8c..8c+7, 0..8c-1)^T, k ascending; the
            //     rows of block c+1 (my slot c+1) are published to RB(c+1) on the way.
            //     RB holds the b operand in pair order (rb_put) so that one LDS.128
            //     yields (b[w][k], b[w+1][k]) register pairs for FFMA2 (f_upd2): two
            //     columns w, w+1 of a row per instruction, the same bits as f_upd.
            if constexpr (c > 0) {
                const float4 *rb = reinterpret_cast<const float4 *>(unit(half, 0)) + q;
                float *rbn = unit(half ^ 1, 0);
                // b operand of k-chunk kq: x[wp][j] = k 4kq+2j, 4kq+2j+1 of rows 2wp, 2wp+1
                auto ldb = [&](float4 (&x)[4][2], int kq) {
#pragma unroll
                    for (int wp = 0; wp < 4; ++wp)
#pragma unroll
                        for (int j = 0; j < 2; ++j) x[wp][j] = rb[((kq * 4 + wp) * 2 + j) * 32];
                };
                auto step = [&](const float4 (&x)[4][2], int kq) {
                    float a[R][4];
                    sfor<c, R>([&](auto r_) {
                        constexpr int r = BSP_CI(r_);
                        tmem_ld4(tb + (uint32_t)(SH::off(r) + 4 * kq), a[r]);
                    });
                    tmem_wait_ld();
                    if constexpr (c + 1 < R) rb_put(rbn, kq, h, q, a[c + 1]);
                    sfor<c, R>([&](auto r_) {
                        constexpr int r = BSP_CI(r_);
#pragma unroll
                        for (int wp = 0; wp < 4; ++wp) {
                            f_upd2(acc[r][2 * wp], acc[r][2 * wp + 1], a[r][0], x[wp][0].x, x[wp][0].y);
                            f_upd2(acc[r][2 * wp], acc[r][2 * wp + 1], a[r][1], x[wp][0].z, x[wp][0].w);
                            f_upd2(acc[r][2 * wp], acc[r][2 * wp + 1], a[r][2], x[wp][1].x, x[wp][1].y);
                            f_upd2(acc[r][2 * wp], acc[r][2 * wp + 1], a[r][3], x[wp][1].z, x[wp][1].w);
                        }
                    });
                };
#pragma unroll 1
                for (int kq = 0; kq < 2 * c; ++kq) {
                    float4 x[4][2];
                    ldb(x, kq);
                    step(x, kq);
                }
            }

            // (c) diagonal block: gather rows 8c..8c+7, factor it in every warp (identical bits)
#pragma unroll
            for (int m = 0; m < 8; ++m)
                if (m == h && 8 * c + m < N) {
#pragma unroll
                    for (int w = 0; w <= m; ++w) DB[SH::dt(m, w) * 32 + q] = acc[c][w];
                }
            __syncthreads();
            float d[36], inv[8];
            rcw_factor_diag<N, c>(DB, q, d, inv, inf);
#pragma unroll
            for (int m = 0; m < 8; ++m)
                if (m == h && 8 * c + m < N) {
#pragma unroll
                    for (int w = 0; w <= m; ++w)
                        if (active) st_stream(ad.at(8 * c + m, 8 * c + w), d[SH::dt(m, w)]);
                }

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
                    rb_put(unit(half ^ 1, 0), 2 * c, h, q, &acc[r][0]);
                    rb_put(unit(half ^ 1, 0), 2 * c + 1, h, q, &acc[r][4]);
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
        tmem_dealloc(tmem_base_sh, SH::COLS);
    }
}

template <int N, int CT, int NCTA>
cudaError_t launch_rcw(const FactorArgs &a) {
    using SH = RcwShape<N, NCTA>;
    auto kern = potrf_rcw_kernel<N, CT, NCTA>;
    // one CTA per SM must own all 512 TMEM columns: ask for enough shared memory
    // that a second CTA never becomes resident (it would spin in tcgen05.alloc)
    size_t sm = SH::SMEM;
    if constexpr (NCTA == 1)
        if (sm < (size_t)116 * 1024) sm = (size_t)116 * 1024;
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    if (e != cudaSuccess) return e;
    int dev = 0, nsm = 0;                                // persistent grid: NCTA CTAs per SM
    e = cudaGetDevice(&dev);                             // (queried per call: reentrant, any device)
    if (e == cudaSuccess) e = cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
    if (e != cudaSuccess) return e;
    const int64_t groups = (a.batch + 31) / 32;
    const int64_t grid = groups < (int64_t)nsm * NCTA ? groups : (int64_t)nsm * NCTA;
    if (const cudaError_t ce = apply_carveout(kern, a.carveout); ce != cudaSuccess) return ce;
    kern<<<(unsigned)grid, 256, sm, a.stream>>>(a.A, a.info, a.nfailed, a.batch, a.cstride);
    return cudaGetLastError();
}

}  // namespace bsp
