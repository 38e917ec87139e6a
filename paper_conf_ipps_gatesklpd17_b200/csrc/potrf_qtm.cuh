// potrf_qtm.cuh -- variant QTM: P threads per matrix, every matrix entirely on
// chip (Tensor Memory + shared memory), for 33 <= n <= 64.
//
// Why a new shape past n = 44.  One matrix at n = 64 is 2080 floats; a B200
// SM holds at most ~1200 floats per thread at 4 warps (registers + 227 KB
// shared + 256 KB TMEM), so one thread per matrix must re-read L from L2
// (variant TILE, 19-25% of HBM bandwidth).  With P = 4 threads per matrix a
// CTA of 128 threads owns 32 matrices and each thread ~520 floats: the whole
// matrix stays on chip, read once from HBM and written once.
//
// Work split (left-looking over 4x4 tiles, the panel order of PTMEM):
//   * tile row rb belongs to thread h = own(rb) of its matrix, reflected so the
//     P threads get balanced work: rb % 2P = 0,1,..,P-1,P-1,..,1,0;
//   * a thread's tile rows are its "slots" s = 0..NS-1 (slot s holds tile row
//     2P*(s/2) + (s even ? h : 2P-1-h)); the off-diagonal tiles of a slot live
//     at slot-uniform TMEM columns (tcgen05.ld/st take a warp-uniform address)
//     or, for the low slots that do not fit, in shared memory;
//   * the input streams in: left-looking reads the original A of tile column CB
//     only when column CB is processed, so each thread cp.async-prefetches its
//     tiles of column CB + 2 into a 3-stage shared buffer while column CB is
//     computed; the slots hold final L tiles only, and diagonal tiles need no
//     slot at all (never read after their column);
//   * column CB: the owner of tile row CB publishes L(CB, 0..CB-1) to a per-
//     matrix row buffer in shared memory (the P threads of a matrix are
//     adjacent lanes of one warp: __syncwarp suffices); every thread then
//     accumulates its tiles (rb, CB), rb >= CB, over PB < CB with
//     acc -= L(rb,PB) L(CB,PB)^T; the owner's diagonal accumulator is
//     broadcast with shuffles, all P threads factor it redundantly (identical
//     bits), and each thread applies the triangular solve to its own tiles.
// Element (m, n) receives its updates in ascending k, one fma each, scaled by
// rcp.rn(L_kk): the same op sequence as every other variant, so the output is
// bitwise identical (pin P8).  Ragged last tile row (n % 4 != 0): padded rows
// are zero (identity on the diagonal), never stored.
#pragma once

#include "common.cuh"
#include "launch.h"
#include "ptx.cuh"
#include "potrf_tmem.cuh"

namespace bsp {

template <int N, int P, int COLS, bool PRE>
struct QtmShape {
    static constexpr int NB = 4;
    static constexpr int TR = (N + NB - 1) / NB;        // tile rows
    static constexpr int MPC = 128 / P;                 // matrices per CTA
    static constexpr int NS = 2 * ((TR + 2 * P - 1) / (2 * P));
    __host__ __device__ static constexpr int rb_of(int h, int s) { return 2 * P * (s / 2) + ((s % 2) == 0 ? h : 2 * P - 1 - h); }
    __host__ __device__ static constexpr int maxrb(int s) {                 // largest real tile row of slot s (-1: none)
        int m = -1;
        for (int h = 0; h < P; ++h)
            if (rb_of(h, s) < TR && rb_of(h, s) > m) m = rb_of(h, s);
        return m;
    }
    __host__ __device__ static constexpr int tiles(int s) { return maxrb(s) > 0 ? maxrb(s) : 0; }   // off-diag columns
    // TMEM placement: greedily from the highest slot down
    __host__ __device__ static constexpr bool in_tmem(int s) {
        int used = 0;
        for (int t = NS - 1; t >= 0; --t) {
            const bool fits = used + tiles(t) * 16 <= COLS;
            if (fits) used += tiles(t) * 16;
            if (t == s) return fits && tiles(t) > 0;
        }
        return false;
    }
    __host__ __device__ static constexpr int tcol(int s) {                  // TMEM column base of slot s
        int c = 0;
        for (int t = NS - 1; t > s; --t)
            if (in_tmem(t)) c += tiles(t) * 16;
        return c;
    }
    __host__ __device__ static constexpr int sbase(int s) {                 // shared-memory tile base of slot s
        int b = 0;
        for (int t = 0; t < s; ++t)
            if (!in_tmem(t)) b += tiles(t);
        return b;
    }
    static constexpr int SMT = sbase(NS);               // shared-memory tiles per thread
    // STREAM mode: input tile columns stream in through STG stages (cp.async, STG-1
    // columns ahead).  PRE mode: the whole input is loaded into the slots up front
    // and the single "stage" holds the input diagonal tiles.
    static constexpr int STG = PRE ? 1 : (COLS == 256 ? 2 : 3);
    // dynamic shared memory, float4 units: slots [t][4][128], stages [stg][s][4][128],
    // row buffer [pb][4][MPC]
    static constexpr int F4_SLOTS = SMT * 4 * 128;
    static constexpr int F4_STAGE = NS * 4 * 128;
    static constexpr int F4_ROWS = (TR > 1 ? TR - 1 : 1) * 4 * MPC;
    static constexpr size_t SMEM = (size_t)(F4_SLOTS + STG * F4_STAGE + F4_ROWS) * 16;
    static_assert(128 % P == 0 && 32 % P == 0, "P must divide a warp");
};

template <int N, int CT, int P, int COLS, bool PRE>
__global__ void __launch_bounds__(128, 1)
potrf_qtm_kernel(float *__restrict__ A, int32_t *__restrict__ info, int32_t *__restrict__ nfailed,
                 int64_t batch, int64_t cs) {
    using SH = QtmShape<N, P, COLS, PRE>;
    constexpr int NB = 4, TR = SH::TR, NS = SH::NS, MPC = SH::MPC;
    constexpr int QB = 1;                               // row-publish tiles per TMEM wait (2+ spills)
    extern __shared__ __align__(16) float4 sm4[];
    __shared__ uint32_t tmem_base_sh;

    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int h = tid % P, q = tid / P;
    const int64_t gm = (int64_t)blockIdx.x * MPC + q;
    const bool active = gm < batch;
    const Addr<N, CT> ad(A, active ? gm : batch - 1, cs);
    float4 *SL = sm4;                                   // [t][4][128]
    float4 *ST = SL + SH::F4_SLOTS;                     // [stg][s][4][128]
    float4 *RW = ST + SH::STG * SH::F4_STAGE;           // [pb][4][MPC]

    if (warp == 0) {
        tmem_alloc(&tmem_base_sh, COLS);
        tmem_relinquish();
    }
    tmem_fence_before();
    __syncthreads();
    tmem_fence_after();
    const uint32_t tbase = tmem_base_sh + ((uint32_t)(32 * (warp & 3)) << 16);

    int rbs[NS];
#pragma unroll
    for (int s = 0; s < NS; ++s) rbs[s] = SH::rb_of(h, s);

    // slot storage: tile (slot s, column cb) -- TMEM (warp-uniform) or shared (per thread)
    auto sl_ld = [&](auto s_, int cb, float *v) {
        constexpr int s = BSP_CI(s_);
        if constexpr (SH::in_tmem(s)) {
            tmem_ld16(tbase + (uint32_t)(SH::tcol(s) + cb * 16), v);
        } else {
            const float4 *p = SL + (size_t)(SH::sbase(s) + cb) * 512 + tid;
#pragma unroll
            for (int e = 0; e < 4; ++e) {
                const float4 x = p[e * 128];
                v[4 * e] = x.x, v[4 * e + 1] = x.y, v[4 * e + 2] = x.z, v[4 * e + 3] = x.w;
            }
        }
    };
    auto sl_st = [&](auto s_, int cb, const float *v, bool mine) {
        constexpr int s = BSP_CI(s_);
        if constexpr (SH::in_tmem(s)) {
            tmem_st16(tbase + (uint32_t)(SH::tcol(s) + cb * 16), v);   // all lanes (uniform)
        } else if (mine) {
            float4 *p = SL + (size_t)(SH::sbase(s) + cb) * 512 + tid;
#pragma unroll
            for (int e = 0; e < 4; ++e) p[e * 128] = make_float4(v[4 * e], v[4 * e + 1], v[4 * e + 2], v[4 * e + 3]);
        }
    };

    // ---- 1. input tile column CB -> stage CB % STG (cp.async, per thread, own rows) ----
    // Left-looking reads the ORIGINAL A of tile column CB only when column CB is
    // processed, so the input streams in STG-1 columns ahead of the arithmetic;
    // TMEM / shared slots hold final L tiles only.  Padded rows (>= N) are zero,
    // with 1 on the diagonal (plain stores; the diagonal tile's upper part is
    // never read).
    auto prefetch = [&](int cb) {
        if (cb < TR) {
            float *stg = reinterpret_cast<float *>(ST + (size_t)(cb % SH::STG) * SH::F4_STAGE);
            sfor<0, NS>([&](auto s_) {
                constexpr int s = BSP_CI(s_);
                const int rb = rbs[s];
                if (SH::maxrb(s) >= cb && rb >= cb && rb < TR) {
                    const float *src = ad.at(rb * NB, cb * NB);        // tile origin
                    float *dst = stg + ((size_t)s * 512 + tid) * 4;
#pragma unroll
                    for (int j = 0; j < NB; ++j)
#pragma unroll
                        for (int i = 0; i < NB; ++i) {
                            const int e = i + j * NB;
                            float *d = dst + (e >> 2) * 512 + (e & 3);
                            if (rb * NB + i < N) {
                                if (rb > cb || i >= j) cp_async4(d, src + (int64_t)(i + j * N) * ad.stride());
                            } else {
                                *d = (rb == cb && i == j) ? 1.0f : 0.0f;
                            }
                        }
                }
            });
        }
        cp_async_commit();
    };
    if constexpr (!PRE) {
#pragma unroll
        for (int c = 0; c < SH::STG - 1; ++c) prefetch(c);
    } else {
        // PRE: every off-diagonal input tile -> its slot, diagonal tiles -> ST[s]
        sfor<0, NS>([&](auto s_) {
            constexpr int s = BSP_CI(s_);
            constexpr int MT = SH::tiles(s);
            const int rb = rbs[s];
            const bool valid = rb < TR;
#pragma unroll 1
            for (int c0 = 0; c0 < MT; c0 += 4) {
                float v[4][16];
#pragma unroll
                for (int u = 0; u < 4; ++u) {
                    const int cb = c0 + u;
                    const float *src = ad.at(rb * NB, cb * NB);
#pragma unroll
                    for (int j = 0; j < NB; ++j)
#pragma unroll
                        for (int i = 0; i < NB; ++i) {
                            const bool ok = valid && cb < rb && rb * NB + i < N;
                            v[u][i + j * NB] = ok ? ld_stream(src + (int64_t)(i + j * N) * ad.stride()) : 0.0f;
                        }
                }
#pragma unroll
                for (int u = 0; u < 4; ++u)
                    if (c0 + u < MT) sl_st(s_, c0 + u, v[u], true);
            }
            if constexpr (SH::maxrb(s) >= 0) {
                float d[16];
                const float *src = ad.at(rb * NB, rb * NB);
#pragma unroll
                for (int j = 0; j < NB; ++j)
#pragma unroll
                    for (int i = 0; i < NB; ++i)
                        d[i + j * NB] = (valid && i >= j && rb * NB + i < N)
                                            ? ld_stream(src + (int64_t)(i + j * N) * ad.stride())
                                            : (i == j ? 1.0f : 0.0f);
                float4 *p = ST + (size_t)s * 512 + tid;
#pragma unroll
                for (int e = 0; e < 4; ++e) p[e * 128] = make_float4(d[4 * e], d[4 * e + 1], d[4 * e + 2], d[4 * e + 3]);
            }
        });
        tmem_wait_st();
    }

    // ---- 2. left-looking over tile columns -------------------------------------------
    int inf = 0;
    float acc[NS][16];
#pragma unroll 1
    for (int CB = 0; CB < TR; ++CB) {
        const int pp = CB % (2 * P);
        const int own = pp < P ? pp : 2 * P - 1 - pp;
        const int sCB = 2 * (CB / (2 * P)) + (pp < P ? 0 : 1);
        const bool owner = h == own;
        if constexpr (!PRE) {
            cp_async_wait<SH::STG - 2>();               // my copies of tile column CB landed
            prefetch(CB + SH::STG - 1);                 // (its stage was consumed at CB - 1)
        }

        // (a) the owner publishes L(CB, 0..CB-1) to the matrix's row buffer (4 tiles
        //     per TMEM wait)
        sfor<0, NS>([&](auto s_) {
            constexpr int s = BSP_CI(s_);
            if (s == sCB) {
#pragma unroll 1
                for (int p0 = 0; p0 < CB; p0 += QB) {
                    float v[QB][16];
#pragma unroll
                    for (int u = 0; u < QB; ++u)
                        if (p0 + u < CB) sl_ld(s_, p0 + u, v[u]);
                    if constexpr (SH::in_tmem(s)) tmem_wait_ld();
                    if (owner) {
#pragma unroll
                        for (int u = 0; u < QB; ++u)
                            if (p0 + u < CB) {
                                float4 *p = RW + (size_t)(p0 + u) * 4 * MPC + q;
#pragma unroll
                                for (int e = 0; e < 4; ++e)
                                    p[e * MPC] = make_float4(v[u][4 * e], v[u][4 * e + 1], v[u][4 * e + 2], v[u][4 * e + 3]);
                            }
                    }
                }
            }
        });
        __syncwarp();

        // (b) accumulators for my tile rows rb >= CB: A(rb, CB) -- from the stage
        //     (STREAM), or from the slots and, for the diagonal tile, ST (PRE)
        if constexpr (PRE) {
            sfor<0, NS>([&](auto s_) {
                constexpr int s = BSP_CI(s_);
                if (SH::maxrb(s) >= CB && CB < SH::tiles(s)) sl_ld(s_, CB, acc[s]);
            });
            tmem_wait_ld();                             // async TMEM loads land before any use
        }
        {
            const float4 *stg = ST + (size_t)(CB % SH::STG) * SH::F4_STAGE;
            sfor<0, NS>([&](auto s_) {
                constexpr int s = BSP_CI(s_);
                if (SH::maxrb(s) >= CB && (!PRE || rbs[s] == CB)) {
                    const float4 *p = stg + (size_t)s * 512 + tid;
#pragma unroll
                    for (int e = 0; e < 4; ++e) {
                        const float4 x = p[e * 128];
                        acc[s][4 * e] = x.x, acc[s][4 * e + 1] = x.y, acc[s][4 * e + 2] = x.z, acc[s][4 * e + 3] = x.w;
                    }
                }
            });
        }

        // (c) acc(rb) -= L(rb, PB) L(CB, PB)^T, PB ascending
#pragma unroll 1
        for (int PB = 0; PB < CB; ++PB) {
            float b[16];
            const float4 *p = RW + (size_t)PB * 4 * MPC + q;
#pragma unroll
            for (int e = 0; e < 4; ++e) {
                const float4 x = p[e * MPC];
                b[4 * e] = x.x, b[4 * e + 1] = x.y, b[4 * e + 2] = x.z, b[4 * e + 3] = x.w;
            }
            float a[NS][16];
            sfor<0, NS>([&](auto s_) {
                constexpr int s = BSP_CI(s_);
                if (SH::maxrb(s) >= CB) sl_ld(s_, PB, a[s]);
            });
            tmem_wait_ld();
            sfor<0, NS>([&](auto s_) {
                constexpr int s = BSP_CI(s_);
                // no per-thread predicate: a lane whose row of this slot is already
                // finished (or padding) updates a dead accumulator -- branch-free,
                // and the slot GEMMs interleave for ILP
                if (SH::maxrb(s) >= CB) {
#pragma unroll
                    for (int k = 0; k < NB; ++k)
#pragma unroll
                        for (int j = 0; j < NB; ++j)
#pragma unroll
                            for (int i = 0; i < NB; ++i)
                                acc[s][i + j * NB] = f_upd(acc[s][i + j * NB], a[s][i + k * NB], b[j + k * NB]);
                }
            });
        }

        // (d) diagonal tile: broadcast the owner's accumulator, factor it everywhere
        float dg[16];
        sfor<0, NS>([&](auto s_) {
            constexpr int s = BSP_CI(s_);
            if (s == sCB) {
#pragma unroll
                for (int e = 0; e < 16; ++e) dg[e] = acc[s][e];
            }
        });
        const int src = (lane & ~(P - 1)) | own;
#pragma unroll
        for (int j = 0; j < NB; ++j)
#pragma unroll
            for (int i = j; i < NB; ++i) dg[i + j * NB] = __shfl_sync(0xffffffffu, dg[i + j * NB], src);
#pragma unroll
        for (int k = 0; k < NB; ++k) {
            const float d = dg[k + k * NB];
            if (CB * NB + k < N) pivot_check(d, CB * NB + k, inf);
            const float sq = f_sqrt(d);
            dg[k + k * NB] = sq;
            const float inv = f_rcp(sq);
#pragma unroll
            for (int i = k + 1; i < NB; ++i) dg[i + k * NB] = f_mul(dg[i + k * NB], inv);
#pragma unroll
            for (int j = k + 1; j < NB; ++j)
#pragma unroll
                for (int i = j; i < NB; ++i) dg[i + j * NB] = f_upd(dg[i + j * NB], dg[i + k * NB], dg[j + k * NB]);
        }
        if (owner && active) {
            float *tb = ad.at(CB * NB, CB * NB);
#pragma unroll
            for (int j = 0; j < NB; ++j)
#pragma unroll
                for (int i = j; i < NB; ++i)
                    if (CB * NB + i < N) st_stream(tb + (int64_t)(i + j * N) * ad.stride(), dg[i + j * NB]);
        }
        float rinv[NB];
#pragma unroll
        for (int k = 0; k < NB; ++k) rinv[k] = f_rcp(dg[k + k * NB]);

        // (e) triangular solve of my tiles below the diagonal; home + HBM
        sfor<0, NS>([&](auto s_) {
            constexpr int s = BSP_CI(s_);
            if (SH::maxrb(s) > CB) {
                const bool mine = rbs[s] > CB && rbs[s] < TR;
                {   // branch-free like (c); only the stores below are predicated
#pragma unroll
                    for (int k = 0; k < NB; ++k) {
#pragma unroll
                        for (int i = 0; i < NB; ++i) acc[s][i + k * NB] = f_mul(acc[s][i + k * NB], rinv[k]);
#pragma unroll
                        for (int j = k + 1; j < NB; ++j)
#pragma unroll
                            for (int i = 0; i < NB; ++i)
                                acc[s][i + j * NB] = f_upd(acc[s][i + j * NB], acc[s][i + k * NB], dg[j + k * NB]);
                    }
                    if (mine && active) {
                        float *tb = ad.at(rbs[s] * NB, CB * NB);
#pragma unroll
                        for (int j = 0; j < NB; ++j)
#pragma unroll
                            for (int i = 0; i < NB; ++i)
                                if (rbs[s] * NB + i < N) st_stream(tb + (int64_t)(i + j * N) * ad.stride(), acc[s][i + j * NB]);
                    }
                }
                sl_st(s_, CB, acc[s], mine);
            }
        });
        tmem_wait_st();
        __syncwarp();                                   // row buffer free for the next column
    }
    if constexpr (!PRE) cp_async_wait<0>();
    if (active && h == 0) info[gm] = inf;
    count_failures(active && h == 0 && inf != 0, nfailed);

    tmem_fence_before();
    __syncthreads();
    if (warp == 0) {
        tmem_fence_after();
        tmem_dealloc(tmem_base_sh, COLS);
    }
}

template <int N, int CT, int P, int COLS, bool PRE>
cudaError_t launch_qtm(const FactorArgs &a) {
    using SH = QtmShape<N, P, COLS, PRE>;
    // 512 TMEM columns: one CTA per SM (request enough shared memory that a second
    // one never waits in tcgen05.alloc); 256: two.
    size_t sm = SH::SMEM;
    if constexpr (COLS == 512)
        if (sm < (size_t)116 * 1024) sm = (size_t)116 * 1024;
    auto kern = potrf_qtm_kernel<N, CT, P, COLS, PRE>;
    const cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    if (e != cudaSuccess) return e;
    if (const cudaError_t ce = apply_carveout(kern, a.carveout); ce != cudaSuccess) return ce;
    kern<<<grid_for(a.batch, SH::MPC), 128, sm, a.stream>>>(a.A, a.info, a.nfailed, a.batch, a.cstride);
    return cudaGetLastError();
}

}  // namespace bsp
