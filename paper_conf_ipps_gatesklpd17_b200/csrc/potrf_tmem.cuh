// potrf_tmem.cuh -- variant PTMEM: the PANEL split with Tensor Memory (TMEM) as
// a third on-chip storage tier, for 24 <= n <= 32.
//
// At n = 32 one matrix's lower triangle is 528 floats.  With registers and
// shared memory alone (PANEL variant) a B200 SM holds 4 warps of matrices
// (50 KB of panel per warp), i.e. ONE warp per scheduler, and ncu shows the
// kernel issue-latency bound (issue active ~32%, "wait" stalls).  TMEM --
// 256 KB per SM, 128 lanes x 512 columns of 32-bit, otherwise idle in a
// kernel without MMAs -- is thread-private per lane when each warp touches
// only its own 32-lane sub-partition (warp w <-> lanes 32*(w%4)..+31), and is
// addressed by a runtime column index (unlike registers).  So:
//   * a CTA is 4 warps (one per TMEM sub-partition) and allocates 256 TMEM
//     columns; two CTAs -> 8 warps per SM (2 per scheduler);
//   * the panel's first CS columns (as 4x4 tiles, tile-major, 16 columns per
//     tile, <= 256 columns) live in TMEM: one tcgen05.ld/st .32x32b.x16 moves
//     a whole tile of a thread's matrix;
//   * the remaining panel columns CS..S-1 live in shared memory (TMA bulk
//     staged, one cp.async.bulk per column run of the warp's 32-matrix chunk);
//   * the trailing (N-S) triangle lives in registers.
// Arithmetic and op order are exactly the PANEL variant's (rolled left-looking
// 4x4 tile loop over the panel, rolled SYRK, unrolled register tail), hence
// bitwise identical to every other variant (pin P8).
#pragma once

#include "common.cuh"
#include "launch.h"
#include "potrs.cuh"
#include "ptx.cuh"
#include "tma2d.cuh"

namespace bsp {

// ---- tcgen05 TMEM primitives (warp-collective, .sync.aligned) --------------
__device__ __forceinline__ void tmem_alloc(uint32_t *dst_smem, uint32_t ncols) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(dst_smem)),
                 "r"(ncols)
                 : "memory");
}
__device__ __forceinline__ void tmem_relinquish() {
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
}
__device__ __forceinline__ void tmem_dealloc(uint32_t taddr, uint32_t ncols) {
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(taddr), "r"(ncols) : "memory");
}
__device__ __forceinline__ void tmem_fence_before() {
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
}
__device__ __forceinline__ void tmem_fence_after() {
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
}
__device__ __forceinline__ void tmem_wait_ld() { asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory"); }
__device__ __forceinline__ void tmem_wait_st() { asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory"); }

__device__ __forceinline__ void tmem_ld16(uint32_t taddr, float *v) {
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
        : "=f"(v[0]), "=f"(v[1]), "=f"(v[2]), "=f"(v[3]), "=f"(v[4]), "=f"(v[5]), "=f"(v[6]), "=f"(v[7]),
          "=f"(v[8]), "=f"(v[9]), "=f"(v[10]), "=f"(v[11]), "=f"(v[12]), "=f"(v[13]), "=f"(v[14]), "=f"(v[15])
        : "r"(taddr)
        : "memory");
}
__device__ __forceinline__ void tmem_ld4(uint32_t taddr, float *v) {
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x4.b32 {%0,%1,%2,%3}, [%4];"
                 : "=f"(v[0]), "=f"(v[1]), "=f"(v[2]), "=f"(v[3])
                 : "r"(taddr)
                 : "memory");
}
__device__ __forceinline__ void tmem_st16(uint32_t taddr, const float *v) {
    asm volatile(
        "tcgen05.st.sync.aligned.32x32b.x16.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16};" ::"r"(
            taddr),
        "f"(v[0]), "f"(v[1]), "f"(v[2]), "f"(v[3]), "f"(v[4]), "f"(v[5]), "f"(v[6]), "f"(v[7]),
        "f"(v[8]), "f"(v[9]), "f"(v[10]), "f"(v[11]), "f"(v[12]), "f"(v[13]), "f"(v[14]), "f"(v[15])
        : "memory");
}

// ---- shape ------------------------------------------------------------------
template <int N, int S>
struct TmemShape {
    static constexpr int NB = 4;
    static constexpr int TR = (N + NB - 1) / NB;   // tile rows
    static constexpr int TC = S / NB;              // panel tile columns
    // TMEM columns per CTA: 256 (two CTAs = 8 warps per SM) up to n = 32; all
    // 512 (one CTA = 4 warps per SM) for 33 <= n <= 44, where a matrix no
    // longer fits twice over in registers + shared memory + half the TMEM.
    static constexpr int COLS = N > 32 ? 512 : 256;
    static constexpr int tiles_in(int tc) { return tc * TR - tc * (tc - 1) / 2; }
    static constexpr int pick_ct() {               // panel tile columns kept in TMEM
        int c = 0;
        while (c < TC && tiles_in(c + 1) * 16 <= COLS) ++c;
        return c;
    }
    static constexpr int CTM = pick_ct();
    static constexpr int CS = CTM * NB;            // panel columns in TMEM
    static constexpr int NT = N - S;
    static constexpr int T = NT * (NT + 1) / 2;
    // shared-memory part: columns CS..S-1, lower-packed
    static constexpr int PSM = (S * N - S * (S - 1) / 2) - (CS * N - CS * (CS - 1) / 2);
    static_assert(S % NB == 0, "panel width must be a multiple of 4");
    static_assert(CTM >= 1, "TMEM must hold at least one tile column");
};

// Runtime-chunk staging of the shared-memory panel columns CS..S-1 by 2-D TMA
// (round 2, tma2d.cuh): one box of 32 matrices x (N - c) rows per column c,
// one tensor map per column (its box height).
template <int K>
struct PtmemMaps {
    CUtensorMap m[K > 0 ? K : 1];
};


// SOLVE: fused SPOSV with one right-hand side: B (n x 1 per
// matrix, interleaved like A) is solved while every column of L is still on
// chip -- forward substitution rides along the panel tile loop and the
// register tail, backward substitution reads L back from TMEM / shared memory /
// registers.  x lives in shared memory ([i][lane], after the panel part).  Op
// order is potrs.cuh's, so X is bitwise identical to factor-then-SPOTRS.
// FILLT: TMEM tiles loaded per warp-synchronised batch of the fill (0 = the
// default: 5 with TMA staging, 1 with per-thread cp.async); a tuning axis
// (bspotrf_tuning.staging 3 = TMA with 12), see the fill below.
template <int N, int CT, int S, bool TMA, bool SOLVE = false, int FILLT = 0, bool TM = false>
__global__ void __launch_bounds__(128, TmemShape<N, S>::COLS == 256 ? 2 : 1)
potrf_ptmem_kernel(float *__restrict__ A, int32_t *__restrict__ info,
                   int32_t *__restrict__ nfailed, int64_t batch, int64_t cs,
                   const __grid_constant__ PtmemMaps<S - TmemShape<N, S>::CS> maps,
                   float *__restrict__ Bx = nullptr) {
    using SH = TmemShape<N, S>;
    constexpr int NB = 4, TR = SH::TR, TC = SH::TC, CTM = SH::CTM, CS = SH::CS;
    constexpr int NT = SH::NT, T = SH::T, PSM = SH::PSM;
    constexpr int SB0 = CS * N - CS * (CS - 1) / 2;   // pslot of (CS, CS)
    static_assert(!TMA || CT == 32, "TMA staging here needs chunk 32 (one chunk per warp)");

    extern __shared__ __align__(128) float smem[];
    __shared__ uint32_t tmem_base_sh;
    __shared__ __align__(8) uint64_t bars[4];

    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int64_t gid = (int64_t)blockIdx.x * 128 + threadIdx.x;
    const bool active = gid < batch;
    const int64_t g = active ? gid : batch - 1;
    const Addr<N, CT> ad(A, g, cs);
    constexpr int QW = (PSM > 0 ? PSM : 1) + (SOLVE ? N : 0);      // floats per lane per warp
    float *Q = smem + (size_t)warp * QW * 32 + lane;                   // lane-private view
    float *X = Q + (PSM > 0 ? PSM : 1) * 32;                           // x_i at X[i * 32]
    auto qs = [&](int m, int c) { return (c * N - (c * (c - 1)) / 2 + (m - c)) - SB0; };

    // ---- TMEM: warp 0 allocates 256 columns for the CTA ---------------------
    if (warp == 0) {
        tmem_alloc(&tmem_base_sh, SH::COLS);
        tmem_relinquish();
    }
    if constexpr ((TMA || TM) && PSM > 0) {
        if (lane == 0) {
            mbar_init(&bars[warp], 1);
            mbar_fence_init();
        }
    }
    tmem_fence_before();
    __syncthreads();
    tmem_fence_after();
    const uint32_t tbase = tmem_base_sh + ((uint32_t)(32 * (warp & 3)) << 16);
    auto tidx = [&](int rb, int pb) { return (uint32_t)(pb * TR - pb * (pb - 1) / 2 + (rb - pb)) * 16u; };

    // ---- shared-memory part of the panel: TMA bulk (chunk 32) or cp.async --
    if constexpr (PSM > 0) {
        if constexpr (TMA) {
            if (lane == 0) {
                int64_t q = ((int64_t)blockIdx.x * 128 + warp * 32) / 32;
                const int64_t qmax = (batch - 1) / 32;
                if (q > qmax) q = qmax;          // idle warp past the end: a valid chunk
                mbar_arrive_expect_tx(&bars[warp], (uint32_t)(PSM * 32 * 4));
                const float *chunk = A + q * 32 * (N * N);
#pragma unroll 1
                for (int c = CS; c < S; ++c)
                    bulk_g2s(smem + (size_t)warp * QW * 32 + qs(c, c) * 32, chunk + (c + c * N) * 32,
                             (uint32_t)((N - c) * 32 * 4), &bars[warp]);
            }
        } else if constexpr (TM) {
            if (lane == 0) {
                int64_t m0 = (int64_t)blockIdx.x * 128 + warp * 32;
                if (m0 >= batch) m0 = (batch - 1) / 32 * 32;   // idle warp past the end: a valid group
                const int x = (int)(m0 % cs), y = (int)((m0 / cs) * (int64_t)(N * N));
                mbar_arrive_expect_tx(&bars[warp], (uint32_t)(PSM * 32 * 4));
#pragma unroll 1
                for (int c = CS; c < S; ++c)
                    tma_load_2d(smem + (size_t)warp * QW * 32 + qs(c, c) * 32, &maps.m[c - CS], x, y + c + c * N,
                                &bars[warp]);
            }
        } else {
#pragma unroll 1
            for (int c = CS; c < S; ++c)
#pragma unroll 4
                for (int m = c; m < N; ++m) cp_async4(Q + qs(m, c) * 32, ad.at(m, c));
        }
    }

    // ---- right-hand side -> shared memory (fused solve) ----------------------
    if constexpr (SOLVE) {
        const RectAddr<N, CT> ba(Bx, g, cs, 1);
#pragma unroll 4
        for (int i = 0; i < N; ++i) X[i * 32] = ld_stream(ba.at(i, 0));
    }

    // ---- trailing triangle -> registers ------------------------------------
    float r[T];
#pragma unroll
    for (int n = S; n < N; ++n)
#pragma unroll
        for (int m = n; m < N; ++m) r[tri<NT>(m - S, n - S)] = ld_stream(ad.at(m, n));

    // ---- TMEM part of the panel: global -> registers -> tcgen05.st ---------
    sfor<0, CTM>([&](auto pb_) {
        constexpr int pb = BSP_CI(pb_);
        sfor<pb, TR>([&](auto rb_) {
            constexpr int rb = BSP_CI(rb_);
            float v[16];
#pragma unroll
            for (int j = 0; j < NB; ++j)
#pragma unroll
                for (int i = 0; i < NB; ++i) {
                    const int m = rb * NB + i, c = pb * NB + j;
                    const bool ok = m < N && (rb > pb || i >= j);
                    v[i + j * NB] = ok ? ld_stream(ad.at(m, c)) : 0.0f;
                }
            tmem_st16(tbase + tidx(rb, pb), v);
            // a warp barrier every FILL tiles keeps ptxas from hoisting every
            // tile's loads above the first tcgen05.st: FILL*16 loads in flight
            // (plus the register triangle's), no spills (round 2: n = 25, 29,
            // 31 spilled 12-216 B, n = 33..42 up to 304 B, at 255 registers)
            // (TMA staging: 5 tiles, or 12 as the FILLT tuning axis -- more bytes
            // in flight per warp at 8 warps/SM: n = 29-31 +1-3.5%, n = 26/28 -7%:
            // the table picks per n, profiles/r02/ptmem_fill.md; both spill-free.
            // Per-thread cp.async: 1, its runtime-stride address arithmetic
            // needs the registers.)
            constexpr int idx = pb * TR - pb * (pb - 1) / 2 + (rb - pb);
            constexpr int FILL = FILLT ? FILLT : (TMA ? 5 : 1);
            if constexpr ((idx + 1) % FILL == 0) __syncwarp();
        });
    });
    tmem_wait_st();
    if constexpr (PSM > 0) {
        if constexpr (TMA || TM) mbar_wait(&bars[warp], 0);
        else cp_async_wait_all();
    }

    int inf = 0;
    const Addr<N, CT> ads = ad.opaque();           // store addresses (see Addr::opaque)
    // smem tile loader (packed columns CS..S-1); rows >= N read as 0
    auto load_tile_smem = [&](int rb, int pb, float *t, bool lower_only) {
#pragma unroll
        for (int j = 0; j < NB; ++j)
#pragma unroll
            for (int i = 0; i < NB; ++i) {
                const int m = rb * NB + i, c = pb * NB + j;
                const bool ok = m < N && (!lower_only || i >= j);
                t[i + j * NB] = ok ? Q[qs(m, c) * 32] : 0.0f;
            }
    };
    // acc -= a * b^T restricted to the lower part when DIAG
    auto gemm = [&](float *acc, const float *a, const float *b, auto diag_) {
        constexpr bool DIAG = decltype(diag_)::value;
#pragma unroll
        for (int k = 0; k < NB; ++k)
#pragma unroll
            for (int j = 0; j < NB; ++j)
#pragma unroll
                for (int i = 0; i < NB; ++i)
                    if (!DIAG || i >= j) acc[i + j * NB] = f_upd(acc[i + j * NB], a[i + k * NB], b[j + k * NB]);
    };
    // store a final tile of panel tile column CB to its on-chip home and to global
    auto put_tile = [&](int rb, const float *acc, auto cb_, auto diag_) {
        constexpr int CB = decltype(cb_)::value;
        constexpr bool DIAG = decltype(diag_)::value;
        if constexpr (CB < CTM) {
            tmem_st16(tbase + tidx(rb, CB), acc);
        } else {
#pragma unroll
            for (int j = 0; j < NB; ++j)
#pragma unroll
                for (int i = 0; i < NB; ++i) {
                    const int m = rb * NB + i;
                    if (m < N && (!DIAG || i >= j)) Q[qs(m, CB * NB + j) * 32] = acc[i + j * NB];
                }
        }
        if (active) {
            float *tb = ads.at(rb * NB, CB * NB);
#pragma unroll
            for (int j = 0; j < NB; ++j)
#pragma unroll
                for (int i = 0; i < NB; ++i)
                    if (rb * NB + i < N && (!DIAG || i >= j))
                        st_stream(tb + (int64_t)(i + j * N) * ads.stride(), acc[i + j * NB]);
        }
    };

    // ---- 1. panel: left-looking over 4x4 tiles; tile columns unrolled at
    //         compile time, tile rows rolled --------------------------------------
    sfor<0, TC>([&](auto cb_) {
        constexpr int CB = BSP_CI(cb_);
        using TRUE_ = std::integral_constant<bool, true>;
        using FALSE_ = std::integral_constant<bool, false>;
        // (a) diagonal tile (CB, CB): SYRK from the tiles to its left, then spotrf_tile
        float dg[16];
        if constexpr (CB < CTM) tmem_ld16(tbase + tidx(CB, CB), dg);
        else load_tile_smem(CB, CB, dg, true);
        sfor<0, CB>([&](auto pb_) {
            constexpr int PB = BSP_CI(pb_);
            float a[16];
            if constexpr (PB < CTM) tmem_ld16(tbase + tidx(CB, PB), a);
            else load_tile_smem(CB, PB, a, false);
            tmem_wait_ld();
            gemm(dg, a, a, TRUE_{});
        });
        tmem_wait_ld();
#pragma unroll
        for (int k = 0; k < NB; ++k) {
            const float d = dg[k + k * NB];
            pivot_check(d, CB * NB + k, inf);
            const float s = f_sqrt_pos(d);
            dg[k + k * NB] = s;
            const float inv = f_rcp_pos(s);
#pragma unroll
            for (int i = k + 1; i < NB; ++i) dg[i + k * NB] = f_mul(dg[i + k * NB], inv);
#pragma unroll
            for (int j = k + 1; j < NB; ++j)
#pragma unroll
                for (int i = j; i < NB; ++i) dg[i + j * NB] = f_upd(dg[i + j * NB], dg[i + k * NB], dg[j + k * NB]);
        }
        put_tile(CB, dg, cb_, TRUE_{});
        float rinv[NB];
#pragma unroll
        for (int k = 0; k < NB; ++k) rinv[k] = f_rcp_pos(dg[k + k * NB]);
        float xcb[NB];                                  // forward substitution, this block
        if constexpr (SOLVE) {
#pragma unroll
            for (int k = 0; k < NB; ++k) xcb[k] = X[(CB * NB + k) * 32];
#pragma unroll
            for (int k = 0; k < NB; ++k) {
                xcb[k] = f_mul(xcb[k], rinv[k]);
#pragma unroll
                for (int i = k + 1; i < NB; ++i) xcb[i] = f_upd(xcb[i], dg[i + k * NB], xcb[k]);
            }
#pragma unroll
            for (int k = 0; k < NB; ++k) X[(CB * NB + k) * 32] = xcb[k];
        }
        // (b) off-diagonal tiles (rb, CB), rb > CB: GEMM updates, then strsm_tile.
        //     ROWS = real rows of the tile row (4, or N % 4 for a ragged last one,
        //     peeled so the padded rows cost no arithmetic)
        auto offdiag = [&](int rb, auto rows_) {
            constexpr int ROWS = decltype(rows_)::value;
            float acc[16];
            if constexpr (CB < CTM) tmem_ld16(tbase + tidx(rb, CB), acc);
            else load_tile_smem(rb, CB, acc, false);
            sfor<0, CB>([&](auto pb_) {
                constexpr int PB = BSP_CI(pb_);
                float a[16], b[16];
                if constexpr (PB < CTM) {
                    tmem_ld16(tbase + tidx(rb, PB), a);
                    tmem_ld16(tbase + tidx(CB, PB), b);
                } else {
                    load_tile_smem(rb, PB, a, false);
                    load_tile_smem(CB, PB, b, false);
                }
                tmem_wait_ld();
#pragma unroll
                for (int k = 0; k < NB; ++k)
#pragma unroll
                    for (int j = 0; j < NB; ++j) {
                        // rows i, i+1 in one FFMA2 (same bits as two f_upd)
#pragma unroll
                        for (int i = 0; i + 1 < ROWS; i += 2)
                            f_upd2(acc[i + j * NB], acc[i + 1 + j * NB], b[j + k * NB], a[i + k * NB],
                                   a[i + 1 + k * NB]);
                        if constexpr (ROWS % 2 == 1)
                            acc[ROWS - 1 + j * NB] = f_upd(acc[ROWS - 1 + j * NB], a[ROWS - 1 + k * NB], b[j + k * NB]);
                    }
            });
            tmem_wait_ld();
#pragma unroll
            for (int k = 0; k < NB; ++k) {
#pragma unroll
                for (int i = 0; i < ROWS; ++i) acc[i + k * NB] = f_mul(acc[i + k * NB], rinv[k]);
#pragma unroll
                for (int j = k + 1; j < NB; ++j)
#pragma unroll
                    for (int i = 0; i < ROWS; ++i)
                        acc[i + j * NB] = f_upd(acc[i + j * NB], acc[i + k * NB], dg[j + k * NB]);
            }
            put_tile(rb, acc, cb_, FALSE_{});
            if constexpr (SOLVE) {                      // x_rows -= L(rb, CB) x_CB, k ascending
                float xr[NB];
#pragma unroll
                for (int i = 0; i < ROWS; ++i) xr[i] = X[(rb * NB + i) * 32];
#pragma unroll
                for (int k = 0; k < NB; ++k)
#pragma unroll
                    for (int i = 0; i < ROWS; ++i) xr[i] = f_upd(xr[i], acc[i + k * NB], xcb[k]);
#pragma unroll
                for (int i = 0; i < ROWS; ++i) X[(rb * NB + i) * 32] = xr[i];
            }
        };
        constexpr int TRF = N / NB;                  // full tile rows
#pragma unroll 1
        for (int rb = CB + 1; rb < TRF; ++rb) offdiag(rb, std::integral_constant<int, NB>{});
        if constexpr (N % NB != 0)
            if constexpr (TR - 1 > CB) offdiag(TR - 1, std::integral_constant<int, N % NB>{});
        if constexpr (CB < CTM) tmem_wait_st();
    });

    // ---- 2. SYRK into the register triangle: rolled over panel columns ------
    constexpr int RB0 = S / NB;                 // first tile row of the trailing part
    constexpr int NV = (TR - RB0) * NB;         // >= NT (ragged last tile row)
    auto syrk = [&](const float *v) {
#pragma unroll
        for (int n = 0; n < NT; ++n)
#pragma unroll
            for (int m = n; m < NT; ++m) r[tri<NT>(m, n)] = f_upd(r[tri<NT>(m, n)], v[m], v[n]);
    };
#pragma unroll 1
    for (int k = 0; k < CS; ++k) {              // panel columns held in TMEM
        float v[NV];
        const uint32_t col = tbase + (uint32_t)((k / NB) * TR - (k / NB) * ((k / NB) - 1) / 2 - (k / NB)) * 16u +
                             (uint32_t)((k % NB) * NB);
#pragma unroll
        for (int rb = RB0; rb < TR; ++rb) tmem_ld4(col + (uint32_t)rb * 16u, v + (rb - RB0) * NB);
        tmem_wait_ld();
        syrk(v);
    }
#pragma unroll 1
    for (int k = CS; k < S; ++k) {              // panel columns held in shared memory
        float v[NT];
        const int kb = qs(S, k);
#pragma unroll
        for (int m = 0; m < NT; ++m) v[m] = Q[(kb + m) * 32];
        syrk(v);
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
        if constexpr (SOLVE) {                          // forward step j = S + k
            const float xk = f_mul(X[(S + k) * 32], inv);
            X[(S + k) * 32] = xk;
#pragma unroll
            for (int i = k + 1; i < NT; ++i) X[(S + i) * 32] = f_upd(X[(S + i) * 32], r[tri<NT>(i, k)], xk);
        }
    });
    if constexpr (SOLVE) {
        // backward substitution (dot form, j ascending), trailing rows from registers
        sfor<0, NT>([&](auto t_) {
            constexpr int i = NT - 1 - BSP_CI(t_);
            float sacc = X[(S + i) * 32];
#pragma unroll
            for (int j = i + 1; j < NT; ++j) sacc = f_upd(sacc, r[tri<NT>(j, i)], X[(S + j) * 32]);
            X[(S + i) * 32] = f_mul(sacc, f_rcp_pos(r[tri<NT>(i, i)]));
        });
        // ... panel rows i = S-1..0: column i of L from TMEM tiles / shared memory
#pragma unroll 1
        for (int i = S - 1; i >= 0; --i) {
            const int cb = i / NB, ii = i - cb * NB;
            float sacc = X[i * 32];
            float lii = 0.0f;
#pragma unroll 1
            for (int rb = cb; rb < TR; ++rb) {
                float l[NB];
                if (cb < CTM) {
                    tmem_ld4(tbase + tidx(rb, cb) + (uint32_t)(ii * NB), l);
                    tmem_wait_ld();
                } else {
#pragma unroll
                    for (int q = 0; q < NB; ++q) {
                        const int m = rb * NB + q;
                        l[q] = (m < N && m >= i) ? Q[qs(m, i) * 32] : 0.0f;
                    }
                }
                if (rb == cb) lii = l[ii];
#pragma unroll
                for (int q = 0; q < NB; ++q) {
                    const int j = rb * NB + q;
                    if (j > i && j < N) sacc = f_upd(sacc, l[q], X[j * 32]);
                }
            }
            X[i * 32] = f_mul(sacc, f_rcp_pos(lii));
        }
        if (active && inf == 0) {                       // SPOSV: failed matrices keep B
            const RectAddr<N, CT> ba(Bx, g, cs, 1);
#pragma unroll 4
            for (int i = 0; i < N; ++i) st_stream(ba.at(i, 0), X[i * 32]);
        }
    }
    if (active) info[gid] = inf;
    count_failures(active && inf != 0, nfailed);

    // ---- release TMEM ---------------------------------------------------------
    tmem_fence_before();
    __syncthreads();
    if (warp == 0) {
        tmem_fence_after();
        tmem_dealloc(tmem_base_sh, SH::COLS);
    }
}

template <int N, int CT, int S, bool TMA, int FILL>
cudaError_t launch_ptmem(const FactorArgs &a) {
    using SH = TmemShape<N, S>;
    // Enough dynamic shared memory that at most 512 / COLS CTAs are resident
    // per SM, so no CTA ever waits in tcgen05.alloc: >= 80 KB for two CTAs of
    // 256 columns, >= 120 KB for one CTA of 512.
    size_t sm = (size_t)4 * SH::PSM * 32 * 4;
    const size_t floor_sm = SH::COLS == 256 ? 80 * 1024 : 120 * 1024;
    if (sm < floor_sm) sm = floor_sm;
    constexpr int K = S - SH::CS;
    PtmemMaps<K> maps{};
    auto go = [&](auto kern) -> cudaError_t {
        cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
        if (e == cudaSuccess) e = apply_carveout(kern, a.carveout);
        if (e != cudaSuccess) return e;
        kern<<<grid_for(a.batch, 128), 128, sm, a.stream>>>(a.A, a.info, a.nfailed, a.batch, a.cstride, maps,
                                                             nullptr);
        return cudaGetLastError();
    };
    // per-thread staging requested (no chunk-32 TMA): the shared-memory panel
    // columns by 2-D TMA where the layout allows (16-B row stride) and where it
    // measured ahead of the per-thread cp.async form: n = 32..38 (+1-3%; n = 25
    // and 40: -1 to -3%, elsewhere within 1%: tuning/sweep_b200_r02_tma2d_ab_*.jsonl)
    if constexpr (!TMA && SH::PSM > 0 && N >= 32 && N <= 38) {
        bool tm = true;
        for (int c = SH::CS; c < S && tm; ++c)
            tm = tma2d_make_map(&maps.m[c - SH::CS], a.A, a.batch, a.cstride, N * N, N - c);
        if (tm) return go(potrf_ptmem_kernel<N, CT, S, TMA, false, FILL, true>);
    }
    return go(potrf_ptmem_kernel<N, CT, S, TMA, false, FILL, false>);
}

template <int N, int CT, int S, bool TMA>
cudaError_t launch_sposv_ptmem(const SolveArgs &a) {
    using SH = TmemShape<N, S>;
    size_t sm = (size_t)4 * ((SH::PSM > 0 ? SH::PSM : 1) + N) * 32 * 4;
    const size_t floor_sm = SH::COLS == 256 ? 80 * 1024 : 120 * 1024;
    if (sm < floor_sm) sm = floor_sm;
    auto kern = potrf_ptmem_kernel<N, CT, S, TMA, true>;
    const cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    if (e != cudaSuccess) return e;
    const PtmemMaps<S - SH::CS> maps{};
    kern<<<grid_for(a.batch, 128), 128, sm, a.stream>>>(a.A, a.info, a.nfailed, a.batch, a.cstride, maps, a.B);
    return cudaGetLastError();
}

}  // namespace bsp
