// potrf_canon.cuh -- variant CANON: the factorization on CANONICAL storage
// (column-major n x n matrices one after another, "the canonical
// storage ... each matrix occupies a contiguous chunk of memory"), with the
// layout conversion fused into the load and the store (round 2, C4's
// "interleaved vs canonical incl. layout-convert cost").
//
// Why.  The paper's point is that one-thread-per-matrix loads do not coalesce
// in the canonical layout: lane l's element (i, j) is n^2
// floats from lane l+1's.  The unfused canonical path converts in, factors and
// converts back: 2 x 8n^2 + 4n(n+1) bytes per matrix and 3 launches.  Here a
// warp owns 32 consecutive matrices (one contiguous 128*n^2-byte block) and
// moves each column's lower runs -- 32 runs of n-j floats, n^2 floats apart --
// with FLAT cp.async copies straight into a per-warp shared image of the 32
// lower triangles ([32][T|1], odd pitch: lane l then reads its own row
// conflict-free): lane l takes flat elements l, l+32, ... of column j's 32
// runs, so a warp instruction moves 32 consecutive run elements (whole runs,
// few sectors); no register holds a value in flight, and all n(n+1)/2 copies
// per lane are issued before the first wait, as REG issues its loads.  The
// stores use the same flat mapping (each final column staged in its own image
// slots).  The factorization is REG's (Fig. 9 op order -> bits identical to
// every interleaved variant on the same matrices, pin P8); each final column is
// written back into its image slots and leaves with flat stores.  Only
// lower-triangle elements are read or written (the strict upper triangle is
// never touched at the instruction level).  Image: 32*(T|1)*4 B per warp --
// 17.5 KB at n = 16 (12 warps per SM), 27 KB at n = 20 (8 warps per SM, as
// REG's 232 registers allow); n <= 20.
#pragma once

#include "common.cuh"
#include "launch.h"
#include "ptx.cuh"

namespace bsp {

template <int N>
struct CanonShape {
    static constexpr int T = N * (N + 1) / 2;
    static constexpr int PT = (T % 2) ? T : T + 1;        // odd image pitch
    static constexpr int WARPS = 4;
    static constexpr size_t SMEM = (size_t)WARPS * 32 * PT * sizeof(float);
    // column j's first slot in the packed lower triangle (= tri<N>(j, j))
    __host__ __device__ static constexpr int off(int j) { return j * N - j * (j - 1) / 2; }
};

// One 32-matrix group per warp.  (Measured alternative, not kept: persistent
// warps issuing the next group's copies while this group is factored -- the
// registers then stay live across the copies, 243 instead of 164 at n = 16, and
// the extra column tile costs a CTA per SM: 0.45-0.95x at n = 4..20, j16c.)
template <int N>
__global__ void __launch_bounds__(32 * CanonShape<N>::WARPS)
potrf_canon_kernel(float *__restrict__ A, int32_t *__restrict__ info, int32_t *__restrict__ nfailed,
                   int64_t batch) {
    using SH = CanonShape<N>;
    constexpr int T = SH::T, PT = SH::PT;
    extern __shared__ float canon_smem[];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    float *im = canon_smem + w * 32 * PT;                 // this warp's image [32][PT]
    const int64_t m0 = ((int64_t)blockIdx.x * SH::WARPS + w) * 32;
    if (m0 >= batch) return;                              // warp-uniform
    const int nact = batch - m0 < 32 ? (int)(batch - m0) : 32;
    float *gb = A + m0 * (int64_t)(N * N);                // the group's canonical block

    // 1. flat copies of every column's 32 lower runs into the image: lane takes
    //    flat elements lane + 32t of the runs (a warp instruction moves 32
    //    consecutive run elements: 2-3 sectors), stepped incrementally by
    //    32 = Q*L + R (no divisions, one live index chain per column).  (Each
    //    lane copying its own matrix -- 32 sectors per instruction -- ran
    //    L1-tag / MIO bound at 0.23 of HBM: j16 ncu.)
    sfor<0, N>([&](auto j_) {
        constexpr int j = BSP_CI(j_), L = N - j;
        constexpr int Q = 32 / L, R = 32 % L;
        int ln = lane;
        asm volatile("" : "+r"(ln));                      // column j's chain starts after column j-1's copies
        int m = ln / L, i = ln - m * L;
        int so = m * PT + SH::off(j) + i, go = m * (N * N) + j * (N + 1) + i;
#pragma unroll
        for (int t = 0; t < L; ++t) {
            if (m < nact) cp_async4(im + so, gb + go);
            m += Q, i += R, so += Q * PT + R, go += Q * (N * N) + R;
            if (i >= L) i -= L, m += 1, so += PT - L, go += N * N - L;
        }
    });
    cp_async_commit();
    cp_async_wait_all();
    __syncwarp();
    float a[T];
#pragma unroll
    for (int s = 0; s < T; ++s) a[s] = im[lane * PT + s];

    // 2. REG's right-looking factorization; column k out through its image slots
    int inf = 0;
    const bool active = lane < nact;
    sfor<0, N>([&](auto k_) {
        constexpr int k = BSP_CI(k_), L = N - k;
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
        float *cb = im + SH::off(k);
#pragma unroll
        for (int i = 0; i < L; ++i) cb[lane * PT + i] = a[tri<N>(k + i, k)];
        __syncwarp();
        // flat element lane + 32t of the 32 runs = (m, i), stepped by 32 = Q*L + R
        constexpr int Q = 32 / L, R = 32 % L;
        int m = lane / L, i = lane - m * L;
        int so = m * PT + i, go = m * (N * N) + k * (N + 1) + i;
#pragma unroll
        for (int t = 0; t < L; ++t) {
            if (m < nact) st_stream(gb + go, cb[so]);
            m += Q, i += R, so += Q * PT + R, go += Q * (N * N) + R;
            if (i >= L) i -= L, m += 1, so += PT - L, go += N * N - L;
        }
    });
    if (active) info[m0 + lane] = inf;
    count_failures(active && inf != 0, nfailed);
}

template <int N>
cudaError_t launch_canon(float *A, int32_t *info, int32_t *nfailed, int64_t batch, cudaStream_t stream) {
    using SH = CanonShape<N>;
    auto kern = potrf_canon_kernel<N>;
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)SH::SMEM);
    if (e != cudaSuccess) return e;
    const int64_t groups = (batch + 31) / 32;
    kern<<<(unsigned)((groups + SH::WARPS - 1) / SH::WARPS), 32 * SH::WARPS, SH::SMEM, stream>>>(A, info, nfailed,
                                                                                                 batch);
    return cudaGetLastError();
}

}  // namespace bsp
