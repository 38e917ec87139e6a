// potrs.cuh -- batched SPOTRS and fused SPOSV on interleaved storage
// ("the step directly after the path", needed by ALS).
//
// "A symmetric positive definite system of linear equations Ax = b can be
// solved by computing the Cholesky factorization A = LL^T, and then applying
// forward substitution and backward substitution to the vector b using the
// factors L and L^T".  One thread per matrix, as for the
// factorization.  The right-hand sides B (n x nrhs per matrix, column-major)
// are interleaved with the SAME chunk C as the matrices: element (i, r) of
// matrix b's block at (b/C)*C*n*nrhs + (i + r*n)*C + b%C.
//
// Op order (identical in both kernels, so the fused solve and factor-then-
// solve agree bit for bit):
//   forward  (L y = b), column-oriented:  for j = 0..n-1:
//            y_j = y_j * rcp.rn(L_jj);  y_i = fma(-L_ij, y_j, y_i)  (i > j)
//   backward (L^T x = y), dot form:        for i = n-1..0:
//            s = y_i; s = fma(-L_ji, x_j, s) (j = i+1..n-1);  x_i = s * rcp.rn(L_ii)
// Both passes walk L by columns, so the standalone kernel streams each column
// of L once per pass with one 128-B line per warp access.
#pragma once

#include "common.cuh"
#include "launch.h"

namespace bsp {

// chunked-interleaved address of (i, r) in an ROWS x COLS block
template <int ROWS, int CT>
struct RectAddr {
    float *base;
    int64_t cs;
    __device__ __forceinline__ RectAddr(float *P, int64_t g, int64_t cstride, int cols) {
        const uint64_t C = CT ? (uint64_t)CT : (uint64_t)cstride;
        cs = (int64_t)C;
        base = P + ((uint64_t)g / C) * C * (uint64_t)(ROWS * cols) + ((uint64_t)g % C);
    }
    __device__ __forceinline__ float *at(int i, int r) const {
        return base + (int64_t)(i + r * ROWS) * (CT ? (int64_t)CT : cs);
    }
};

// ---- standalone SPOTRS: L streamed from global memory -------------------------
// Right-hand sides are processed NR at a time (x in registers); L is read once
// per pass per group.  rhs0/nr select the group inside the nrhs columns.
template <int N, int NR, int CT>
__global__ void __launch_bounds__(256)
potrs_kernel(const float *__restrict__ L, float *__restrict__ B, const int32_t *__restrict__ skip_info,
             int64_t batch, int64_t cs, int nrhs, int rhs0) {
    const int64_t gid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const bool active = gid < batch;
    const int64_t g = active ? gid : batch - 1;
    const Addr<N, CT> la(const_cast<float *>(L), g, cs);
    const RectAddr<N, CT> ba(B, g, cs, nrhs);
    float x[NR][N];
#pragma unroll
    for (int r = 0; r < NR; ++r)
#pragma unroll
        for (int i = 0; i < N; ++i) x[r][i] = ld_stream(ba.at(i, rhs0 + r));
    // forward: L y = b
    sfor<0, N>([&](auto j_) {
        constexpr int j = BSP_CI(j_);
        const float inv = f_rcp(__ldg(la.at(j, j)));
        float l[N];
#pragma unroll
        for (int i = j + 1; i < N; ++i) l[i] = __ldg(la.at(i, j));
#pragma unroll
        for (int r = 0; r < NR; ++r) {
            x[r][j] = f_mul(x[r][j], inv);
#pragma unroll
            for (int i = j + 1; i < N; ++i) x[r][i] = f_upd(x[r][i], l[i], x[r][j]);
        }
    });
    // backward: L^T x = y
    sfor<0, N>([&](auto t_) {
        constexpr int i = N - 1 - BSP_CI(t_);
        const float inv = f_rcp(__ldg(la.at(i, i)));
        float l[N];
#pragma unroll
        for (int j = i + 1; j < N; ++j) l[j] = __ldg(la.at(j, i));
#pragma unroll
        for (int r = 0; r < NR; ++r) {
            float s = x[r][i];
#pragma unroll
            for (int j = i + 1; j < N; ++j) s = f_upd(s, l[j], x[r][j]);
            x[r][i] = f_mul(s, inv);
        }
    });
    // skip_info (nullable): SPOSV semantics for the unfused path -- a matrix
    // whose factorization failed keeps its right-hand sides
    if (active && (skip_info == nullptr || skip_info[gid] == 0)) {
#pragma unroll
        for (int r = 0; r < NR; ++r)
#pragma unroll
            for (int i = 0; i < N; ++i) st_stream(ba.at(i, rhs0 + r), x[r][i]);
    }
}

template <int N, int NR, int CT>
cudaError_t launch_potrs(const SolveArgs &a, int rhs0) {
    const int tpb = 128;
    potrs_kernel<N, NR, CT><<<grid_for(a.batch, tpb), tpb, 0, a.stream>>>(a.A, a.B, a.info, a.batch,
                                                                          a.cstride, a.nrhs, rhs0);
    return cudaGetLastError();
}

// ---- fused SPOSV: factor in registers (REG order), solve with L in registers --
// LAPACK SPOSV semantics: a matrix whose factorization fails (info > 0) keeps
// its right-hand sides unchanged.
template <int N, int NR, int CT>
__global__ void __launch_bounds__(256)
sposv_reg_kernel(float *__restrict__ A, float *__restrict__ B, int32_t *__restrict__ info,
                 int32_t *__restrict__ nfailed, int64_t batch, int64_t cs) {
    constexpr int T = N * (N + 1) / 2;
    const int64_t gid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const bool active = gid < batch;
    const int64_t g = active ? gid : batch - 1;
    const Addr<N, CT> ad(A, g, cs);
    const RectAddr<N, CT> ba(B, g, cs, NR);
    float a[T];
#pragma unroll
    for (int j = 0; j < N; ++j)
#pragma unroll
        for (int i = j; i < N; ++i) a[tri<N>(i, j)] = ld_stream(ad.at(i, j));
    float x[NR][N];
#pragma unroll
    for (int r = 0; r < NR; ++r)
#pragma unroll
        for (int i = 0; i < N; ++i) x[r][i] = ld_stream(ba.at(i, r));

    int inf = 0;
    sfor<0, N>([&](auto k_) {                    // Fig. 9 order, as potrf_reg_kernel
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
            for (int m = k; m < N; ++m) st_stream(ad.at(m, k), a[tri<N>(m, k)]);
        }
        // forward substitution step j = k (column k of L is final; inv = rcp.rn(L_kk))
#pragma unroll
        for (int r = 0; r < NR; ++r) {
            x[r][k] = f_mul(x[r][k], inv);
#pragma unroll
            for (int i = k + 1; i < N; ++i) x[r][i] = f_upd(x[r][i], a[tri<N>(i, k)], x[r][k]);
        }
    });
    sfor<0, N>([&](auto t_) {                    // backward, dot form
        constexpr int i = N - 1 - BSP_CI(t_);
        const float iinv = f_rcp(a[tri<N>(i, i)]);
#pragma unroll
        for (int r = 0; r < NR; ++r) {
            float s = x[r][i];
#pragma unroll
            for (int j = i + 1; j < N; ++j) s = f_upd(s, a[tri<N>(j, i)], x[r][j]);
            x[r][i] = f_mul(s, iinv);
        }
    });
    if (active) {
        info[gid] = inf;
        if (inf == 0) {
#pragma unroll
            for (int r = 0; r < NR; ++r)
#pragma unroll
                for (int i = 0; i < N; ++i) st_stream(ba.at(i, r), x[r][i]);
        }
    }
    count_failures(active && inf != 0, nfailed);
}

template <int N, int NR, int CT>
cudaError_t launch_sposv(const SolveArgs &a) {
    const int tpb = 128;
    sposv_reg_kernel<N, NR, CT><<<grid_for(a.batch, tpb), tpb, 0, a.stream>>>(a.A, a.B, a.info, a.nfailed,
                                                                              a.batch, a.cstride);
    return cudaGetLastError();
}

}  // namespace bsp
