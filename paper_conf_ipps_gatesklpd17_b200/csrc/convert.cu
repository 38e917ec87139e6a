// convert.cu -- layout conversion canonical <-> (chunked-)interleaved
// (PAPER.md:128 canonical; Figs. 7-8 interleaved; SURVEY
// §8(a) row a7).  Pure data movement: a batched transpose.  Matrix m's element
// e (= i + j*n, E = n*n elements) is at m*E in canonical storage and at
// (m/C)*C*E + e*C + m%C in interleaved storage.
//
// Tiles of R = 32*G consecutive matrices x TE elements (TE = min(E, 128), G a
// power of two with R*TE <= 4096): on the canonical side a tile is R row
// segments of TE contiguous floats (for small n one contiguous run); on the
// interleaved side every 32-matrix group (never split by a chunk boundary,
// C % 32 == 0) gives TE segments of 32 contiguous floats -- one 128-B line
// each.  Both sides fully coalesced.
//
// Persistent CTAs (a few per SM) walk the tiles with a two-stage pipeline:
// the source tile t+1 streams into shared memory with per-thread cp.async
// (no register staging, 16 copies in flight per thread) while tile t is
// written out from the other buffer -- so loads are always in flight, which
// a load-all / sync / store-all kernel cannot sustain.  The padded shared
// tile (odd pitch) is conflict-free in both directions.  Pad lanes are never
// touched.
#include <cuda_runtime.h>
#include <stdint.h>

#include "ptx.cuh"

namespace bsp {

constexpr int CV_THREADS = 256;
constexpr int CV_TILE = 4096;    // max floats per tile
constexpr int CV_TE = 128;       // max elements per tile
constexpr int CV_GMAX = 128;     // max 32-matrix groups per tile
constexpr int CV_PER = CV_TILE / CV_THREADS;

struct CvShape {
    int64_t batch, C;
    int E, TE, G, R, ld, elem_tiles, rmask, rshift;
    int64_t tiles;
};

__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int K>
__device__ __forceinline__ void cp_async_wait() { asm volatile("cp.async.wait_group %0;" ::"n"(K) : "memory"); }

// interleaved offset of lane 0 of the 32-matrix group starting at matrix m
__device__ __forceinline__ int64_t group_base(int64_t m, int64_t C, int E) {
    return (m / C) * C * (int64_t)E + (m % C);
}

template <int DIR>
__device__ __forceinline__ void cv_issue_loads(const float *__restrict__ src, float *buf, const CvShape &s,
                                               int64_t t, const int64_t *gb) {
    const int64_t rt = t / s.elem_tiles;
    const int te = (int)(t - rt * s.elem_tiles);
    const int64_t m0 = rt * s.R;
    const int e0 = te * s.TE;
    const int ecount = (s.E - e0) < s.TE ? (s.E - e0) : s.TE;
    const int rcount = (int)((s.batch - m0) < s.R ? (s.batch - m0) : s.R);
    const int n_el = s.R * ecount;
    // idx / ecount without a division: idx < 2^14, ecount <= 128 -> exact
    // (64-bit product: idx * mg exceeds 2^32 for ecount = 1)
    const uint32_t mg = (1u << 22) / (uint32_t)ecount + 1u;
#pragma unroll
    for (int k = 0; k < CV_PER; ++k) {
        const int idx = threadIdx.x + k * CV_THREADS;
        if (idx >= n_el) break;
        if (DIR == 0) {                       // canonical rows: lanes -> consecutive elements
            const int r = (int)(((uint64_t)idx * mg) >> 22), e = idx - r * ecount;
            if (r < rcount) cp_async4(buf + r * s.ld + e, src + (m0 + r) * s.E + e0 + e);
        } else {                              // interleaved lines: lanes -> consecutive matrices
            const int r = idx & s.rmask, e = idx >> s.rshift;
            if (r < rcount) cp_async4(buf + r * s.ld + e, src + gb[r >> 5] + (int64_t)(e0 + e) * s.C + (r & 31));
        }
    }
}

template <int DIR>
__device__ __forceinline__ void cv_store(float *__restrict__ dst, const float *buf, const CvShape &s, int64_t t,
                                         const int64_t *gb) {
    const int64_t rt = t / s.elem_tiles;
    const int te = (int)(t - rt * s.elem_tiles);
    const int64_t m0 = rt * s.R;
    const int e0 = te * s.TE;
    const int ecount = (s.E - e0) < s.TE ? (s.E - e0) : s.TE;
    const int rcount = (int)((s.batch - m0) < s.R ? (s.batch - m0) : s.R);
    const int n_el = s.R * ecount;
    const uint32_t mg = (1u << 22) / (uint32_t)ecount + 1u;
#pragma unroll 4
    for (int idx = threadIdx.x; idx < n_el; idx += CV_THREADS) {
        if (DIR == 0) {
            const int r = idx & s.rmask, e = idx >> s.rshift;
            if (r < rcount) dst[gb[r >> 5] + (int64_t)(e0 + e) * s.C + (r & 31)] = buf[r * s.ld + e];
        } else {
            const int r = (int)(((uint64_t)idx * mg) >> 22), e = idx - r * ecount;
            if (r < rcount) dst[(m0 + r) * s.E + e0 + e] = buf[r * s.ld + e];
        }
    }
}

template <int DIR>
__global__ void __launch_bounds__(CV_THREADS, 4)
convert_kernel(const float *__restrict__ src, float *__restrict__ dst, CvShape s) {
    extern __shared__ float smem[];                 // 2 x [R][ld]
    __shared__ int64_t gbase[2][CV_GMAX];
    const size_t bsz = (size_t)s.R * s.ld;
    auto buf = [&](int i) { return smem + i * bsz; };
    auto fill_gbase = [&](int slot, int64_t t) {
        const int64_t m0 = (t / s.elem_tiles) * s.R;
        for (int g = threadIdx.x; g < s.G; g += CV_THREADS) gbase[slot][g] = group_base(m0 + 32 * g, s.C, s.E);
    };
    int64_t t = blockIdx.x;
    if (t >= s.tiles) return;
    fill_gbase(0, t);
    __syncthreads();
    cv_issue_loads<DIR>(src, buf(0), s, t, gbase[0]);
    cp_async_commit();
    int cur = 0;
    for (; t < s.tiles; t += gridDim.x) {
        const int64_t tn = t + gridDim.x;
        if (tn < s.tiles) {                         // prefetch the next tile into the other buffer
            fill_gbase(cur ^ 1, tn);
            __syncthreads();
            cv_issue_loads<DIR>(src, buf(cur ^ 1), s, tn, gbase[cur ^ 1]);
        }
        cp_async_commit();
        cp_async_wait<1>();                         // tile t has landed (this thread's copies)
        __syncthreads();                            // ... and everybody else's
        cv_store<DIR>(dst, buf(cur), s, t, gbase[cur]);
        __syncthreads();                            // buffer cur is free again
        cur ^= 1;
    }
    cp_async_wait<0>();
}

cudaError_t launch_convert(int dir, int n, int64_t batch, int64_t C, const float *src, float *dst,
                           cudaStream_t stream) {
    CvShape s;
    s.batch = batch;
    s.C = C;
    s.E = n * n;
    s.TE = s.E < CV_TE ? s.E : CV_TE;
    int G = CV_TILE / (32 * s.TE);
    if (G < 1) G = 1;
    if (G > CV_GMAX) G = CV_GMAX;
    while (G & (G - 1)) G &= G - 1;                 // power of two: r = idx & (R-1)
    s.G = G;
    s.R = 32 * G;
    s.ld = (s.TE & 1) ? s.TE : s.TE + 1;
    s.rmask = s.R - 1;
    s.rshift = 0;
    while ((1 << s.rshift) < s.R) ++s.rshift;
    s.elem_tiles = (s.E + s.TE - 1) / s.TE;
    s.tiles = ((batch + s.R - 1) / s.R) * s.elem_tiles;
    const size_t sm = 2 * (size_t)s.R * s.ld * sizeof(float);
    int dev = 0, sms = 148, per_sm = 4;
    if (cudaGetDevice(&dev) == cudaSuccess) cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    if (dir == 0) cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, convert_kernel<0>, CV_THREADS, sm);
    else cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, convert_kernel<1>, CV_THREADS, sm);
    if (per_sm < 1) per_sm = 1;
    int64_t grid = (int64_t)sms * per_sm;           // persistent: exactly the resident CTAs
    if (grid > s.tiles) grid = s.tiles;
    if (grid < 1) grid = 1;
    if (dir == 0)
        convert_kernel<0><<<(unsigned)grid, CV_THREADS, sm, stream>>>(src, dst, s);
    else
        convert_kernel<1><<<(unsigned)grid, CV_THREADS, sm, stream>>>(src, dst, s);
    return cudaGetLastError();
}

}  // namespace bsp
