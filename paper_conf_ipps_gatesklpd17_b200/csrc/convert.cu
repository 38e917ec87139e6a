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
// Persistent CTAs (the resident count) walk the tiles with a two-stage
// pipeline in registers: each thread's 16 loads of tile t+1 are issued before
// tile t is written out of shared memory, so loads stay in flight during the
// store phase (a load-all / sync / store-all kernel idles HBM reads half the
// time; per-thread 4-byte cp.async was measured slower: LSU-issue bound).
// The padded shared tile (odd pitch) is conflict-free in both directions.
// Pad lanes are never touched.
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


// interleaved offset of lane 0 of the 32-matrix group starting at matrix m
__device__ __forceinline__ int64_t group_base(int64_t m, int64_t C, int E) {
    return (m / C) * C * (int64_t)E + (m % C);
}

// Tile geometry of tile t.
struct CvTile {
    int64_t m0;
    int e0, ecount, rcount, n_el;
    uint32_t mg;
};
__device__ __forceinline__ CvTile cv_tile(const CvShape &s, int64_t t) {
    CvTile x;
    const int64_t rt = t / s.elem_tiles;
    const int te = (int)(t - rt * s.elem_tiles);
    x.m0 = rt * s.R;
    x.e0 = te * s.TE;
    x.ecount = (s.E - x.e0) < s.TE ? (s.E - x.e0) : s.TE;
    x.rcount = (int)((s.batch - x.m0) < s.R ? (s.batch - x.m0) : s.R);
    x.n_el = s.R * x.ecount;
    // idx / ecount without a division: idx < 2^14, ecount <= 128 -> exact
    // (64-bit product: idx * mg exceeds 2^32 for ecount = 1)
    x.mg = (1u << 22) / (uint32_t)x.ecount + 1u;
    return x;
}

// source element idx of tile x -> (smem slot, global offset); false if padding
template <int DIR>
__device__ __forceinline__ bool cv_src(const CvShape &s, const CvTile &x, const int64_t *gb, int idx, int &slot,
                                       int64_t &off) {
    if (idx >= x.n_el) return false;
    int r, e;
    if (DIR == 0) {                          // canonical rows: lanes -> consecutive elements
        r = (int)(((uint64_t)idx * x.mg) >> 22);
        e = idx - r * x.ecount;
        off = (x.m0 + r) * s.E + x.e0 + e;
    } else {                                 // interleaved lines: lanes -> consecutive matrices
        r = idx & s.rmask;
        e = idx >> s.rshift;
        off = gb[r >> 5] + (int64_t)(x.e0 + e) * s.C + (r & 31);
    }
    slot = r * s.ld + e;
    return r < x.rcount;
}

template <int DIR>
__device__ __forceinline__ void cv_store(float *__restrict__ dst, const float *buf, const CvShape &s,
                                         const CvTile &x, const int64_t *gb) {
#pragma unroll 4
    for (int idx = threadIdx.x; idx < x.n_el; idx += CV_THREADS) {
        if (DIR == 0) {
            const int r = idx & s.rmask, e = idx >> s.rshift;
            if (r < x.rcount) dst[gb[r >> 5] + (int64_t)(x.e0 + e) * s.C + (r & 31)] = buf[r * s.ld + e];
        } else {
            const int r = (int)(((uint64_t)idx * x.mg) >> 22), e = idx - r * x.ecount;
            if (r < x.rcount) dst[(x.m0 + r) * s.E + x.e0 + e] = buf[r * s.ld + e];
        }
    }
}

// Software pipeline in registers: the 16 loads of tile t+1 are issued before
// tile t is written out, so loads stay in flight during the store phase.
template <int DIR>
__global__ void __launch_bounds__(CV_THREADS, 4)
convert_kernel(const float *__restrict__ src, float *__restrict__ dst, CvShape s) {
    extern __shared__ float buf[];                  // [R][ld]
    __shared__ int64_t gbase[2][CV_GMAX];
    auto fill_gbase = [&](int slot, int64_t t) {
        const int64_t m0 = (t / s.elem_tiles) * s.R;
        for (int g = threadIdx.x; g < s.G; g += CV_THREADS) gbase[slot][g] = group_base(m0 + 32 * g, s.C, s.E);
    };
    int64_t t = blockIdx.x;
    if (t >= s.tiles) return;
    float v[CV_PER];
    int slot[CV_PER];
    fill_gbase(0, t);
    __syncthreads();
    CvTile x = cv_tile(s, t);
#pragma unroll
    for (int k = 0; k < CV_PER; ++k) {
        int64_t off;
        slot[k] = -1;
        if (cv_src<DIR>(s, x, gbase[0], threadIdx.x + k * CV_THREADS, slot[k], off)) v[k] = src[off];
        else slot[k] = -1;
    }
    int cur = 0;
    for (; t < s.tiles; t += gridDim.x) {
#pragma unroll
        for (int k = 0; k < CV_PER; ++k)
            if (slot[k] >= 0) buf[slot[k]] = v[k];
        const int64_t tn = t + gridDim.x;
        const bool more = tn < s.tiles;
        if (more) fill_gbase(cur ^ 1, tn);
        __syncthreads();                            // tile t in smem, next gbase visible
        if (more) {                                 // next tile's loads, in flight during the stores
            const CvTile xn = cv_tile(s, tn);
#pragma unroll
            for (int k = 0; k < CV_PER; ++k) {
                int64_t off;
                if (cv_src<DIR>(s, xn, gbase[cur ^ 1], threadIdx.x + k * CV_THREADS, slot[k], off)) v[k] = src[off];
                else slot[k] = -1;
            }
        }
        cv_store<DIR>(dst, buf, s, x, gbase[cur]);
        __syncthreads();                            // buf and gbase[cur] free
        if (more) x = cv_tile(s, tn);
        cur ^= 1;
    }
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
    const size_t sm = (size_t)s.R * s.ld * sizeof(float);
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
