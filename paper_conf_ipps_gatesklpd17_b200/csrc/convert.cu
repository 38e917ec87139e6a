// convert.cu -- layout conversion canonical <-> (chunked-)interleaved
// (PAPER.md:128 canonical; Figs. 7-8 interleaved; SURVEY
// §8(a) row a7).  Pure data movement: a batched transpose.  Chunk q of C
// matrices is a [C][E] row-major block in canonical storage (matrix-major,
// E = n*n) and an [E][C] block in interleaved storage (element-major).
//
// One CTA moves a tile of 32 matrices x TE elements (TE = min(E, 128)):
// canonical side = 32 row segments of TE contiguous floats, interleaved side =
// TE segments of 32 contiguous floats (one full 128-B line each) -- both sides
// fully coalesced -- through a padded [32][TE+1] shared tile (conflict-free in
// both directions).  Each thread has 16 independent loads in flight.  Pad
// lanes of the interleaved side are never read or written.
#include <cuda_runtime.h>
#include <stdint.h>

namespace bsp {

constexpr int CV_R = 32;     // matrices per tile
constexpr int CV_TE = 128;   // max elements per tile
constexpr int CV_THREADS = 256;

// dir 0: canonical -> interleaved; dir 1: interleaved -> canonical
template <int DIR>
__global__ void __launch_bounds__(CV_THREADS)
convert_kernel(const float *__restrict__ src, float *__restrict__ dst, int64_t batch, int64_t C,
               int E, int TE, int64_t row_tiles, int elem_tiles) {
    __shared__ float tile[CV_R][CV_TE + 1];
    const int64_t t = blockIdx.x;
    const int64_t per_chunk = row_tiles * elem_tiles;
    const int64_t q = t / per_chunk;                  // chunk
    const int64_t rem = t - q * per_chunk;
    const int64_t tr = rem / elem_tiles;              // 32-matrix tile inside the chunk
    const int te = (int)(rem - tr * elem_tiles);      // element tile
    const int64_t lanes = (batch - q * C) < C ? (batch - q * C) : C;   // real matrices in chunk
    const int64_t r0 = tr * CV_R;
    const int e0 = te * TE;
    const int ecount = (E - e0) < TE ? (E - e0) : TE;
    const int rcount = (int)((lanes - r0) < CV_R ? (lanes - r0) : CV_R);
    const int64_t cbase = q * C * (int64_t)E;         // same offset on both sides
    const int n_el = CV_R * ecount;
    // idx / ecount without a division: idx < 4096 and ecount <= 128, so
    // (idx * m) >> 20 with m = 2^20/ecount + 1 is exact (error < 1/256 < 1/ecount)
    const uint32_t m = (1u << 20) / (uint32_t)ecount + 1u;

    constexpr int PER = CV_R * CV_TE / CV_THREADS;   // 16 elements per thread per phase
    float v[PER];
    if (DIR == 0) {
        // all 16 loads issued before any shared-memory store: 16 lines in flight per thread
#pragma unroll
        for (int k = 0; k < PER; ++k) {
            const int idx = threadIdx.x + k * CV_THREADS;
            const int r = (int)(((uint32_t)idx * m) >> 20), e = idx - r * ecount;
            v[k] = (idx < n_el && r < rcount) ? src[cbase + (r0 + r) * E + e0 + e] : 0.0f;
        }
#pragma unroll
        for (int k = 0; k < PER; ++k) {
            const int idx = threadIdx.x + k * CV_THREADS;
            const int r = (int)(((uint32_t)idx * m) >> 20), e = idx - r * ecount;
            if (idx < n_el) tile[r][e] = v[k];
        }
        __syncthreads();
#pragma unroll
        for (int k = 0; k < PER; ++k) {
            const int idx = threadIdx.x + k * CV_THREADS;
            const int e = idx >> 5, r = idx & 31;
            if (idx < n_el && r < rcount) dst[cbase + (int64_t)(e0 + e) * C + r0 + r] = tile[r][e];
        }
    } else {
#pragma unroll
        for (int k = 0; k < PER; ++k) {
            const int idx = threadIdx.x + k * CV_THREADS;
            const int e = idx >> 5, r = idx & 31;
            v[k] = (idx < n_el && r < rcount) ? src[cbase + (int64_t)(e0 + e) * C + r0 + r] : 0.0f;
        }
#pragma unroll
        for (int k = 0; k < PER; ++k) {
            const int idx = threadIdx.x + k * CV_THREADS;
            const int e = idx >> 5, r = idx & 31;
            if (idx < n_el) tile[r][e] = v[k];
        }
        __syncthreads();
#pragma unroll
        for (int k = 0; k < PER; ++k) {
            const int idx = threadIdx.x + k * CV_THREADS;
            const int r = (int)(((uint32_t)idx * m) >> 20), e = idx - r * ecount;
            if (idx < n_el && r < rcount) dst[cbase + (r0 + r) * E + e0 + e] = tile[r][e];
        }
    }
}

cudaError_t launch_convert(int dir, int n, int64_t batch, int64_t C, const float *src, float *dst,
                           cudaStream_t stream) {
    const int E = n * n;
    const int TE = E < CV_TE ? E : CV_TE;
    const int64_t nchunks = (batch + C - 1) / C;
    const int64_t row_tiles = (C + CV_R - 1) / CV_R;
    const int elem_tiles = (E + TE - 1) / TE;
    const int64_t blocks = nchunks * row_tiles * elem_tiles;
    if (blocks > 0x7fffffffLL) return cudaErrorInvalidConfiguration;
    if (dir == 0)
        convert_kernel<0><<<(unsigned)blocks, CV_THREADS, 0, stream>>>(src, dst, batch, C, E, TE, row_tiles,
                                                                       elem_tiles);
    else
        convert_kernel<1><<<(unsigned)blocks, CV_THREADS, 0, stream>>>(src, dst, batch, C, E, TE, row_tiles,
                                                                       elem_tiles);
    return cudaGetLastError();
}

}  // namespace bsp
