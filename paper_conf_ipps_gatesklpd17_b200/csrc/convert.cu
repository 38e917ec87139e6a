// convert.cu -- layout conversion canonical <-> (chunked-)interleaved
// (PAPER.md:128 canonical; Figs. 7-8 interleaved; SURVEY
// §8(a) row a7).  Pure data movement: a batched transpose.  Chunk q of C
// matrices is a [C][n*n] row-major block in canonical storage (matrix-major)
// and a [n*n][C] block in interleaved storage (element-major), so converting
// is transposing each chunk.  32 x 32 tiles through padded shared memory: both
// the global read and the global write are 128-B coalesced.  Pad lanes of the
// interleaved side are never read or written.
#include <cuda_runtime.h>
#include <stdint.h>

namespace bsp {

constexpr int TT = 32;   // tile edge
constexpr int TR = 8;    // threads per tile row group (block = 32 x 8)

// dir 0: canonical -> interleaved; dir 1: interleaved -> canonical
template <int DIR>
__global__ void __launch_bounds__(256)
convert_kernel(const float *__restrict__ src, float *__restrict__ dst, int64_t batch,
               int64_t C, int E, int64_t row_tiles, int64_t elem_tiles) {
    __shared__ float tile[TT][TT + 1];
    const int64_t t = blockIdx.x;
    const int64_t per_chunk = row_tiles * elem_tiles;
    const int64_t q = t / per_chunk;
    const int64_t rem = t - q * per_chunk;
    const int64_t tr = rem / elem_tiles;
    const int64_t te = rem - tr * elem_tiles;
    const int64_t rows = (batch - q * C) < C ? (batch - q * C) : C;   // valid lanes
    const int64_t r0 = tr * TT;
    const int e0 = (int)(te * TT);
    const int64_t cbase = q * C * (int64_t)E;                          // same for both sides
    const int tx = threadIdx.x, ty = threadIdx.y;

    if (DIR == 0) {
        // read canonical rows r (matrix), cols e: src[cbase + r*E + e]
#pragma unroll
        for (int i = 0; i < TT; i += TR) {
            const int64_t r = r0 + ty + i;
            const int e = e0 + tx;
            if (r < rows && e < E) tile[ty + i][tx] = src[cbase + r * E + e];
        }
        __syncthreads();
        // write interleaved: dst[cbase + e*C + r]
#pragma unroll
        for (int i = 0; i < TT; i += TR) {
            const int e = e0 + ty + i;
            const int64_t r = r0 + tx;
            if (r < rows && e < E) dst[cbase + (int64_t)e * C + r] = tile[tx][ty + i];
        }
    } else {
#pragma unroll
        for (int i = 0; i < TT; i += TR) {
            const int e = e0 + ty + i;
            const int64_t r = r0 + tx;
            if (r < rows && e < E) tile[tx][ty + i] = src[cbase + (int64_t)e * C + r];
        }
        __syncthreads();
#pragma unroll
        for (int i = 0; i < TT; i += TR) {
            const int64_t r = r0 + ty + i;
            const int e = e0 + tx;
            if (r < rows && e < E) dst[cbase + r * E + e] = tile[ty + i][tx];
        }
    }
}

cudaError_t launch_convert(int dir, int n, int64_t batch, int64_t C, const float *src, float *dst,
                           cudaStream_t stream) {
    const int E = n * n;
    const int64_t nchunks = (batch + C - 1) / C;
    const int64_t row_tiles = (C + TT - 1) / TT;
    const int64_t elem_tiles = (E + TT - 1) / TT;
    const int64_t blocks = nchunks * row_tiles * elem_tiles;
    if (blocks > 0x7fffffffLL) return cudaErrorInvalidConfiguration;
    dim3 blk(TT, TR);
    if (dir == 0)
        convert_kernel<0><<<(unsigned)blocks, blk, 0, stream>>>(src, dst, batch, C, E, row_tiles, elem_tiles);
    else
        convert_kernel<1><<<(unsigned)blocks, blk, 0, stream>>>(src, dst, batch, C, E, row_tiles, elem_tiles);
    return cudaGetLastError();
}

}  // namespace bsp
