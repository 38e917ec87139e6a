// convert.cu -- layout conversion canonical <-> (chunked-)interleaved
// (PAPER.md:128 canonical; Figs. 7-8 interleaved; SURVEY
// §8(a) row a7).  Pure data movement: a batched transpose.  Matrix m's element
// e (= i + j*n, E = n*n elements) is at m*E in canonical storage and at
// (m/C)*C*E + e*C + m%C in interleaved storage.
//
// A CTA moves a tile of R = 32*G consecutive matrices x TE elements
// (TE = min(E, 128), G a power of two with R*TE <= 4096): on the canonical
// side the tile is R row segments of TE contiguous floats (consecutive
// matrices are contiguous, so for small n the tile is one contiguous run); on
// the interleaved side every 32-matrix group (never split by a chunk boundary,
// C % 32 == 0) gives TE segments of 32 contiguous floats -- one 128-B line
// each.  Both sides are fully coalesced; the transposition goes through a
// padded shared tile (odd row pitch: conflict-free both ways).  The grouping G
// is what keeps small n efficient: one CTA per 32 matrices would move only
// 128*E bytes.  Pad lanes are never touched.
#include <cuda_runtime.h>
#include <stdint.h>

namespace bsp {

constexpr int CV_THREADS = 256;
constexpr int CV_TILE = 4096;    // max floats per CTA tile
constexpr int CV_TE = 128;       // max elements per tile
constexpr int CV_GMAX = 128;     // max 32-matrix groups per tile

// dir 0: canonical -> interleaved; dir 1: interleaved -> canonical
template <int DIR>
__global__ void __launch_bounds__(CV_THREADS)
convert_kernel(const float *__restrict__ src, float *__restrict__ dst, int64_t batch, int64_t C, int E,
               int TE, int G, int elem_tiles) {
    extern __shared__ float tile[];                 // [R][ld]
    __shared__ int64_t gbase[CV_GMAX];              // interleaved offset of each group's lane 0
    const int R = 32 * G;
    const int ld = (TE & 1) ? TE : TE + 1;
    const int64_t t = blockIdx.x;
    const int64_t rt = t / elem_tiles;              // matrix tile
    const int te = (int)(t - rt * elem_tiles);      // element tile
    const int64_t m0 = rt * R;                      // first matrix of the tile
    const int e0 = te * TE;
    const int ecount = (E - e0) < TE ? (E - e0) : TE;
    const int rcount = (int)((batch - m0) < R ? (batch - m0) : R);
    for (int g = threadIdx.x; g < G; g += CV_THREADS) {
        const int64_t m = m0 + 32 * g;
        gbase[g] = (m / C) * C * (int64_t)E + (m % C);
    }
    const int n_el = R * ecount;
    // idx / ecount without a division: idx < 2^14 and ecount <= 128, so
    // (idx * mg) >> 22 with mg = 2^22/ecount + 1 is exact (error < 1/256).
    const uint32_t mg = (1u << 22) / (uint32_t)ecount + 1u;
    const int rmask = R - 1, rshift = __ffs(R) - 1;
    __syncthreads();

    for (int base = 0; base < n_el; base += CV_THREADS * 8) {
        float v[8];
#pragma unroll
        for (int k = 0; k < 8; ++k) {                // 8 independent loads in flight per thread
            const int idx = base + threadIdx.x + k * CV_THREADS;
            if (DIR == 0) {
                const int r = (int)(((uint32_t)idx * mg) >> 22), e = idx - r * ecount;
                v[k] = (idx < n_el && r < rcount) ? src[(m0 + r) * E + e0 + e] : 0.0f;
            } else {
                const int r = idx & rmask, e = idx >> rshift;
                v[k] = (idx < n_el && r < rcount) ? src[gbase[r >> 5] + (int64_t)(e0 + e) * C + (r & 31)] : 0.0f;
            }
        }
#pragma unroll
        for (int k = 0; k < 8; ++k) {
            const int idx = base + threadIdx.x + k * CV_THREADS;
            if (idx < n_el) {
                if (DIR == 0) {
                    const int r = (int)(((uint32_t)idx * mg) >> 22), e = idx - r * ecount;
                    tile[r * ld + e] = v[k];
                } else {
                    const int r = idx & rmask, e = idx >> rshift;
                    tile[r * ld + e] = v[k];
                }
            }
        }
    }
    __syncthreads();
    for (int idx = threadIdx.x; idx < n_el; idx += CV_THREADS) {
        if (DIR == 0) {
            const int r = idx & rmask, e = idx >> rshift;     // lanes -> consecutive matrices
            if (r < rcount) dst[gbase[r >> 5] + (int64_t)(e0 + e) * C + (r & 31)] = tile[r * ld + e];
        } else {
            const int r = (int)(((uint32_t)idx * mg) >> 22), e = idx - r * ecount;
            if (r < rcount) dst[(m0 + r) * E + e0 + e] = tile[r * ld + e];
        }
    }
}

cudaError_t launch_convert(int dir, int n, int64_t batch, int64_t C, const float *src, float *dst,
                           cudaStream_t stream) {
    const int E = n * n;
    const int TE = E < CV_TE ? E : CV_TE;
    int G = CV_TILE / (32 * TE);
    if (G < 1) G = 1;
    if (G > CV_GMAX) G = CV_GMAX;
    while (G & (G - 1)) G &= G - 1;                 // power of two: r = idx & (R-1)
    const int R = 32 * G;
    const int ld = (TE & 1) ? TE : TE + 1;
    const int64_t row_tiles = (batch + R - 1) / R;
    const int elem_tiles = (E + TE - 1) / TE;
    const int64_t blocks = row_tiles * elem_tiles;
    if (blocks > 0x7fffffffLL) return cudaErrorInvalidConfiguration;
    const size_t sm = (size_t)R * ld * sizeof(float);
    if (dir == 0)
        convert_kernel<0><<<(unsigned)blocks, CV_THREADS, sm, stream>>>(src, dst, batch, C, E, TE, G, elem_tiles);
    else
        convert_kernel<1><<<(unsigned)blocks, CV_THREADS, sm, stream>>>(src, dst, batch, C, E, TE, G, elem_tiles);
    return cudaGetLastError();
}

}  // namespace bsp
