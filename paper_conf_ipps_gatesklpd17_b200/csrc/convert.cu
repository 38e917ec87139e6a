// convert.cu -- layout conversion canonical <-> (chunked-)interleaved
// (PAPER.md:128 canonical; Figs. 7-8 interleaved; SURVEY
// §8(a) row a7).  Pure data movement: a batched transpose.  Matrix m's element
// e (= i + j*n, E = n*n elements) is at m*E in canonical storage and at
// (m/C)*C*E + e*C + m%C in interleaved storage.
//
// Work unit: a warp tile of one 32-matrix group (matrices 32g..32g+31, never
// split by a chunk boundary since C % 32 == 0, or C = batch) x 32 consecutive
// elements e0..e0+31.  On the interleaved side the tile is 32 lines of 32
// contiguous floats (128 B each); on the canonical side 32 row segments of
// 32 contiguous floats.  Every warp works alone (no block barriers): it loads
// the tile into registers, transposes it through its own 32x33 shared tile
// (pitch 33: conflict-free for every access pattern below) and stores it.
// The next tile's loads are issued before the current tile is stored, so each
// warp keeps 4 KB of reads in flight across its store phase.
//
// Access widths (chosen per launch, warp-uniform):
//   interleaved side  -- 128-bit (4 matrices x 1 element per lane) when C % 4
//                        == 0 and the group is full; else 32-bit, one matrix
//                        per lane, masked to the real matrices (pad lanes are
//                        never read or written);
//   canonical side    -- 128-bit (4 elements x 1 matrix per lane) when E % 4
//                        == 0 (n even: every row starts 16-B aligned); else
//                        32-bit, one element per lane.
// The previous version (block-wide smem tile, 32-bit accesses, __syncthreads
// between load and store phases) reached 2.4-2.9 TB/s (profiles/r01/c4_nsweep_r17.md).
#include <cuda_runtime.h>
#include <stdint.h>

namespace bsp {

constexpr int CV_THREADS = 256;
constexpr int CV_WARPS = CV_THREADS / 32;
constexpr int CV_PITCH = 33;

struct CvShape {
    int64_t batch, C;
    int E, slices;          // slices = ceil(E / 32)
    int64_t tiles;          // ceil(batch / 32) * slices
    int vec_i, vec_c;       // 128-bit interleaved / canonical accesses allowed
};

struct CvTile {
    int64_t m0, ib;         // first matrix of the group, interleaved offset of its lane 0
    int e0, te, rows;       // first element, elements in the tile (<= 32), real matrices (<= 32)
    bool full;              // rows == 32 and the 128-bit interleaved path is allowed
};

__device__ __forceinline__ CvTile cv_tile(const CvShape &s, int64_t t) {
    CvTile x;
    const int64_t g = t / s.slices;
    const int sl = (int)(t - g * s.slices);
    x.m0 = g * 32;
    x.ib = (x.m0 / s.C) * s.C * (int64_t)s.E + (x.m0 % s.C);
    x.e0 = sl * 32;
    x.te = min(32, s.E - x.e0);
    x.rows = (s.batch - x.m0) < 32 ? (int)(s.batch - x.m0) : 32;
    x.full = s.vec_i && x.rows == 32;
    return x;
}

__device__ __forceinline__ float4 ldg4(const float *p) {
    float4 v;
    asm volatile("ld.global.nc.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];"
                 : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w)
                 : "l"(p));
    return v;
}
__device__ __forceinline__ float ldg1(const float *p) {
    float v;
    asm volatile("ld.global.nc.L1::no_allocate.f32 %0, [%1];" : "=f"(v) : "l"(p));
    return v;
}
__device__ __forceinline__ void stg4(float *p, float a, float b, float c, float d) {
    asm volatile("st.global.cs.v4.f32 [%0], {%1,%2,%3,%4};" ::"l"(p), "f"(a), "f"(b), "f"(c), "f"(d)
                 : "memory");
}
__device__ __forceinline__ void stg1(float *p, float a) {
    asm volatile("st.global.cs.f32 [%0], %1;" ::"l"(p), "f"(a) : "memory");
}

// Register image of one tile (32 floats per lane).  Which (matrix, element)
// each register holds depends on the side and access width it was loaded with;
// put() writes it to the shared tile T[matrix][element].
struct CvRegs {
    float v[32];
};

// ---- canonical side ----------------------------------------------------------
// vec:    lane l, step k: matrix r = 4k + l/8, elements 4(l%8) .. +3
// scalar: lane l, step k: matrix r = k,        element  l
template <bool VEC>
__device__ __forceinline__ void canon_load(const CvShape &s, const CvTile &x, const float *__restrict__ src,
                                           int lane, CvRegs &R) {
    if (VEC) {
        const int rq = lane >> 3, c = (lane & 7) * 4;
        const bool ok_c = c < x.te;
#pragma unroll
        for (int k = 0; k < 8; ++k) {
            const int r = 4 * k + rq;
            if (ok_c && r < x.rows) {
                const float4 q = ldg4(src + (x.m0 + r) * s.E + x.e0 + c);
                R.v[4 * k] = q.x, R.v[4 * k + 1] = q.y, R.v[4 * k + 2] = q.z, R.v[4 * k + 3] = q.w;
            }
        }
    } else {
        const bool ok_e = lane < x.te;
#pragma unroll
        for (int k = 0; k < 32; ++k)
            if (ok_e && k < x.rows) R.v[k] = ldg1(src + (x.m0 + k) * s.E + x.e0 + lane);
    }
}
template <bool VEC>
__device__ __forceinline__ void canon_put(float *T, int lane, const CvRegs &R) {
    if (VEC) {
        const int rq = lane >> 3, c = (lane & 7) * 4;
#pragma unroll
        for (int k = 0; k < 8; ++k)
#pragma unroll
            for (int j = 0; j < 4; ++j) T[(4 * k + rq) * CV_PITCH + c + j] = R.v[4 * k + j];
    } else {
#pragma unroll
        for (int k = 0; k < 32; ++k) T[k * CV_PITCH + lane] = R.v[k];
    }
}
template <bool VEC>
__device__ __forceinline__ void canon_store(const CvShape &s, const CvTile &x, float *__restrict__ dst,
                                            const float *T, int lane) {
    if (VEC) {
        const int rq = lane >> 3, c = (lane & 7) * 4;
        if (c < x.te) {
#pragma unroll
            for (int k = 0; k < 8; ++k) {
                const int r = 4 * k + rq;
                const float *t = T + r * CV_PITCH + c;
                if (r < x.rows) stg4(dst + (x.m0 + r) * s.E + x.e0 + c, t[0], t[1], t[2], t[3]);
            }
        }
    } else {
        if (lane < x.te) {
#pragma unroll
            for (int k = 0; k < 32; ++k)
                if (k < x.rows) stg1(dst + (x.m0 + k) * s.E + x.e0 + lane, T[k * CV_PITCH + lane]);
        }
    }
}

// ---- interleaved side ----------------------------------------------------------
// full (vec): lane l, step k: matrices 4(l%8) .. +3, element 4k + l/8
// masked:     lane l, step k: matrix l, element k
__device__ __forceinline__ void inter_load(const CvShape &s, const CvTile &x, const float *__restrict__ src,
                                           int lane, CvRegs &R) {
    if (x.full) {
        const int eq = lane >> 3, c = (lane & 7) * 4;
#pragma unroll
        for (int k = 0; k < 8; ++k) {
            const int e = 4 * k + eq;
            if (e < x.te) {
                const float4 q = ldg4(src + x.ib + (int64_t)(x.e0 + e) * s.C + c);
                R.v[4 * k] = q.x, R.v[4 * k + 1] = q.y, R.v[4 * k + 2] = q.z, R.v[4 * k + 3] = q.w;
            }
        }
    } else {
        const bool ok = lane < x.rows;
#pragma unroll
        for (int k = 0; k < 32; ++k)
            if (ok && k < x.te) R.v[k] = ldg1(src + x.ib + (int64_t)(x.e0 + k) * s.C + lane);
    }
}
__device__ __forceinline__ void inter_put(float *T, bool full, int lane, const CvRegs &R) {
    if (full) {
        const int eq = lane >> 3, c = (lane & 7) * 4;
#pragma unroll
        for (int k = 0; k < 8; ++k)
#pragma unroll
            for (int j = 0; j < 4; ++j) T[(c + j) * CV_PITCH + 4 * k + eq] = R.v[4 * k + j];
    } else {
#pragma unroll
        for (int k = 0; k < 32; ++k) T[lane * CV_PITCH + k] = R.v[k];
    }
}
__device__ __forceinline__ void inter_store(const CvShape &s, const CvTile &x, float *__restrict__ dst,
                                            const float *T, int lane) {
    if (x.full) {
        const int eq = lane >> 3, c = (lane & 7) * 4;
#pragma unroll
        for (int k = 0; k < 8; ++k) {
            const int e = 4 * k + eq;
            if (e < x.te)
                stg4(dst + x.ib + (int64_t)(x.e0 + e) * s.C + c, T[c * CV_PITCH + e], T[(c + 1) * CV_PITCH + e],
                     T[(c + 2) * CV_PITCH + e], T[(c + 3) * CV_PITCH + e]);
        }
    } else if (lane < x.rows) {
#pragma unroll
        for (int k = 0; k < 32; ++k)
            if (k < x.te) stg1(dst + x.ib + (int64_t)(x.e0 + k) * s.C + lane, T[lane * CV_PITCH + k]);
    }
}

// DIR 0: canonical -> interleaved; DIR 1: interleaved -> canonical.
// Persistent: global warp w walks tiles w, w + W, ...  (consecutive warps take
// consecutive element slices of the same group: both sides stay local in DRAM).
template <int DIR, bool VEC_C>
__global__ void __launch_bounds__(CV_THREADS, 4)
convert_kernel(const float *__restrict__ src, float *__restrict__ dst, CvShape s) {
    __shared__ float tiles[CV_WARPS][32 * CV_PITCH];
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    float *T = tiles[wid];
    const int64_t W = (int64_t)gridDim.x * CV_WARPS;
    int64_t t = (int64_t)blockIdx.x * CV_WARPS + wid;
    if (t >= s.tiles) return;
    CvRegs R;
    CvTile x = cv_tile(s, t);
    if (DIR == 0) canon_load<VEC_C>(s, x, src, lane, R);
    else inter_load(s, x, src, lane, R);
    for (;;) {
        if (DIR == 0) canon_put<VEC_C>(T, lane, R);
        else inter_put(T, x.full, lane, R);
        __syncwarp();
        const int64_t tn = t + W;
        const bool more = tn < s.tiles;
        CvTile xn;
        if (more) {                              // next tile's loads in flight during the stores
            xn = cv_tile(s, tn);
            if (DIR == 0) canon_load<VEC_C>(s, xn, src, lane, R);
            else inter_load(s, xn, src, lane, R);
        }
        if (DIR == 0) inter_store(s, x, dst, T, lane);
        else canon_store<VEC_C>(s, x, dst, T, lane);
        if (!more) break;
        __syncwarp();                            // T free for the next tile
        t = tn;
        x = xn;
    }
}

template <int DIR, bool VEC_C>
static cudaError_t launch_dir(const CvShape &s, const float *src, float *dst, cudaStream_t stream) {
    int dev = 0, sms = 148, per_sm = 4;
    if (cudaGetDevice(&dev) == cudaSuccess) cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, convert_kernel<DIR, VEC_C>, CV_THREADS, 0);
    if (per_sm < 1) per_sm = 1;
    int64_t grid = (int64_t)sms * per_sm;        // persistent: exactly the resident CTAs
    const int64_t need = (s.tiles + CV_WARPS - 1) / CV_WARPS;
    if (grid > need) grid = need;
    if (grid < 1) grid = 1;
    convert_kernel<DIR, VEC_C><<<(unsigned)grid, CV_THREADS, 0, stream>>>(src, dst, s);
    return cudaGetLastError();
}

cudaError_t launch_convert(int dir, int n, int64_t batch, int64_t C, const float *src, float *dst,
                           cudaStream_t stream) {
    CvShape s;
    s.batch = batch;
    s.C = C;
    s.E = n * n;
    s.slices = (s.E + 31) / 32;
    s.tiles = ((batch + 31) / 32) * s.slices;
    // 128-bit accesses need 16-B aligned bases (the ABI guarantees 16-B aligned pointers)
    const bool al = ((uintptr_t)src % 16 == 0) && ((uintptr_t)dst % 16 == 0);
    s.vec_i = al && (C % 4 == 0);
    s.vec_c = al && (s.E % 4 == 0);
    if (dir == 0)
        return s.vec_c ? launch_dir<0, true>(s, src, dst, stream) : launch_dir<0, false>(s, src, dst, stream);
    return s.vec_c ? launch_dir<1, true>(s, src, dst, stream) : launch_dir<1, false>(s, src, dst, stream);
}

}  // namespace bsp
