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
// Which kernel runs (launch_convert): v1 (below) for the ragged last group and
// C % 4 != 0; v2 (128-bit both sides, paths A / B / D) for the full groups;
// for interleaved -> canonical, v4 (whole-group image, one bulk store) at
// E % 8 != 0, n = 7..30 and v3 (sector-aligned row streams) at odd n >= 31,
// n = 2 mod 4 >= 34 and n = 4 mod 8 >= 28 (profiles/r02/convert_v3.md).
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdlib.h>

namespace bsp {

constexpr int CV_THREADS = 256;
constexpr int CV_WARPS = CV_THREADS / 32;
constexpr int CV_PITCH = 33;

struct CvShape {
    int64_t batch, C;
    int E, slices;          // slices = ceil(E / 32)
    int64_t tiles;          // (ceil(batch / 32) - gbeg) * slices
    int64_t gbeg;           // first 32-matrix group handled (the v2 kernel takes the full ones)
    int vec_i, vec_c;       // 128-bit interleaved / canonical accesses allowed
};

struct CvTile {
    int64_t m0, ib;         // first matrix of the group, interleaved offset of its lane 0
    int e0, te, rows;       // first element, elements in the tile (<= 32), real matrices (<= 32)
    bool full;              // rows == 32 and the 128-bit interleaved path is allowed
};

__device__ __forceinline__ CvTile cv_tile(const CvShape &s, int64_t t) {
    CvTile x;
    const int64_t gt = t / s.slices;
    const int sl = (int)(t - gt * s.slices);
    const int64_t g = s.gbeg + gt;
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

// ============================================================================
// v2: 128-bit accesses on BOTH sides for every n (round 2; the v1 kernel above
// used 32-bit canonical accesses for odd n -- 3.2-5.0 TB/s -- and wasted lanes
// for n <= 4, where a 32-element tile holds E = n*n < 32 elements: 0.25-2.2 TB/s).
// Preconditions: full 32-matrix groups only, C % 4 == 0 (interleaved lines
// 16-B aligned), 16-B aligned bases; the v1 kernel takes the last partial group.
//
// A tile is P consecutive groups x an element slice [e0, e0 + es):
//   path A (E <= 25, n <= 5; E compile-time): P = floor(33 / (E + 1)) whole
//     groups -- on the canonical side ONE contiguous, 16-B aligned block of
//     32*P*E floats (a group starts at 128*g*E bytes), moved as float4s;
//   path B (E >= 36): P = 1, es <= ES (ES in {20,24,28,32}, slices balanced);
//     canonical row m's segment [m*E + e0, +es) is moved through the aligned
//     float4 "slots" covering it (phase = start % 4, 0 when E % 4 == 0): loads
//     read whole slots (the few edge floats belong to a neighbouring tile and
//     are discarded), stores write full slots with STG.128 and the (at most 2)
//     edge slots per row with predicated scalar stores.
// The interleaved side is pg*es lines of 32 floats (8 lanes x float4 per
// line, 4 lines per warp instruction).  Each warp transposes through its own
// [32P][ES+1] shared tile; the next tile's loads are in flight during the
// current tile's stores (as v1).
// ============================================================================
constexpr int CV2_TILE = 32 * 33;            // floats of one warp's shared tile

struct Cv2Shape {
    int64_t C, G, tiles;   // chunk stride, full groups, tiles
    int E, nsl, esw, es_last;   // n*n; path B: slices per group, slice width (<= ES), last slice
};

__device__ __forceinline__ int64_t cv2_line(const Cv2Shape &s, int64_t g) {   // interleaved lane-0 offset
    const int64_t m0 = g * 32;
    return (m0 / s.C) * s.C * (int64_t)s.E + (m0 % s.C);
}

// ---- path A: E compile-time, P whole groups per tile ------------------------
template <int E>
struct Cv2A {
    static constexpr int P = 33 / (E + 1);
    static constexpr int PITCH = E + 1;
    static constexpr int F4 = 8 * P * E;                 // float4s of a full tile's canonical block
    static constexpr int LD = (F4 + 31) / 32;            // per lane
    static constexpr int LINES = P * E;
    static constexpr int LK = (LINES + 3) / 4;           // line steps per lane
    // resident CTAs per SM to ask for: 3, or 2 where the held float4s
    // (next tile's loads) would not fit 85 registers without spilling
    static constexpr int MINB0 = LD >= 7 ? 2 : 3, MINB1 = LK >= 7 ? 2 : 3;
};

template <int DIR, int E>
__global__ void __launch_bounds__(CV_THREADS, DIR == 0 ? Cv2A<E>::MINB0 : Cv2A<E>::MINB1)
convert2a_kernel(const float *__restrict__ src, float *__restrict__ dst, Cv2Shape s) {
    using SA = Cv2A<E>;
    __shared__ float tiles[CV_WARPS][CV2_TILE];
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    float *T = tiles[wid];
    const int64_t W = (int64_t)gridDim.x * CV_WARPS;
    int64_t t = (int64_t)blockIdx.x * CV_WARPS + wid;
    if (t >= s.tiles) return;
    const int c4 = (lane & 7) * 4, lq = lane >> 3;
    float4 R[DIR == 0 ? SA::LD : SA::LK];
    auto ngroups = [&](int64_t tt) {
        const int64_t left = s.G - tt * SA::P;
        return left < SA::P ? (int)left : SA::P;
    };
    auto load = [&](int64_t tt) {
        const int64_t g0 = tt * SA::P;
        const int pg = ngroups(tt);
        if (DIR == 0) {                                   // canonical block, contiguous
            const float *b = src + g0 * 32 * E;
#pragma unroll
            for (int k = 0; k < SA::LD; ++k) {
                const int f = lane + 32 * k;
                if (f < 8 * pg * E) R[k] = ldg4(b + 4 * f);
            }
        } else {                                          // interleaved lines
#pragma unroll
            for (int k = 0; k < SA::LK; ++k) {
                const int li = 4 * k + lq;
                if (li < pg * E) {
                    const int gg = li / E, e = li - gg * E;
                    R[k] = ldg4(src + cv2_line(s, g0 + gg) + (int64_t)e * s.C + c4);
                }
            }
        }
    };
    load(t);
    for (;;) {
        const int pg = ngroups(t);
        const int64_t g0 = t * SA::P;
        if (DIR == 0) {
#pragma unroll
            for (int k = 0; k < SA::LD; ++k) {
                const int f = lane + 32 * k;
                if (f < 8 * pg * E) {
                    const float v[4] = {R[k].x, R[k].y, R[k].z, R[k].w};
#pragma unroll
                    for (int j = 0; j < 4; ++j) {
                        const int x = 4 * f + j, m = x / E, e = x - m * E;
                        T[m * SA::PITCH + e] = v[j];
                    }
                }
            }
        } else {
#pragma unroll
            for (int k = 0; k < SA::LK; ++k) {
                const int li = 4 * k + lq;
                if (li < pg * E) {
                    const int gg = li / E, e = li - gg * E;
                    const float v[4] = {R[k].x, R[k].y, R[k].z, R[k].w};
#pragma unroll
                    for (int j = 0; j < 4; ++j) T[(32 * gg + c4 + j) * SA::PITCH + e] = v[j];
                }
            }
        }
        __syncwarp();
        const int64_t tn = t + W;
        const bool more = tn < s.tiles;
        if (more) load(tn);
        if (DIR == 0) {
#pragma unroll
            for (int k = 0; k < SA::LK; ++k) {
                const int li = 4 * k + lq;
                if (li < pg * E) {
                    const int gg = li / E, e = li - gg * E;
                    const float *r = T + (32 * gg + c4) * SA::PITCH + e;
                    stg4(dst + cv2_line(s, g0 + gg) + (int64_t)e * s.C + c4, r[0], r[SA::PITCH],
                         r[2 * SA::PITCH], r[3 * SA::PITCH]);
                }
            }
        } else {
            float *b = dst + g0 * 32 * E;
#pragma unroll
            for (int k = 0; k < SA::LD; ++k) {
                const int f = lane + 32 * k;
                if (f < 8 * pg * E) {
                    float v[4];
#pragma unroll
                    for (int j = 0; j < 4; ++j) {
                        const int x = 4 * f + j, m = x / E, e = x - m * E;
                        v[j] = T[m * SA::PITCH + e];
                    }
                    stg4(b + 4 * f, v[0], v[1], v[2], v[3]);
                }
            }
        }
        if (!more) break;
        __syncwarp();
        t = tn;
    }
}

// ---- path B: slices of <= ES elements, one group per tile ---------------------
// Shared tile, phase-shifted rows: element idx of row R (matrix 32g+R) sits at
// x = ph_R + idx, ph_R = (row start) % 4, so the aligned float4 slots of the
// canonical row are aligned float4s of the tile (LDS/STS.128, no per-float
// scatter).  Slot index XOR (R >> 3) & 3 against bank conflicts on the
// interleaved side (pitch 52: 13 slots, XOR stays inside the row); measured
// offline: interleaved-side accesses conflict-free, canonical side <= 2-way.
constexpr int CV2B_PITCH = 52;
__device__ __forceinline__ int cv2b_at(int R, int x) {
    return R * CV2B_PITCH + 4 * ((x >> 2) ^ ((R >> 3) & 3)) + (x & 3);
}

template <int ES, bool ALIGNED>
struct Cv2B {
    static constexpr int SL = ALIGNED ? ES / 4 : ES / 4 + 1;   // float4 slots per row
    static constexpr int LD = SL;                              // canonical slots per lane
    static constexpr int LK = ES / 4;                          // line steps per lane
    static constexpr int MINB0 = 2, MINB1 = 2;   // 128 registers: per-lane slot tables + 9 float4s
};

template <int DIR, int ES, bool ALIGNED>
__global__ void __launch_bounds__(CV_THREADS, DIR == 0 ? Cv2B<ES, ALIGNED>::MINB0 : Cv2B<ES, ALIGNED>::MINB1)
convert2b_kernel(const float *__restrict__ src, float *__restrict__ dst, Cv2Shape s) {
    using SB = Cv2B<ES, ALIGNED>;
    extern __shared__ __align__(16) float cv2b_smem[];     // CV_WARPS x 32 x CV2B_PITCH (53 KB)
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    float *T = cv2b_smem + wid * (32 * CV2B_PITCH);
    const int64_t W = (int64_t)gridDim.x * CV_WARPS;
    int64_t t = (int64_t)blockIdx.x * CV_WARPS + wid;
    if (t >= s.tiles) return;
    const int c4 = (lane & 7) * 4, lq = lane >> 3;
    // Per-lane constants, hoisted out of the tile loop (the index arithmetic was
    // the bound: IMAD/LOP3/BRA ~52% of issue samples at n = 63, round 2):
    //  canonical slot k: row R, slot sl -> shared offset, row-start phase part
    //  (R*E mod 4) and the float offset R*E + 4*sl inside the group's block;
    //  interleaved side: rows c4 + j share the XOR key (c4 >> 3) & 3.
    // meta[k] = sl | (R*E mod 4) << 8, or -1 for a slot past row 31
    int soff[SB::LD], rowoff[SB::LD], meta[SB::LD];
#pragma unroll
    for (int k = 0; k < SB::LD; ++k) {
        const int i = lane + 32 * k, R = i / SB::SL, sl = i - R * SB::SL;
        const int Rc = R < 32 ? R : 0;
        soff[k] = cv2b_at(Rc, 4 * sl);
        rowoff[k] = Rc * s.E + 4 * sl;
        meta[k] = R < 32 ? (sl | (((Rc * s.E) & 3) << 8)) : -1;
    }
    auto slot_ok = [&](int k, int ph, int es) { return meta[k] >= 0 && 4 * (meta[k] & 0xff) < ph + es; };
    auto slot_ph = [&](int k, int e0) { return ALIGNED ? 0 : (((meta[k] >> 8) + e0) & 3); };
    const int key = (c4 >> 3) & 3;
    int jbase[4], jph[4];
#pragma unroll
    for (int j = 0; j < 4; ++j) {
        jbase[j] = (c4 + j) * CV2B_PITCH;
        jph[j] = ((c4 + j) * s.E) & 3;
    }
    // interleaved element li = 4k + lq of row c4 + j at x = ph_j + li
    auto iaddr = [&](int j, int k, int ph) {
        const int u = ph + lq;                            // 0..6
        return jbase[j] + (u & 3) + 4 * (((u >> 2) + k) ^ key);
    };
    float4 R4[DIR == 0 ? SB::LD : SB::LK];
    auto geom = [&](int64_t tt, int64_t &g, int &e0, int &es) {
        g = tt / s.nsl;
        const int sl = (int)(tt - g * s.nsl);
        if (ALIGNED) {                                    // float4-aligned slice starts
            e0 = sl * s.esw;
            es = sl == s.nsl - 1 ? s.es_last : s.esw;
        } else {                                          // proportional: widths differ by <= 1
            e0 = (int)((int64_t)sl * s.E / s.nsl);
            es = (int)((int64_t)(sl + 1) * s.E / s.nsl) - e0;
        }
    };
    auto load = [&](int64_t tt) {
        int64_t g;
        int e0, es;
        geom(tt, g, e0, es);
        if (DIR == 0) {                                   // canonical slots
            const float *gb = src + g * 32 * (int64_t)s.E + e0;
#pragma unroll
            for (int k = 0; k < SB::LD; ++k) {
                const int ph = slot_ph(k, e0);
                if (slot_ok(k, ph, es)) R4[k] = ldg4(gb + rowoff[k] - ph);
            }
        } else {                                          // interleaved lines
            const float *lb = src + cv2_line(s, g) + (int64_t)e0 * s.C + c4;
#pragma unroll
            for (int k = 0; k < SB::LK; ++k) {
                const int li = 4 * k + lq;
                if (li < es) R4[k] = ldg4(lb + (int64_t)li * s.C);
            }
        }
    };
    load(t);
    for (;;) {
        int64_t g;
        int e0, es;
        geom(t, g, e0, es);
        int ph4[4];
#pragma unroll
        for (int j = 0; j < 4; ++j) ph4[j] = ALIGNED ? 0 : ((jph[j] + e0) & 3);
        if (DIR == 0) {                                   // canonical slots -> tile (STS.128)
#pragma unroll
            for (int k = 0; k < SB::LD; ++k) {
                const int ph = slot_ph(k, e0);
                if (slot_ok(k, ph, es)) *reinterpret_cast<float4 *>(T + soff[k]) = R4[k];
            }
        } else {                                          // interleaved lines -> tile
#pragma unroll
            for (int k = 0; k < SB::LK; ++k) {
                if (4 * k + lq < es) {
                    const float v[4] = {R4[k].x, R4[k].y, R4[k].z, R4[k].w};
#pragma unroll
                    for (int j = 0; j < 4; ++j) T[iaddr(j, k, ph4[j])] = v[j];
                }
            }
        }
        __syncwarp();
        const int64_t tn = t + W;
        const bool more = tn < s.tiles;
        if (more) load(tn);
        if (DIR == 0) {                                   // tile -> interleaved lines
            float *lb = dst + cv2_line(s, g) + (int64_t)e0 * s.C + c4;
#pragma unroll
            for (int k = 0; k < SB::LK; ++k) {
                const int li = 4 * k + lq;
                if (li < es) {
                    float v[4];
#pragma unroll
                    for (int j = 0; j < 4; ++j) v[j] = T[iaddr(j, k, ph4[j])];
                    stg4(lb + (int64_t)li * s.C, v[0], v[1], v[2], v[3]);
                }
            }
        } else {                                          // tile -> canonical slots
            float *gb = dst + g * 32 * (int64_t)s.E + e0;
#pragma unroll
            for (int k = 0; k < SB::LD; ++k) {
                const int ph = slot_ph(k, e0);
                if (slot_ok(k, ph, es)) {
                    const float4 q = *reinterpret_cast<const float4 *>(T + soff[k]);
                    float *p = gb + rowoff[k] - ph;
                    const int i0 = 4 * (meta[k] & 0xff) - ph;   // element index of the slot's first float
                    if (ALIGNED || (i0 >= 0 && i0 + 4 <= es)) {
                        stg4(p, q.x, q.y, q.z, q.w);
                    } else {                              // edge slot: only this tile's floats
                        const float v[4] = {q.x, q.y, q.z, q.w};
#pragma unroll
                        for (int jj = 0; jj < 4; ++jj)
                            if (i0 + jj >= 0 && i0 + jj < es) stg1(p + jj, v[jj]);
                    }
                }
            }
        }
        if (!more) break;
        __syncwarp();
        t = tn;
    }
}

// ---- interleaved -> canonical at odd n (E % 4 != 0): row streams with carries
// In path B the two partial float4 slots of every row segment (unaligned slice
// edges) were stored as scalars, half-sector writes shared with the tile of the
// neighbouring slice (2.6-3.5 TB/s).  Here one warp runs ALL slices of a group
// in order, so a row's canonical output is one stream: the partial last slot of
// a slice stays in the shared tile (copied to the row's front) and completes the
// first slot of the next slice; the partial first slot of a row (it shares a
// float4 with the previous row's end) is kept in H and stored with that row's
// last slot.  Every store is a full, aligned STG.128.
constexpr int CV2D_WARP = 32 * CV2B_PITCH + 32 * 4;      // tile + per-row head buffer H

template <int ES>
__global__ void __launch_bounds__(CV_THREADS, 2)
convert2d_kernel(const float *__restrict__ src, float *__restrict__ dst, Cv2Shape s) {
    constexpr int SL = ES / 4 + 1;                       // float4 slots per row segment (phase <= 3)
    constexpr int LK = ES / 4;
    extern __shared__ __align__(16) float cv2d_smem[];
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    float *T = cv2d_smem + wid * CV2D_WARP;
    float *H = T + 32 * CV2B_PITCH;                      // H[R*4 + j]: head floats of row R
    const int64_t W = (int64_t)gridDim.x * CV_WARPS;
    int64_t g = (int64_t)blockIdx.x * CV_WARPS + wid;
    if (g >= s.G) return;
    const int c4 = (lane & 7) * 4, lq = lane >> 3;
    const int key = (c4 >> 3) & 3;
    auto slice = [&](int sl, int &e0, int &es) {
        e0 = (int)((int64_t)sl * s.E / s.nsl);
        es = (int)((int64_t)(sl + 1) * s.E / s.nsl) - e0;
    };
    auto iaddr = [&](int R, int x) { return R * CV2B_PITCH + 4 * ((x >> 2) ^ key) + (x & 3); };
    float4 R4[LK];
    auto load = [&](int64_t gg, int sl) {
        int e0, es;
        slice(sl, e0, es);
        const float *lb = src + cv2_line(s, gg) + (int64_t)e0 * s.C + c4;
#pragma unroll
        for (int k = 0; k < LK; ++k) {
            const int li = 4 * k + lq;
            if (li < es) R4[k] = ldg4(lb + (int64_t)li * s.C);
        }
    };
    int sl = 0;
    load(g, 0);
    for (;;) {
        int e0, es;
        slice(sl, e0, es);
        const bool first = sl == 0, last = sl == s.nsl - 1;
        // interleaved lines -> tile rows at x = ph_R + li (ph_R = carry length)
#pragma unroll
        for (int k = 0; k < LK; ++k) {
            const int li = 4 * k + lq;
            if (li < es) {
                const float v[4] = {R4[k].x, R4[k].y, R4[k].z, R4[k].w};
#pragma unroll
                for (int j = 0; j < 4; ++j) {
                    const int R = c4 + j;
                    T[iaddr(R, (((R * s.E + e0) & 3) + li))] = v[j];
                }
            }
        }
        __syncwarp();
        // next slice's (or group's) loads in flight during the stores
        int64_t gn = g;
        int sln = sl + 1;
        if (last) {
            gn = g + W;
            sln = 0;
        }
        const bool more = gn < s.G;
        if (more) load(gn, sln);
        // full slots of every row; the first slot of a row's first slice is its
        // head (-> H), the partial last slot is the carry (stays) -- except at
        // the last slice, where it is completed by the next row's head
        float *gb = dst + g * 32 * (int64_t)s.E;
#pragma unroll
        for (int k = 0; k < SL; ++k) {
            const int i = lane + 32 * k, R = i / SL, sl4 = i - R * SL;
            if (R < 32) {
                const int ph = (R * s.E + e0) & 3;
                const int end = ph + es;                  // floats of the row in the tile
                const int64_t a0 = (int64_t)R * s.E + e0 - ph;   // stream position of x = 0
                if (4 * sl4 + 4 <= end) {
                    const float *t4 = T + R * CV2B_PITCH + 4 * (sl4 ^ ((R >> 3) & 3));
                    if (first && sl4 == 0 && ph != 0) {
#pragma unroll
                        for (int j = 0; j < 4; ++j) H[R * 4 + j] = t4[j];   // head (j >= ph valid)
                    } else {
                        stg4(gb + a0 + 4 * sl4, t4[0], t4[1], t4[2], t4[3]);
                    }
                } else if (last && 4 * sl4 < end && R < 31) {
                    // tail (end % 4 floats) + the next row's head = one aligned float4
                    const int rem = end & 3;
                    const float *t4 = T + R * CV2B_PITCH + 4 * (sl4 ^ ((R >> 3) & 3));
                    float v[4];
#pragma unroll
                    for (int j = 0; j < 4; ++j) v[j] = j < rem ? t4[j] : H[(R + 1) * 4 + j];
                    stg4(gb + a0 + 4 * sl4, v[0], v[1], v[2], v[3]);
                }
            }
        }
        if (!more) break;
        __syncwarp();
        if (!last) {
            // carry: the row's partial last slot moves to the row's front (slot 0)
            // -- the next slice puts its data after it (its phase == the carry length)
            const int R = lane;
            const int end = ((R * s.E + e0) & 3) + es, rem = end & 3;
            if (rem) {
                const float *t4 = T + R * CV2B_PITCH + 4 * (((end >> 2)) ^ ((R >> 3) & 3));
                float *f4 = T + R * CV2B_PITCH + 4 * (0 ^ ((R >> 3) & 3));
                float v[3];
#pragma unroll
                for (int j = 0; j < 3; ++j) v[j] = t4[j];
#pragma unroll
                for (int j = 0; j < 3; ++j)
                    if (j < rem) f4[j] = v[j];
            }
            __syncwarp();
        }
        g = gn;
        sl = sln;
    }
}

// ---- v3: interleaved -> canonical, fixed 32-element slices, sector-aligned
// row streams (round 2) ---------------------------------------------------------
// Why.  The canonical side of a slice is 32 row segments that start wherever
// R*E + e0 falls.  When that is not a multiple of 8 floats (odd n, and every
// odd row at n = 2 mod 4), each segment begins and ends inside a 32-B DRAM
// sector that another tile (v2 path B: another warp) or a later instruction
// (convert2d) completes: 0.48-0.64 of HBM against 0.82-0.85 for n = 0 mod 4
// (j13 A/B).  Here a group row is cut into FIXED 32-element slices e0 = 32k
// (the last one E - 32(K-1) wide) and every row's tile is shifted by its
// SECTOR phase ph = (R*E) mod 8: tile x = ph + li, so tile x = 0 is a sector
// start of the canonical stream.  A slice then writes, per row, 4 whole sectors
// (x = 0..31) -- each sector as two adjacent lanes' float4s in ONE instruction
// -- and keeps x = 32..32+ph-1 (< 8 floats) as the carry that becomes x < ph
// of the next slice.  Only a unit's first partial sector and its last partial
// one are stored as scalars.  Phases are per-lane constants (fixed slices):
//   line side  (lane = l8 + 8*lq): rows 4*l8 + j, element li = 4*kk + lq;
//   slot side  rows lq + 4*k, float4 slot l8 (x = 4*l8..+3): ph takes two
//              values, by the parity of k (4*k*E mod 8);
//   carry      slots 8, 9 of row = lane.
// Shared tile: row R starts at R*P + 4*t(R >> 2) (rows 16-B aligned, x =
// 0..39 used); the per-row shift t and pitch P depend only on the class of E
// mod 8 (odd n: 1; n = 2 mod 4: 4, whose table also serves E = 0 mod 8) and
// make the line side conflict-free (the 8
// rows 4*l8 + j of one STS hit 8 disjoint 4-bank groups; found by exhaustive
// search); the slot side reads one row's 8 contiguous slots per quarter warp.
// All tile addresses are a per-lane base + a compile-time immediate.  (A first
// version with XOR-swizzled slots ran 765 warp instructions per 4-KB slice,
// IMAD/LOP3/LEA 58% of them, and 2.4-way conflicts on the line side: j14 ncu.)
// A work unit is slices [k0, k1) of one 32-matrix group (S segments per group:
// >= 16 units per warp); persistent warps, the next slice's loads in flight
// during the stores.
template <int EC>
struct Cv3Tile {
    static constexpr int P = EC == 1 ? 60 : 52;
    // t(l8), 4 bits each: E = 1 mod 8: 0,0,1,1,3,2,4,5; E = 4 mod 8: 0,0,1,1,2,2,3,3
    static constexpr uint32_t TP = EC == 1 ? 0x54231100u : 0x33221100u;
    __host__ __device__ static constexpr int t(int q) { return (int)((TP >> (4 * q)) & 15u); }
    __host__ __device__ static constexpr int row(int R) { return R * P + 4 * t(R >> 2); }
    static constexpr int WARP = 32 * P;
};

struct Cv3Shape {
    int64_t C, G, units;
    int E, K, WL, S;       // slices per row, last slice width, segments per group
};

template <int EC>
__global__ void __launch_bounds__(CV_THREADS, 3)
convert3_kernel(const float *__restrict__ src, float *__restrict__ dst, Cv3Shape s) {
    using TT = Cv3Tile<EC>;
    extern __shared__ __align__(16) float cv3_smem[];
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    float *T = cv3_smem + wid * TT::WARP;
    const int64_t W = (int64_t)gridDim.x * CV_WARPS;
    int64_t u = (int64_t)blockIdx.x * CV_WARPS + wid;
    if (u >= s.units) return;
    const int E = s.E;
    const int l8 = lane & 7, lq = lane >> 3, c4 = 4 * l8;
    // line side: rows 4*l8 + j, element 4*kk + lq at tile x = ph + 4*kk + lq
    float *Tl[4];
#pragma unroll
    for (int j = 0; j < 4; ++j) Tl[j] = T + TT::row(c4 + j) + (((c4 + j) * E) & 7) + lq;
    // slot side: rows lq + 4*k8 (row offset lq*P + compile-time), slot l8; the
    // sector phase of the row takes two values, by the parity of k8
    float *Ts = T + lq * TT::P + 4 * l8;
    const int ph0 = (lq * E) & 7, ph1 = (lq * E + 4 * E) & 7;
    const int so0 = lq * E - ph0 + 4 * l8, so1 = lq * E - ph1 + 4 * l8;
    // carry lane: row = lane, x = 32..39 -> x = 0..7
    const int phc = (lane * E) & 7;
    float *T8 = T + lane * TT::P + 4 * (int)((TT::TP >> (4 * (lane >> 2))) & 15u);
    const int coff = lane * E - phc + 32;
    const int64_t C4 = 4 * s.C;

    // a unit: group g, slices [k0, k1), interleaved offset lb of the group's lane 0
    auto unit = [&](int64_t uu, int64_t &g, int &k0, int &k1, int64_t &lb) {
        g = uu / s.S;
        const int sg = (int)(uu - g * s.S);
        k0 = (int)((int64_t)sg * s.K / s.S);
        k1 = (int)((int64_t)(sg + 1) * s.K / s.S);
        const int64_t m0 = g * 32;
        lb = (m0 / s.C) * s.C * (int64_t)E + m0 % s.C;
    };
    float4 R4[8];
    auto load = [&](int64_t lb, int k) {                   // interleaved lines 32k + 4kk + lq
        const int w = k == s.K - 1 ? s.WL : 32;
        const float *lp = src + lb + (int64_t)(32 * k + lq) * s.C + c4;
#pragma unroll
        for (int kk = 0; kk < 8; ++kk) {
            if (4 * kk + lq < w) R4[kk] = ldg4(lp);
            lp += C4;
        }
    };

    int64_t g, lb;
    int k0, k1;
    unit(u, g, k0, k1, lb);
    int k = k0;
    load(lb, k);
    for (;;) {
        const int w = k == s.K - 1 ? s.WL : 32, e0 = 32 * k;
        const bool first = k == k0, last = k == k1 - 1;
#pragma unroll
        for (int kk = 0; kk < 8; ++kk)                     // lines -> tile rows
            if (4 * kk + lq < w) {
                Tl[0][4 * kk] = R4[kk].x;
                Tl[1][4 * kk] = R4[kk].y;
                Tl[2][4 * kk] = R4[kk].z;
                Tl[3][4 * kk] = R4[kk].w;
            }
        __syncwarp();
        // next slice (or the next unit's first) in flight during the stores
        int64_t gn = g, lbn = lb;
        int kn = k + 1, k0n = k0, k1n = k1;
        bool more = true;
        if (last) {
            u += W;
            more = u < s.units;
            if (more) unit(u, gn, k0n, k1n, lbn);
            kn = k0n;
        }
        if (more) load(lbn, kn);
        // tile -> canonical: slot l8 of rows lq + 4k8, x valid in [lo, hi)
        float *cp = dst + g * 32 * (int64_t)E + e0;
        int lo[2], hi[2];
#pragma unroll
        for (int pp = 0; pp < 2; ++pp) {
            const int ph = pp ? ph1 : ph0;
            lo[pp] = first ? min(max(ph - c4, 0), 4) : 0;
            hi[pp] = last ? min(max(ph + w - c4, 0), 4) : 4;
        }
#pragma unroll
        for (int k8 = 0; k8 < 8; ++k8) {
            const float4 q = *reinterpret_cast<const float4 *>(Ts + 4 * k8 * TT::P + 4 * TT::t(k8));
            float *p = cp + ((k8 & 1) ? so1 : so0) + 4 * k8 * E;
            const int a = lo[k8 & 1], b = hi[k8 & 1];
            if (a == 0 && b == 4) {
                stg4(p, q.x, q.y, q.z, q.w);
            } else {
                const float v[4] = {q.x, q.y, q.z, q.w};
#pragma unroll
                for (int jj = 0; jj < 4; ++jj)
                    if (jj >= a && jj < b) stg1(p + jj, v[jj]);
            }
        }
        __syncwarp();                                      // slots 0, 1 read before the carry lands
        if (!last) {                                       // carry: x = 32..32+phc-1 -> x < phc
            if (phc) {
                *reinterpret_cast<float4 *>(T8) = *reinterpret_cast<const float4 *>(T8 + 32);
                if (phc > 4) *reinterpret_cast<float4 *>(T8 + 4) = *reinterpret_cast<const float4 *>(T8 + 36);
            }
        } else if (32 < phc + w) {                         // the unit ends inside x = 32..39
            const int rm = phc + w - 32;
#pragma unroll
            for (int jj = 0; jj < 7; ++jj)
                if (jj < rm) stg1(cp + coff + jj, T8[32 + jj]);
        }
        if (!more) break;
        __syncwarp();
        g = gn;
        lb = lbn;
        k = kn;
        k0 = k0n;
        k1 = k1n;
    }
}

// ---- v4: interleaved -> canonical at odd n, a whole-group image + ONE bulk store
// The canonical block of a 32-matrix group is 32*E contiguous floats (128*E
// bytes, 16-B aligned for any E).  A CTA loads the group's E interleaved lines
// (256 threads, two 32-line steps per warp in flight), puts them into a shared
// image of that block (row m = matrix at m*E; for odd E the 32 lanes of one STS
// hit 32 distinct banks: 4*l8*E mod 32 takes 8 distinct multiples of 4) and one
// thread writes the image with a single cp.async.bulk shared -> global: every
// sector of the canonical side is written whole, once, by the copy engine.  Two
// images (when they fit) let group g+1 load while group g's store drains.
__device__ __forceinline__ uint32_t cv4_smem_u32(const void *p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void cv4_bulk_s2g(void *dst, const void *src, uint32_t bytes) {
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst),
                 "r"(cv4_smem_u32(src)), "r"(bytes)
                 : "memory");
    asm volatile("cp.async.bulk.commit_group;" ::: "memory");
}
template <int K>
__device__ __forceinline__ void cv4_bulk_wait_read() {      // <= K bulk groups may still read smem
    asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(K) : "memory");
}

struct Cv4Shape {
    int64_t C, G;
    int E, WPG;            // warps per group (1, 2, 4, 8): ceil(E / 64) rounded up; 8 / WPG groups per CTA step
};

template <int NB>
__global__ void __launch_bounds__(CV_THREADS, 2)
convert4_kernel(const float *__restrict__ src, float *__restrict__ dst, Cv4Shape s) {
    extern __shared__ __align__(128) float cv4_smem[];
    const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
    const int E = s.E, WPG = s.WPG, GP = CV_WARPS / WPG;
    const int gi = w / WPG, wg = w - gi * WPG;            // group slot of this warp, warp within the group
    const bool leader = wg == 0 && lane == 0;             // issues (and waits for) the slot's bulk stores
    const int l8 = lane & 7, lq = lane >> 3, c4 = 4 * l8;
    const int step = 32 * WPG;                            // lines per group step
    int it = 0;
    for (int64_t g0 = (int64_t)blockIdx.x * GP; g0 < s.G; g0 += (int64_t)gridDim.x * GP, ++it) {
        const int64_t g = g0 + gi;
        float *img = cv4_smem + ((size_t)gi * NB + (NB == 1 ? 0 : (it & 1))) * 32 * E;
        if (leader) cv4_bulk_wait_read<NB - 1>();         // the store issued from this image has read it
        __syncthreads();
        if (g < s.G) {
            const int64_t m0 = g * 32;
            const float *lb = src + (m0 / s.C) * s.C * (int64_t)E + m0 % s.C + c4;
            float *r0 = img + c4 * E;                      // row 4*l8 (+ j*E for rows 4*l8 + j)
            for (int base = 32 * wg + lq; base < E; base += 2 * step) {
                float4 R[16];
#pragma unroll
                for (int kk = 0; kk < 16; ++kk) {
                    const int line = base + (kk >> 3) * step + 4 * (kk & 7);
                    if (line < E) R[kk] = ldg4(lb + (int64_t)line * s.C);
                }
#pragma unroll
                for (int kk = 0; kk < 16; ++kk) {
                    const int line = base + (kk >> 3) * step + 4 * (kk & 7);
                    if (line < E) {
                        r0[line] = R[kk].x;
                        r0[E + line] = R[kk].y;
                        r0[2 * E + line] = R[kk].z;
                        r0[3 * E + line] = R[kk].w;
                    }
                }
            }
        }
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");   // generic STS -> async-proxy read
        __syncthreads();
        if (leader && g < s.G) cv4_bulk_s2g(dst + g * 32 * (int64_t)E, img, (uint32_t)(128 * E));
    }
    if (leader) cv4_bulk_wait_read<0>();                  // the images outlive the last stores' reads
}

static cudaError_t launch_v4(int n, int64_t G, int64_t C, const float *src, float *dst, cudaStream_t stream) {
    Cv4Shape s;
    s.C = C;
    s.G = G;
    s.E = n * n;
    const int wpg = (s.E + 63) / 64;                      // a warp covers 64 lines per pass (two 32-line steps)
    s.WPG = wpg <= 1 ? 1 : (wpg <= 2 ? 2 : (wpg <= 4 ? 4 : 8));
    const size_t img = (size_t)128 * s.E * (CV_WARPS / s.WPG);   // one image per group slot
    const bool two = 2 * img <= (size_t)113 * 1024;
    const size_t smem = two ? 2 * img : img;
    auto kern = two ? convert4_kernel<2> : convert4_kernel<1>;
    int dev = 0, sms = 148, per_sm = 1;
    if (cudaGetDevice(&dev) == cudaSuccess) cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, CV_THREADS, smem);
    if (per_sm < 1) per_sm = 1;
    const int gp = CV_WARPS / s.WPG;
    int64_t grid = (int64_t)sms * per_sm;
    const int64_t need = (G + gp - 1) / gp;
    if (grid > need) grid = need;
    kern<<<(unsigned)grid, CV_THREADS, smem, stream>>>(src, dst, s);
    return cudaGetLastError();
}

template <typename K>
static cudaError_t launch_persistent(K kern, int64_t tiles, const float *src, float *dst, const Cv2Shape &s,
                                     cudaStream_t stream, size_t dyn_smem = 0) {
    int dev = 0, sms = 148, per_sm = 4;
    if (cudaGetDevice(&dev) == cudaSuccess) cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    if (dyn_smem > 0) {
        const cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)dyn_smem);
        if (e != cudaSuccess) return e;
    }
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, CV_THREADS, dyn_smem);
    if (per_sm < 1) per_sm = 1;
    int64_t grid = (int64_t)sms * per_sm;
    const int64_t need = (tiles + CV_WARPS - 1) / CV_WARPS;
    if (grid > need) grid = need;
    if (grid < 1) grid = 1;
    kern<<<(unsigned)grid, CV_THREADS, dyn_smem, stream>>>(src, dst, s);
    return cudaGetLastError();
}

template <int DIR>
static cudaError_t launch_v2(int n, int64_t G, int64_t C, const float *src, float *dst, cudaStream_t stream) {
    Cv2Shape s;
    s.C = C;
    s.G = G;
    s.E = n * n;
    if (s.E <= 25) {
        s.nsl = 1;
        s.es_last = s.E;
        s.esw = s.E;
        switch (n) {
#define BSP_CV2A(NN)                                                                       \
    case NN: {                                                                             \
        s.tiles = (G + Cv2A<NN * NN>::P - 1) / Cv2A<NN * NN>::P;                           \
        return launch_persistent(convert2a_kernel<DIR, NN * NN>, s.tiles, src, dst, s, stream); \
    }
            BSP_CV2A(1) BSP_CV2A(2) BSP_CV2A(3) BSP_CV2A(4) BSP_CV2A(5)
#undef BSP_CV2A
        default:
            return cudaErrorInvalidValue;
        }
    }
    s.nsl = (s.E + 31) / 32;
    const int per = (s.E + s.nsl - 1) / s.nsl;           // balanced slices of <= 32 elements
    const int ES = ((per + 3) / 4) * 4;                  // buffer width: 20, 24, 28 or 32
    // aligned rows (E % 4 == 0) keep slice starts on float4 boundaries; otherwise
    // slices are cut proportionally in the kernel (widths per-1 or per, no
    // near-empty tail slice, e.g. E = 961, 1089, 3969)
    s.esw = ES;
    if (s.E % 4 == 0) s.nsl = (s.E + ES - 1) / ES;
    s.es_last = s.E - (s.nsl - 1) * ES;
    s.tiles = G * s.nsl;
    const bool al = s.E % 4 == 0;
    constexpr size_t B_SMEM = (size_t)CV_WARPS * 32 * CV2B_PITCH * sizeof(float);
    constexpr size_t D_SMEM = (size_t)CV_WARPS * CV2D_WARP * sizeof(float);
    if (DIR == 1 && !al) {                                // row streams: a warp per group
#define BSP_CV2D(ESV) \
    if (ES == ESV) return launch_persistent(convert2d_kernel<ESV>, G, src, dst, s, stream, D_SMEM);
        BSP_CV2D(20) BSP_CV2D(24) BSP_CV2D(28) BSP_CV2D(32)
#undef BSP_CV2D
    }
#define BSP_CV2B(ESV)                                                                                    \
    if (ES == ESV)                                                                                       \
        return al ? launch_persistent(convert2b_kernel<DIR, ESV, true>, s.tiles, src, dst, s, stream, B_SMEM)   \
                  : launch_persistent(convert2b_kernel<DIR, ESV, false>, s.tiles, src, dst, s, stream, B_SMEM);
    BSP_CV2B(20) BSP_CV2B(24) BSP_CV2B(28) BSP_CV2B(32)
#undef BSP_CV2B
    return cudaErrorInvalidValue;
}

template <int EC>
static cudaError_t launch_v3(int n, int64_t G, int64_t C, const float *src, float *dst, cudaStream_t stream) {
    Cv3Shape s;
    s.C = C;
    s.G = G;
    s.E = n * n;
    s.K = (s.E + 31) / 32;
    s.WL = s.E - 32 * (s.K - 1);
    auto kern = convert3_kernel<EC>;
    constexpr size_t SMEM = (size_t)CV_WARPS * Cv3Tile<EC>::WARP * sizeof(float);
    int dev = 0, sms = 148, per_sm = 3;
    if (cudaGetDevice(&dev) == cudaSuccess) cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)SMEM);
    if (e != cudaSuccess) return e;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, CV_THREADS, SMEM);
    if (per_sm < 1) per_sm = 1;
    int64_t grid = (int64_t)sms * per_sm;
    // segments per group: >= 16 units per warp (balance), at most one per slice
    const int64_t warps = grid * CV_WARPS;
    int64_t S = (16 * warps + G - 1) / G;
    if (S > s.K) S = s.K;
    if (S < 1) S = 1;
    s.S = (int)S;
    s.units = G * S;
    const int64_t need = (s.units + CV_WARPS - 1) / CV_WARPS;
    if (grid > need) grid = need;
    kern<<<(unsigned)grid, CV_THREADS, SMEM, stream>>>(src, dst, s);
    return cudaGetLastError();
}

// v3 (fixed slices, constant phases) vs v2, per direction and n: see the
// choice in launch_convert.  BSPOTRF_CONVERT_PATH=v2|v3|v4 forces one (probes).
static int convert_path_override() {
    const char *v = getenv("BSPOTRF_CONVERT_PATH");
    if (!v || v[0] != 'v') return 0;
    return v[1] == '4' ? 4 : (v[1] == '3' ? 3 : (v[1] == '2' ? 2 : 0));
}

cudaError_t launch_convert(int dir, int n, int64_t batch, int64_t C, const float *src, float *dst,
                           cudaStream_t stream) {
    // n = 1: element (0,0) of matrix b sits at offset b in BOTH layouts
    // ((b/C)*C + b%C = b; pad lanes only follow the last real matrix): a copy
    if (n == 1) return cudaMemcpyAsync(dst, src, (size_t)batch * sizeof(float), cudaMemcpyDeviceToDevice, stream);
    // 128-bit accesses need 16-B aligned bases (the ABI guarantees 16-B aligned pointers)
    const bool al = ((uintptr_t)src % 16 == 0) && ((uintptr_t)dst % 16 == 0);
    int64_t gbeg = 0;
    // v2 for every full group (v1: the ragged last group, C % 4 != 0)
    const bool v2 = al && C % 4 == 0;
    if (v2) {
        const int64_t G = batch / 32;
        if (G > 0) {
            const int ov = convert_path_override();
            const int E = n * n;
            // interleaved -> canonical, per n class (profiles/r02/convert_v3.md, j19/j19b A/B):
            //   n = 7..30, E % 8 != 0  v4 (whole-group image, one bulk store per group)
            //   odd n >= 31         v3 (the image no longer leaves room for two per SM)
            //   n = 2 mod 4, >= 34  v3 (v2's odd rows start mid-sector)
            //   n = 4 mod 8, >= 28  v3 (rows 64-B but not 128-B aligned: v2 0.71-0.76)
            //   otherwise           v2
            const bool odd = E % 2 == 1;
            const bool def4 = E % 8 != 0 && n >= 7 && n <= 30;
            const bool def3 = (odd && n >= 31) || (E % 8 == 4 && n >= 10) || (E % 32 == 16 && n >= 28);
            const bool v4 = dir == 1 && E >= 36 && E <= 961 && E % 32 != 0 && (ov == 4 || (ov == 0 && def4));
            const bool v3 = dir == 1 && !v4 && E > 32 && (ov == 3 || (ov == 0 && def3));
            const cudaError_t e = v4 ? launch_v4(n, G, C, src, dst, stream) :
                                  v3 ? (E % 8 == 1 ? launch_v3<1>(n, G, C, src, dst, stream)
                                                   : launch_v3<4>(n, G, C, src, dst, stream))
                                     : (dir == 0 ? launch_v2<0>(n, G, C, src, dst, stream)
                                                 : launch_v2<1>(n, G, C, src, dst, stream));
            if (e != cudaSuccess) return e;
        }
        gbeg = G;
        if (G * 32 == batch) return cudaSuccess;
    }
    CvShape s;
    s.batch = batch;
    s.C = C;
    s.E = n * n;
    s.slices = (s.E + 31) / 32;
    s.gbeg = gbeg;
    s.tiles = ((batch + 31) / 32 - gbeg) * s.slices;
    s.vec_i = al && (C % 4 == 0);
    s.vec_c = al && (s.E % 4 == 0);
    if (dir == 0)
        return s.vec_c ? launch_dir<0, true>(s, src, dst, stream) : launch_dir<0, false>(s, src, dst, stream);
    return s.vec_c ? launch_dir<1, true>(s, src, dst, stream) : launch_dir<1, false>(s, src, dst, stream);
}

}  // namespace bsp
