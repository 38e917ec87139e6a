// synth.cu -- on-device seeded synthetic SPD batches (bench / test utility).
// Independent implementation of the counter-based generator documented in
// include/bspotrf_synth.h and DESIGN.md "Input recipe"; the host module
// synth/__init__.py implements the same recipe and the GPU tests compare the
// two bit for bit.  One thread per matrix, written straight into the
// interleaved layout (coalesced stores).  Untimed; not part of the method.
#include <cuda_runtime.h>
#include <stdint.h>

#include "../../include/bspotrf_synth.h"

namespace bsp {

__device__ __forceinline__ uint64_t mix64(uint64_t z) {
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}
__device__ __forceinline__ uint64_t hash3(uint64_t seed, uint64_t b, uint64_t e) {
    const uint64_t hb = mix64(seed * 0x9E3779B97F4A7C15ull + b);
    return mix64(hb ^ (e * 0xD1B54A32D192ED03ull + 0x632BE59BD9B4E019ull));
}
__device__ __forceinline__ uint32_t fmix32(uint32_t x) {
    x ^= x >> 16;
    x *= 0x85EBCA6Bu;
    x ^= x >> 13;
    x *= 0xC2B2AE35u;
    x ^= x >> 16;
    return x;
}

constexpr uint64_t E_KB = 1ull << 20;
constexpr uint64_t E_Y = 1ull << 21;
constexpr uint64_t E_FAIL = 1ull << 22;
constexpr uint32_t UPPER_NAN = 0x7FC0FFEEu;

__device__ __forceinline__ int l0_entry(uint64_t seed, uint64_t b, int i, int j, int n) {
    const uint64_t h = hash3(seed, b, (uint64_t)(i + j * n));
    if (i == j) {
        const int sel = (int)(h % 3ull);
        return sel == 0 ? 1 : (sel == 1 ? 2 : 4);
    }
    return (int)(h % 7ull) - 3;
}

__global__ void synth_kernel(int n, int64_t batch, int64_t C, int64_t b0, int kind, uint64_t seed,
                             int upper, uint64_t fseed, int64_t fperiod, float *__restrict__ A) {
    const int64_t g = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (g >= batch) return;
    const uint64_t b = (uint64_t)(b0 + g);
    float *base = A + (g / C) * C * (int64_t)n * n + (g % C);

    int fail_k = -1;
    if (fperiod > 0) {
        const uint64_t hf = hash3(fseed, b, E_FAIL);
        if (hf % (uint64_t)fperiod == 0) fail_k = (int)((hf >> 32) % (uint64_t)n);
    }
    int kb = 0;
    uint32_t key = 0;
    if (kind == BSPOTRF_SYNTH_ALS) {
        kb = 1 + (int)(hash3(seed, b, E_KB) % (uint64_t)(2 * n));
        key = (uint32_t)(hash3(seed, b, E_Y) & 0xFFFFFFFFull);
    }

    for (int j = 0; j < n; ++j) {
        for (int i = j; i < n; ++i) {
            float v;
            if (kind == BSPOTRF_SYNTH_DD) {
                const uint64_t h = hash3(seed, b, (uint64_t)(i + j * n));
                if (i == j) v = (float)n + (float)(uint32_t)(h >> 48) * (1.0f / 65536.0f);
                else v = (float)((int32_t)(h >> 40) - (1 << 23)) * (1.0f / 8388608.0f);
            } else if (kind == BSPOTRF_SYNTH_ALS) {
                int32_t acc = 0;
                for (int r = 0; r < kb; ++r) {
                    const int32_t yi = (int32_t)(fmix32(key ^ ((uint32_t)(r * n + i) * 0x9E3779B1u)) >> 23) - 256;
                    const int32_t yj = (int32_t)(fmix32(key ^ ((uint32_t)(r * n + j) * 0x9E3779B1u)) >> 23) - 256;
                    acc += yi * yj;
                }
                v = (float)acc * (1.0f / 65536.0f);
                if (i == j) v = v + (float)kb * (1.0f / 16.0f);
            } else {  // L0
                int acc = 0;
                for (int p = 0; p <= j; ++p) acc += l0_entry(seed, b, i, p, n) * l0_entry(seed, b, j, p, n);
                v = (float)acc;
            }
            if (i == j && i == fail_k) {
                if (kind == BSPOTRF_SYNTH_L0) {
                    int acc = 0;
                    for (int p = 0; p < i; ++p) {
                        const int l = l0_entry(seed, b, i, p, n);
                        acc += l * l;
                    }
                    v = (float)(acc - 1);
                } else {
                    v = -1.0f;
                }
            }
            base[(int64_t)(i + j * n) * C] = v;
            if (i != j) {
                if (upper == BSPOTRF_UPPER_MIRROR) base[(int64_t)(j + i * n) * C] = v;
                else if (upper == BSPOTRF_UPPER_NAN) base[(int64_t)(j + i * n) * C] = __uint_as_float(UPPER_NAN);
            }
        }
    }
}

__global__ void fill_u32_kernel(uint32_t *p, int64_t n, uint32_t v) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
         i += (int64_t)gridDim.x * blockDim.x)
        p[i] = v;
}

}  // namespace bsp

extern "C" int bspotrf_synth_generate(int n, int64_t batch, int chunk, int64_t b0, int kind,
                                      uint64_t seed, int upper_mode, uint64_t fail_seed,
                                      int64_t fail_period, float *A, bspotrf_stream_t stream) {
    if (n < 0 || n > BSPOTRF_MAX_N) return -1;
    if (batch < 0) return -2;
    if (chunk < 0 || (chunk % 32) != 0) return -3;
    if (n == 0 || batch == 0) return 0;
    if (A == nullptr) return -4;
    if (kind < 0 || kind > 2) return -5;
    if (upper_mode < 0 || upper_mode > 2) return -6;
    const int64_t C = chunk > 0 ? chunk : batch;
    const int tpb = 128;
    bsp::synth_kernel<<<(unsigned)((batch + tpb - 1) / tpb), tpb, 0, (cudaStream_t)stream>>>(
        n, batch, C, b0, kind, seed, upper_mode, fail_seed, fail_period, A);
    return (int)cudaGetLastError();
}

extern "C" int bspotrf_fill_u32(float *A, int64_t elems, uint32_t value_bits, bspotrf_stream_t stream) {
    if (elems < 0) return -2;
    if (elems == 0) return 0;
    if (A == nullptr) return -1;
    bsp::fill_u32_kernel<<<148 * 8, 256, 0, (cudaStream_t)stream>>>(reinterpret_cast<uint32_t *>(A),
                                                                     elems, value_bits);
    return (int)cudaGetLastError();
}
