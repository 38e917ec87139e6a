// Issue-rate probe: 3-register FFMA vs packed FFMA2 (fma.rn.f32x2) on one B200.
// Same number of FMAs either way; 16 independent accumulator lanes per thread;
// prints FMA/clk/SM for each form.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 scripts/r02/ffma2_probe.cu -o /tmp/ffma2 && /tmp/ffma2
#include <cstdio>
#include "../../paper_conf_ipps_gatesklpd17_b200/csrc/common.cuh"

template <bool PACKED>
__global__ void __launch_bounds__(256) probe(float *out, float l0, float m0, int iters) {
    float c[16];
#pragma unroll
    for (int i = 0; i < 16; ++i) c[i] = threadIdx.x * 1e-3f + i;
    float l = l0 + threadIdx.x * 1e-7f, m[16];
#pragma unroll
    for (int i = 0; i < 16; ++i) m[i] = m0 + i * 1e-6f;
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int i = 0; i < 16; i += 2) {
            if (PACKED) bsp::f_upd2(c[i], c[i + 1], l, m[i], m[i + 1]);
            else {
                c[i] = bsp::f_upd(c[i], l, m[i]);
                c[i + 1] = bsp::f_upd(c[i + 1], l, m[i + 1]);
            }
        }
    }
    float s = 0;
#pragma unroll
    for (int i = 0; i < 16; ++i) s += c[i];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

int main() {
    int sms = 0, clk = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);   // kHz
    float *out;
    cudaMalloc(&out, sizeof(float) * sms * 8 * 256);
    const int iters = 1 << 16;
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    for (int rep = 0; rep < 2; ++rep)
        for (int packed = 0; packed < 2; ++packed) {
            cudaEventRecord(a);
            if (packed) probe<true><<<sms * 8, 256>>>(out, 0.5f, 1e-3f, iters);
            else probe<false><<<sms * 8, 256>>>(out, 0.5f, 1e-3f, iters);
            cudaEventRecord(b);
            cudaEventSynchronize(b);
            float ms = 0;
            cudaEventElapsedTime(&ms, a, b);
            const double fmas = (double)sms * 8 * 256 * iters * 16;
            const double per_clk_sm = fmas / (ms * 1e-3) / (clk * 1e3) / sms;
            if (rep) printf("{\"form\": \"%s\", \"ms\": %.3f, \"fma_per_clk_per_sm\": %.1f, \"max_clock_khz\": %d}\n",
                            packed ? "FFMA2" : "FFMA", ms, per_clk_sm, clk);
        }
    return 0;
}
