// Exhaustive check of the branch-free sqrt.rn / rcp.rn fast paths
// (common.cuh f_sqrt_fast / f_rcp_fast) against the IEEE intrinsics
// __fsqrt_rn / __frcp_rn over ALL 2^32 float bit patterns: wherever the
// fast path reports ok, its bits must equal the intrinsic's.  Also counts
// how many positive normal inputs fall outside the fast range.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I include \
//        scripts/r02/verify_fast_sqrt_rcp.cu -o /tmp/vfsr && /tmp/vfsr
#include <cstdio>
#include <cstdint>
#include "../../paper_conf_ipps_gatesklpd17_b200/csrc/common.cuh"

__global__ void check(unsigned long long *bad, unsigned long long *slow) {
    unsigned long long b[2] = {0, 0}, s[2] = {0, 0};
    const uint64_t total = 1ull << 32;
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < total;
         i += (uint64_t)gridDim.x * blockDim.x) {
        const float x = __uint_as_float((uint32_t)i);
        bool ok1 = true, ok2 = true;
        const float fs = bsp::f_sqrt_fast(x, ok1);
        const float fr = bsp::f_rcp_fast(x, ok2);
        if (ok1 && __float_as_uint(fs) != __float_as_uint(__fsqrt_rn(x))) ++b[0];
        if (ok2 && __float_as_uint(fr) != __float_as_uint(__frcp_rn(x))) ++b[1];
        const bool posnorm = x >= 1.17549435e-38f && x <= 3.40282347e38f;
        if (posnorm && !ok1) ++s[0];
        if (posnorm && !ok2) ++s[1];
        // the full-range positive forms (f_sqrt_pos / f_rcp_pos): every positive
        // finite x, and the reciprocal of its root
        if (i >= 1 && i <= 0x7f7fffffu) {
            const float r = __fsqrt_rn(x);
            if (__float_as_uint(bsp::f_sqrt_pos(x)) != __float_as_uint(r)) ++b[0];
            if (__float_as_uint(bsp::f_rcp_pos(r)) != __float_as_uint(__frcp_rn(r))) ++b[1];
        }
    }
    atomicAdd(&bad[0], b[0]); atomicAdd(&bad[1], b[1]);
    atomicAdd(&slow[0], s[0]); atomicAdd(&slow[1], s[1]);
}

int main() {
    unsigned long long *d;
    cudaMalloc(&d, 4 * sizeof(unsigned long long));
    cudaMemset(d, 0, 4 * sizeof(unsigned long long));
    check<<<148 * 16, 256>>>(d, d + 2);
    unsigned long long h[4];
    cudaMemcpy(h, d, sizeof h, cudaMemcpyDeviceToHost);
    const cudaError_t e = cudaGetLastError();
    printf("{\"sqrt_mismatch\": %llu, \"rcp_mismatch\": %llu, \"sqrt_slow_posnormal\": %llu, "
           "\"rcp_slow_posnormal\": %llu, \"cuda\": \"%s\"}\n", h[0], h[1], h[2], h[3], cudaGetErrorString(e));
    return (h[0] || h[1] || e != cudaSuccess) ? 1 : 0;
}
