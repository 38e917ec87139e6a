// host_pipeline.cu -- batch_spotrf_interleaved_host: the end-to-end call on
// host-resident interleaved storage (include/bspotrf.h).
//
// Two paths.  (1) slab == 0 and both host buffers pinned (mapped): zero-copy,
// the factorization kernel reads and writes host memory directly over PCIe.
// (2) otherwise: the copy pipeline below.
//
// The batch is cut into slabs of whole chunks.  Each slab flows through three
// streams -- H2D copy, factorization kernel, D2H copy -- with three device
// buffers in rotation, so PCIe in both directions and the kernel overlap.
// Only the lower triangle crosses PCIe: in the chunked layout the lower part
// of column j of a chunk is one contiguous run of (n-j)*C floats, and the runs
// of consecutive chunks are n*n*C floats apart, so ONE cudaMemcpy2DAsync per
// column moves that column for every full chunk of the slab (pitch n*n*C).
// A partial last chunk is copied lane-exactly (its pad lanes are not touched,
// reading R7).  In the simple interleaved layout (chunk 0) column j of a slab
// of matrices [b0, b0+cnt) is n-j rows of cnt floats, batch floats apart: one
// 2-D copy per column into a device buffer laid out simple-interleaved with
// stride cnt.
#include <cuda_runtime.h>
#include <stdint.h>

#include <algorithm>
#include <mutex>

#include "../../include/bspotrf.h"

namespace {

struct Slot {
    float *dA = nullptr;
    int32_t *dinfo = nullptr;
    cudaEvent_t h2d_done = nullptr, cmp_done = nullptr, d2h_done = nullptr;
    bool used = false;
};

cudaError_t copy_lower(int n, int64_t C, int chunk, int64_t batch, int64_t b0, int64_t cnt,
                       float *host, float *dev, cudaMemcpyKind kind, cudaStream_t s) {
    const int64_t E = (int64_t)n * n;
    cudaError_t e = cudaSuccess;
    if (chunk > 0) {
        const int64_t q0 = b0 / C;                       // first chunk of the slab
        const int64_t full = cnt / C;                    // full chunks
        const int64_t tail = cnt - full * C;             // lanes of a partial chunk
        float *hbase = host + q0 * C * E;
        for (int j = 0; j < n && e == cudaSuccess; ++j) {
            const int64_t off = (int64_t)(j + j * n) * C;
            const size_t pitch = (size_t)(C * E * 4);
            if (full > 0) {
                if (kind == cudaMemcpyHostToDevice)
                    e = cudaMemcpy2DAsync(dev + off, pitch, hbase + off, pitch,
                                          (size_t)((n - j) * C * 4), (size_t)full, kind, s);
                else
                    e = cudaMemcpy2DAsync(hbase + off, pitch, dev + off, pitch,
                                          (size_t)((n - j) * C * 4), (size_t)full, kind, s);
            }
            if (e == cudaSuccess && tail > 0) {
                const int64_t toff = full * C * E + off;
                if (kind == cudaMemcpyHostToDevice)
                    e = cudaMemcpy2DAsync(dev + toff, (size_t)C * 4, hbase + toff, (size_t)C * 4,
                                          (size_t)tail * 4, (size_t)(n - j), kind, s);
                else
                    e = cudaMemcpy2DAsync(hbase + toff, (size_t)C * 4, dev + toff, (size_t)C * 4,
                                          (size_t)tail * 4, (size_t)(n - j), kind, s);
            }
        }
    } else {
        for (int j = 0; j < n && e == cudaSuccess; ++j) {
            const int64_t e0 = j + (int64_t)j * n;
            float *h = host + e0 * batch + b0;
            float *d = dev + e0 * cnt;
            if (kind == cudaMemcpyHostToDevice)
                e = cudaMemcpy2DAsync(d, (size_t)cnt * 4, h, (size_t)batch * 4, (size_t)cnt * 4,
                                      (size_t)(n - j), kind, s);
            else
                e = cudaMemcpy2DAsync(h, (size_t)batch * 4, d, (size_t)cnt * 4, (size_t)cnt * 4,
                                      (size_t)(n - j), kind, s);
        }
    }
    return e;
}

// Device view of pinned (page-locked, mapped) host memory, or false.
bool device_view(void *h, void **d) {
    cudaPointerAttributes at;
    if (cudaPointerGetAttributes(&at, h) != cudaSuccess) {
        cudaGetLastError();
        return false;
    }
    if (at.type != cudaMemoryTypeHost || at.devicePointer == nullptr) return false;
    *d = at.devicePointer;
    return true;
}

// Zero-copy path: the factorization kernel itself reads and writes the pinned
// host storage over PCIe (every warp access is one 128-B line of 32 matrices,
// and each thread has its whole triangle's loads in flight, so both PCIe
// directions stream at once).  TMA-staged variants are swapped for their
// per-thread-load forms (the bulk engine is not used on host memory).
// The library's own stream-ordered memory pool on the current device (one per
// device, created on first use, never destroyed).  Its release threshold is
// "keep everything", so the slab buffers of one host call are reused by the
// next without a cudaMalloc; the process-wide default pool is left untouched.
cudaError_t library_pool(cudaMemPool_t *out) {
    static std::mutex mu;
    static cudaMemPool_t pools[64] = {};
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return e;
    if (dev < 0 || dev >= 64) return cudaErrorInvalidDevice;
    std::lock_guard<std::mutex> g(mu);
    if (pools[dev] == nullptr) {
        cudaMemPoolProps props = {};
        props.allocType = cudaMemAllocationTypePinned;
        props.handleTypes = cudaMemHandleTypeNone;
        props.location.type = cudaMemLocationTypeDevice;
        props.location.id = dev;
        cudaMemPool_t p = nullptr;
        e = cudaMemPoolCreate(&p, &props);
        if (e != cudaSuccess) return e;
        uint64_t thr = UINT64_MAX;
        cudaMemPoolSetAttribute(p, cudaMemPoolAttrReleaseThreshold, &thr);
        pools[dev] = p;
    }
    *out = pools[dev];
    return cudaSuccess;
}

int zero_copy(int n, int64_t batch, int chunk, float *dA, int32_t *dinfo, int32_t *nfailed_out,
              cudaStream_t stream) {
    // Kernel choice for PCIe-resident data (scripts/zerocopy_probe.py on B200,
    // profiles/r01/zerocopy_probe.json): what matters is bytes in flight over
    // PCIe, not on-chip reuse.  n <= 20: REG, 128 threads (37 GB/s each way at
    // n=16); 20 < n <= 32: the PANEL split with TMA bulk staging (40 GB/s at
    // n=32; cp.async.bulk reads mapped host memory fine) where the chunk allows
    // it, else the table's choice with per-thread staging.
    bspotrf_tuning t;
    bspotrf_get_tuning(n, chunk, &t);
    if (n <= 20) {
        t = bspotrf_tuning{BSPOTRF_VARIANT_REG, 128, 0, 0};
    } else if (n <= 32 && (chunk == 32 || chunk == 64 || chunk == 128)) {
        t = bspotrf_tuning{BSPOTRF_VARIANT_PANEL, 0, n - 16 >= 4 ? ((n - 16 + 3) / 4) * 4 : 4, 1};
        if (n - t.param > 16 || t.param > n - 8) t.param = ((n - 12) / 4) * 4;
    } else {
        if (t.variant == BSPOTRF_VARIANT_RTMA) t = bspotrf_tuning{BSPOTRF_VARIANT_REG, 128, 0, 0};
        if (t.variant == BSPOTRF_VARIANT_SMEM || t.variant == BSPOTRF_VARIANT_PANEL) {
            t.staging = 2;
            if (t.threads_per_block == 0) t.threads_per_block = 32;
        }
        if (t.variant == BSPOTRF_VARIANT_PTMEM) t.staging = 2;
    }
    int32_t *dcount = nullptr;
    cudaMemPool_t pool = nullptr;
    cudaError_t e = library_pool(&pool);
    if (e == cudaSuccess) e = cudaMallocFromPoolAsync((void **)&dcount, sizeof(int32_t), pool, stream);
    if (e != cudaSuccess) return (int)e;
    int rc = 0;
    e = cudaMemsetAsync(dcount, 0, sizeof(int32_t), stream);
    if (e == cudaSuccess) {
        rc = batch_spotrf_interleaved_ex(n, batch, chunk, dA, dinfo, dcount, &t, (bspotrf_stream_t)stream);
        if (rc == 0 && nfailed_out)
            e = cudaMemcpyAsync(nfailed_out, dcount, sizeof(int32_t), cudaMemcpyDeviceToHost, stream);
    }
    cudaFreeAsync(dcount, stream);
    const cudaError_t e2 = cudaStreamSynchronize(stream);
    if (rc != 0) return rc;
    if (e != cudaSuccess) return (int)e;
    return e2 == cudaSuccess ? 0 : (int)e2;
}

}  // namespace

extern "C" int64_t batch_spotrf_host_bytes(int n, int64_t batch, int chunk) {
    if (n < 0 || n > BSPOTRF_MAX_N || batch < 0 || chunk < 0 || chunk % 32) return -1;
    return (int64_t)4 * n * (n + 1) / 2 * batch;
}

extern "C" int batch_spotrf_interleaved_host(int n, int64_t batch, int chunk, float *hA,
                                             int32_t *hinfo, int32_t *nfailed_out, int64_t slab,
                                             bspotrf_stream_t stream) {
    if (n < 0 || n > BSPOTRF_MAX_N) return -1;
    if (batch < 0) return -2;
    if (chunk < 0 || (chunk % 32) != 0) return -3;
    if (slab < 0) return -6;
    if (n == 0 || batch == 0) {
        if (nfailed_out) *nfailed_out = 0;
        return 0;
    }
    if (hA == nullptr) return -4;
    if (hinfo == nullptr) return -5;

    void *dA_view = nullptr, *dinfo_view = nullptr;
    if (slab == 0 && device_view(hA, &dA_view) && device_view(hinfo, &dinfo_view) &&
        (reinterpret_cast<uintptr_t>(dA_view) & 15u) == 0)
        return zero_copy(n, batch, chunk, (float *)dA_view, (int32_t *)dinfo_view, nfailed_out,
                         (cudaStream_t)stream);

    const int64_t C = chunk > 0 ? chunk : batch;
    const int64_t lower_bytes = (int64_t)4 * n * (n + 1) / 2;
    int64_t S = slab;
    if (S == 0) S = std::max<int64_t>(1, (int64_t)(32ll << 20) / lower_bytes);  // ~32 MB per slab
    if (chunk > 0) S = std::max<int64_t>(C, (S / C) * C);
    else S = std::max<int64_t>(32, ((S + 31) / 32) * 32);
    S = std::min<int64_t>(S, chunk > 0 ? ((batch + C - 1) / C) * C : batch);
    const int64_t nslabs = (batch + S - 1) / S;
    const int NS = (int)std::min<int64_t>(3, nslabs);
    const int64_t slab_elems = (chunk > 0 ? ((S + C - 1) / C) * C : S) * (int64_t)n * n;

    cudaError_t e = cudaSuccess;
    cudaStream_t sh = nullptr, sc = nullptr, sd = nullptr;
    cudaEvent_t start = nullptr;
    Slot slots[3];
    int32_t *dcount = nullptr;
    int rc = 0;
#define BSP_TRY(x)                       \
    do {                                 \
        e = (x);                         \
        if (e != cudaSuccess) goto done; \
    } while (0)

    BSP_TRY(cudaStreamCreateWithFlags(&sh, cudaStreamNonBlocking));
    BSP_TRY(cudaStreamCreateWithFlags(&sc, cudaStreamNonBlocking));
    BSP_TRY(cudaStreamCreateWithFlags(&sd, cudaStreamNonBlocking));
    BSP_TRY(cudaEventCreateWithFlags(&start, cudaEventDisableTiming));
    BSP_TRY(cudaEventRecord(start, (cudaStream_t)stream));
    BSP_TRY(cudaStreamWaitEvent(sh, start, 0));
    {
        cudaMemPool_t pool = nullptr;
        BSP_TRY(library_pool(&pool));
        BSP_TRY(cudaMallocFromPoolAsync((void **)&dcount, sizeof(int32_t), pool, sh));
        BSP_TRY(cudaMemsetAsync(dcount, 0, sizeof(int32_t), sh));
        for (int i = 0; i < NS; ++i) {
            BSP_TRY(cudaMallocFromPoolAsync((void **)&slots[i].dA, (size_t)slab_elems * 4, pool, sh));
            BSP_TRY(cudaMallocFromPoolAsync((void **)&slots[i].dinfo, (size_t)S * 4, pool, sh));
            BSP_TRY(cudaEventCreateWithFlags(&slots[i].h2d_done, cudaEventDisableTiming));
            BSP_TRY(cudaEventCreateWithFlags(&slots[i].cmp_done, cudaEventDisableTiming));
            BSP_TRY(cudaEventCreateWithFlags(&slots[i].d2h_done, cudaEventDisableTiming));
        }
    }
    for (int64_t s = 0; s < nslabs; ++s) {
        Slot &sl = slots[s % NS];
        const int64_t b0 = s * S;
        const int64_t cnt = std::min<int64_t>(S, batch - b0);
        if (sl.used) BSP_TRY(cudaStreamWaitEvent(sh, sl.d2h_done, 0));
        BSP_TRY(copy_lower(n, C, chunk, batch, b0, cnt, hA, sl.dA, cudaMemcpyHostToDevice, sh));
        BSP_TRY(cudaEventRecord(sl.h2d_done, sh));
        BSP_TRY(cudaStreamWaitEvent(sc, sl.h2d_done, 0));
        rc = batch_spotrf_interleaved_ex(n, cnt, chunk, sl.dA, sl.dinfo, dcount, nullptr,
                                         (bspotrf_stream_t)sc);
        if (rc != 0) goto done;
        BSP_TRY(cudaEventRecord(sl.cmp_done, sc));
        BSP_TRY(cudaStreamWaitEvent(sd, sl.cmp_done, 0));
        BSP_TRY(copy_lower(n, C, chunk, batch, b0, cnt, hA, sl.dA, cudaMemcpyDeviceToHost, sd));
        BSP_TRY(cudaMemcpyAsync(hinfo + b0, sl.dinfo, (size_t)cnt * 4, cudaMemcpyDeviceToHost, sd));
        BSP_TRY(cudaEventRecord(sl.d2h_done, sd));
        sl.used = true;
    }
    if (nfailed_out) {
        BSP_TRY(cudaStreamWaitEvent(sd, slots[(nslabs - 1) % NS].cmp_done, 0));
        BSP_TRY(cudaMemcpyAsync(nfailed_out, dcount, sizeof(int32_t), cudaMemcpyDeviceToHost, sd));
    }
    BSP_TRY(cudaStreamSynchronize(sd));
done:
    if (sh) cudaStreamSynchronize(sh);
    if (sc) cudaStreamSynchronize(sc);
    if (sd) cudaStreamSynchronize(sd);
    for (int i = 0; i < 3; ++i) {
        if (slots[i].dA) cudaFreeAsync(slots[i].dA, sh);
        if (slots[i].dinfo) cudaFreeAsync(slots[i].dinfo, sh);
        if (slots[i].h2d_done) cudaEventDestroy(slots[i].h2d_done);
        if (slots[i].cmp_done) cudaEventDestroy(slots[i].cmp_done);
        if (slots[i].d2h_done) cudaEventDestroy(slots[i].d2h_done);
    }
    if (dcount) cudaFreeAsync(dcount, sh);
    if (sh) cudaStreamSynchronize(sh);
    if (start) cudaEventDestroy(start);
    if (sh) cudaStreamDestroy(sh);
    if (sc) cudaStreamDestroy(sc);
    if (sd) cudaStreamDestroy(sd);
#undef BSP_TRY
    if (rc != 0) return rc;
    return e == cudaSuccess ? 0 : (int)e;
}
