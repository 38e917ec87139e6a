// api.cu -- the C ABI of libbspotrf (include/bspotrf.h): argument checks,
// tuning-table lookup and dispatch to the per-(n, variant, chunk) kernel
// instances registered in gen/registry.inc.
#include <cuda_runtime.h>
#include <stdint.h>

#include <mutex>
#include <unordered_map>

#include "../../include/bspotrf.h"
#include "launch.h"

namespace bsp {

cudaError_t launch_convert(int dir, int n, int64_t batch, int64_t C, const float *src, float *dst,
                           cudaStream_t stream);

struct InstEntry {
    int variant;  // BSPOTRF_VARIANT_*
    int n;
    int param;    // SMEM/PANEL: S; TILE: NB; REG: min warps per SM (0 = none)
    int ct;       // compile-time chunk (0 = runtime stride)
    int tma;      // SMEM staging: 1 = TMA bulk, 0 = cp.async
    LaunchFn fn;
};

struct TuneEntry {
    int n;
    int chunk;  // exact chunk (0 = simple interleaved), or -1 = any other chunk
    bspotrf_tuning t;
};

struct SolveEntry {
    int kind;  // 0 = potrs (standalone), 1 = sposv (fused, REG), 2 = sposv (fused, PTMEM)
    int n;
    int nr;    // right-hand sides per pass (kind 2: 2*S + tma)
    int ct;
    PotrsFn potrs;
    SposvFn sposv;
};

#include "gen/registry.inc"      // kInstances[], kSolveInstances[]
#include "gen/tuning_table.inc"  // kTuning[]

static inline uint64_t key_of(int variant, int n, int param, int ct, int tma) {
    return ((uint64_t)variant << 40) | ((uint64_t)n << 32) | ((uint64_t)param << 20) |
           ((uint64_t)ct << 4) | (uint64_t)tma;
}

static std::once_flag g_once;
static std::unordered_map<uint64_t, LaunchFn> *g_inst = nullptr;
static std::unordered_map<uint64_t, const SolveEntry *> *g_solve = nullptr;

static inline uint64_t solve_key(int kind, int n, int nr, int ct) {
    return ((uint64_t)kind << 40) | ((uint64_t)n << 24) | ((uint64_t)nr << 12) | (uint64_t)ct;
}

static void init_tables() {
    std::call_once(g_once, [] {
        auto *m = new std::unordered_map<uint64_t, LaunchFn>();
        for (const auto &e : kInstances) (*m)[key_of(e.variant, e.n, e.param, e.ct, e.tma)] = e.fn;
        g_inst = m;
        auto *sv = new std::unordered_map<uint64_t, const SolveEntry *>();
        for (const auto &e : kSolveInstances) (*sv)[solve_key(e.kind, e.n, e.nr, e.ct)] = &e;
        g_solve = sv;
    });
}

static const SolveEntry *find_solve(int kind, int n, int nr, int chunk) {
    auto it = g_solve->find(solve_key(kind, n, nr, chunk == 32 ? 32 : 0));
    return it == g_solve->end() ? nullptr : it->second;
}

static LaunchFn find(int variant, int n, int param, int ct, int tma) {
    auto it = g_inst->find(key_of(variant, n, param, ct, tma));
    return it == g_inst->end() ? nullptr : it->second;
}

static bool default_tuning(int n, int chunk, bspotrf_tuning *t) {
    for (const auto &e : kTuning)       // exact (n, chunk) row first
        if (e.n == n && e.chunk == chunk) {
            *t = e.t;
            return true;
        }
    for (const auto &e : kTuning)       // then the row for "any other chunk"
        if (e.n == n && e.chunk == -1) {
            *t = e.t;
            return true;
        }
    return false;
}

// Resolve a tuning to a launcher.  Returns nullptr if unavailable.
static LaunchFn resolve(int n, int chunk, const bspotrf_tuning &t, int *tpb_out) {
    const bool tmpl_chunk = chunk == 32 || chunk == 64 || chunk == 128;
    *tpb_out = t.threads_per_block;
    switch (t.variant) {
    case BSPOTRF_VARIANT_REG:
        return find(BSPOTRF_VARIANT_REG, n, t.param, tmpl_chunk ? chunk : 0, 0);
    case BSPOTRF_VARIANT_SMEM:
    case BSPOTRF_VARIANT_PANEL: {
        int staging = t.staging;
        if (staging == 0) staging = tmpl_chunk ? 1 : 2;
        if (staging == 1) {
            if (!tmpl_chunk) return nullptr;
            *tpb_out = chunk;
            return find(t.variant, n, t.param, chunk, 1);
        }
        LaunchFn f = find(t.variant, n, t.param, chunk == 32 ? 32 : 0, 0);
        return f ? f : find(t.variant, n, t.param, 0, 0);
    }
    case BSPOTRF_VARIANT_PTMEM: {
        int staging = t.staging == 0 ? (chunk == 32 ? 1 : 2) : t.staging;
        *tpb_out = 128;
        // 1: TMA, fill batches of 5 tiles; 3: TMA, batches of 12 (instance tma = 3)
        if (staging == 1 || staging == 3)
            return chunk == 32 ? find(BSPOTRF_VARIANT_PTMEM, n, t.param, 32, staging) : nullptr;
        LaunchFn f = find(BSPOTRF_VARIANT_PTMEM, n, t.param, chunk == 32 ? 32 : 0, 0);
        return f ? f : find(BSPOTRF_VARIANT_PTMEM, n, t.param, 0, 0);
    }
    case BSPOTRF_VARIANT_RTMA:
    case BSPOTRF_VARIANT_RTMAP:
        *tpb_out = t.param * 32;
        return chunk == 32 ? find(t.variant, n, t.param, 32, 1) : nullptr;
    case BSPOTRF_VARIANT_TILE:
        return find(BSPOTRF_VARIANT_TILE, n, t.param, 0, 0);
    case BSPOTRF_VARIANT_REGX:
        return find(BSPOTRF_VARIANT_REGX, n, t.param, 0, t.staging == 1 ? 1 : 0);
    case BSPOTRF_VARIANT_QTM: {
        *tpb_out = 128;
        const int st = t.staging == 0 ? 2 : t.staging;   // 1/2: 256/512 TMEM columns, streamed;
                                                          // 3/4: the same, preloaded
        LaunchFn f = find(BSPOTRF_VARIANT_QTM, n, t.param, chunk == 32 ? 32 : 0, st);
        return f ? f : find(BSPOTRF_VARIANT_QTM, n, t.param, 0, st);
    }
    case BSPOTRF_VARIANT_RCW16: {
        *tpb_out = 512;
        LaunchFn f = find(BSPOTRF_VARIANT_RCW16, n, 0, chunk == 32 ? 32 : 0, 0);
        return f ? f : find(BSPOTRF_VARIANT_RCW16, n, 0, 0, 0);
    }
    case BSPOTRF_VARIANT_RCWD: {
        *tpb_out = 288;
        LaunchFn f = find(BSPOTRF_VARIANT_RCWD, n, 0, chunk == 32 ? 32 : 0, 0);
        return f ? f : find(BSPOTRF_VARIANT_RCWD, n, 0, 0, 0);
    }
    case BSPOTRF_VARIANT_RCWP: {
        *tpb_out = 256;
        LaunchFn f = find(BSPOTRF_VARIANT_RCWP, n, t.param, chunk == 32 ? 32 : 0, 0);
        return f ? f : find(BSPOTRF_VARIANT_RCWP, n, t.param, 0, 0);
    }
    case BSPOTRF_VARIANT_REGV:
        return find(BSPOTRF_VARIANT_REGV, n, 0, 0, 0);
    case BSPOTRF_VARIANT_RCW: {
        *tpb_out = 256;
        LaunchFn f = find(BSPOTRF_VARIANT_RCW, n, t.param, chunk == 32 ? 32 : 0, 0);
        return f ? f : find(BSPOTRF_VARIANT_RCW, n, t.param, 0, 0);
    }
    default:
        return nullptr;
    }
}

static int check_common(int n, int64_t batch, int chunk) {
    if (n < 0 || n > BSPOTRF_MAX_N) return -1;
    if (batch < 0) return -2;
    if (chunk < 0 || (chunk % 32) != 0) return -3;
    return 0;
}

}  // namespace bsp

using namespace bsp;

extern "C" int bspotrf_version(void) { return 10000; }

extern "C" int64_t batch_interleaved_elems(int n, int64_t batch, int chunk) {
    if (check_common(n, batch, chunk) != 0) return -1;
    if (n == 0 || batch == 0) return 0;
    const int64_t C = chunk > 0 ? chunk : batch;
    return ((batch + C - 1) / C) * C * (int64_t)n * n;
}

extern "C" int bspotrf_get_tuning(int n, int chunk, bspotrf_tuning *out) {
    const int rc = check_common(n, 1, chunk);
    if (rc != 0) return rc;
    if (out == nullptr) return -3;
    if (!default_tuning(n, chunk, out)) {
        out->variant = BSPOTRF_VARIANT_TILE;
        out->threads_per_block = 128;
        out->param = n <= 8 ? 4 : 8;
        out->staging = 0;
        out->carveout = 0;
    }
    return 0;
}

extern "C" int bspotrf_tuning_available(int n, int chunk, const bspotrf_tuning *tune) {
    const int rc = check_common(n, 1, chunk);
    if (rc != 0) return rc;
    if (tune == nullptr) return -3;
    if (n == 0) return 1;
    init_tables();
    bspotrf_tuning t = *tune;
    if (t.variant == BSPOTRF_VARIANT_AUTO) bspotrf_get_tuning(n, chunk, &t);
    int tpb = 0;
    return resolve(n, chunk, t, &tpb) != nullptr ? 1 : 0;
}

extern "C" int batch_spotrf_interleaved_ex(int n, int64_t batch, int chunk, float *A, int32_t *info,
                                           int32_t *nfailed, const bspotrf_tuning *tune,
                                           bspotrf_stream_t stream) {
    int rc = check_common(n, batch, chunk);
    if (rc != 0) return rc;
    if (n == 0 || batch == 0) return 0;
    if (A == nullptr || (reinterpret_cast<uintptr_t>(A) & 15u) != 0) return -4;
    if (info == nullptr) return -5;
    init_tables();
    bspotrf_tuning t;
    if (tune) {
        t = *tune;
        if (t.variant == BSPOTRF_VARIANT_AUTO) bspotrf_get_tuning(n, chunk, &t);
        if (t.threads_per_block < 0 || t.threads_per_block > 1024 || (t.threads_per_block % 32) != 0)
            return -7;
        if (t.carveout < 0 || t.carveout > 100) return -7;
    } else {
        bspotrf_get_tuning(n, chunk, &t);
    }
    int tpb = 0;
    LaunchFn fn = resolve(n, chunk, t, &tpb);
    if (fn == nullptr && tune == nullptr &&
        (t.variant == BSPOTRF_VARIANT_SMEM || t.variant == BSPOTRF_VARIANT_PANEL)) {
        t.staging = 2;                       // table row needs TMA: fall back to cp.async
        if (t.threads_per_block == 0) t.threads_per_block = 32;
        fn = resolve(n, chunk, t, &tpb);
    }
    if (fn == nullptr) return -7;
    FactorArgs a;
    a.A = A;
    a.info = info;
    a.nfailed = nfailed;
    a.batch = batch;
    a.cstride = chunk > 0 ? chunk : batch;
    a.tpb = tpb;
    a.stream = (cudaStream_t)stream;
    a.carveout = t.carveout;
    const cudaError_t e = fn(a);
    return e == cudaSuccess ? 0 : (int)e;
}

extern "C" int batch_spotrf_interleaved(int n, int64_t batch, int chunk, float *A, int32_t *info,
                                        bspotrf_stream_t stream) {
    return batch_spotrf_interleaved_ex(n, batch, chunk, A, info, nullptr, nullptr, stream);
}

static int convert_common(int dir, int n, int64_t batch, int chunk, const float *src, float *dst,
                          bspotrf_stream_t stream) {
    int rc = check_common(n, batch, chunk);
    if (rc != 0) return rc;
    if (n == 0 || batch == 0) return 0;
    if (src == nullptr) return -4;
    if (dst == nullptr) return -5;
    const int64_t inter = batch_interleaved_elems(n, batch, chunk);
    const int64_t canon = batch * (int64_t)n * n;
    const int64_t src_n = dir == 0 ? canon : inter, dst_n = dir == 0 ? inter : canon;
    const uintptr_t s0 = (uintptr_t)src, s1 = s0 + (uintptr_t)src_n * 4;
    const uintptr_t d0 = (uintptr_t)dst, d1 = d0 + (uintptr_t)dst_n * 4;
    if (s0 < d1 && d0 < s1) return -5;
    const cudaError_t e = launch_convert(dir, n, batch, chunk > 0 ? chunk : batch, src, dst,
                                         (cudaStream_t)stream);
    return e == cudaSuccess ? 0 : (int)e;
}

extern "C" int batch_canonical_to_interleaved(int n, int64_t batch, int chunk, const float *src,
                                              float *dst, bspotrf_stream_t stream) {
    return convert_common(0, n, batch, chunk, src, dst, stream);
}

extern "C" int batch_interleaved_to_canonical(int n, int64_t batch, int chunk, const float *src,
                                              float *dst, bspotrf_stream_t stream) {
    return convert_common(1, n, batch, chunk, src, dst, stream);
}

extern "C" int64_t batch_interleaved_rhs_elems(int n, int nrhs, int64_t batch, int chunk) {
    if (check_common(n, batch, chunk) != 0 || nrhs < 0) return -1;
    if (n == 0 || nrhs == 0 || batch == 0) return 0;
    const int64_t C = chunk > 0 ? chunk : batch;
    return ((batch + C - 1) / C) * C * (int64_t)n * nrhs;
}

// Standalone solve in groups of 4 / 2 / 1 right-hand sides (L re-read per group).
static int potrs_groups(const SolveArgs &a, int n, int chunk) {
    int rhs0 = 0;
    while (rhs0 < a.nrhs) {
        const int rem = a.nrhs - rhs0;
        const SolveEntry *e = nullptr;
        int nr = 0;
        for (int cand : {4, 2, 1}) {
            if (cand > rem) continue;
            e = find_solve(0, n, cand, chunk);
            if (e) {
                nr = cand;
                break;
            }
        }
        if (e == nullptr) return -7;
        const cudaError_t err = e->potrs(a, rhs0);
        if (err != cudaSuccess) return (int)err;
        rhs0 += nr;
    }
    return 0;
}

extern "C" int batch_spotrs_interleaved(int n, int nrhs, int64_t batch, int chunk, const float *L,
                                        float *B, bspotrf_stream_t stream) {
    if (n < 0 || n > BSPOTRF_MAX_N) return -1;
    if (nrhs < 0) return -2;
    if (batch < 0) return -3;
    if (chunk < 0 || (chunk % 32) != 0) return -4;
    if (n == 0 || nrhs == 0 || batch == 0) return 0;
    if (L == nullptr) return -5;
    if (B == nullptr) return -6;
    init_tables();
    SolveArgs a{const_cast<float *>(L), B, nullptr, nullptr, batch, chunk > 0 ? chunk : batch, nrhs,
                (cudaStream_t)stream};
    return potrs_groups(a, n, chunk);
}

extern "C" int batch_sposv_interleaved(int n, int nrhs, int64_t batch, int chunk, float *A, float *B,
                                       int32_t *info, int32_t *nfailed, bspotrf_stream_t stream) {
    if (n < 0 || n > BSPOTRF_MAX_N) return -1;
    if (nrhs < 0) return -2;
    if (batch < 0) return -3;
    if (chunk < 0 || (chunk % 32) != 0) return -4;
    if (n == 0 || batch == 0) return 0;
    if (A == nullptr || (reinterpret_cast<uintptr_t>(A) & 15u) != 0) return -5;
    if (B == nullptr && nrhs > 0) return -6;
    if (info == nullptr) return -7;
    init_tables();
    SolveArgs a{A, B, info, nfailed, batch, chunk > 0 ? chunk : batch, nrhs, (cudaStream_t)stream};
    if (nrhs > 0) {
        if (const SolveEntry *e = find_solve(1, n, nrhs, chunk)) {   // fused: L never re-read
            const cudaError_t err = e->sposv(a);
            return err == cudaSuccess ? 0 : (int)err;
        }
        if (nrhs == 1) {                                  // fused on the PTMEM structure
            bspotrf_tuning t;
            bspotrf_get_tuning(n, chunk, &t);
            const bool tma_ok = chunk == 32;
            const SolveEntry *e = nullptr;
            if (t.variant == BSPOTRF_VARIANT_PTMEM)
                e = find_solve(2, n, 2 * t.param + (tma_ok && t.staging != 2 ? 1 : 0), chunk);
            for (int s : {16, 20, 24, 28, 12, 8}) {
                if (e == nullptr && tma_ok) e = find_solve(2, n, 2 * s + 1, chunk);
                if (e == nullptr) e = find_solve(2, n, 2 * s, chunk);
            }
            if (e != nullptr) {
                const cudaError_t err = e->sposv(a);
                return err == cudaSuccess ? 0 : (int)err;
            }
        }
    }
    // unfused: factor (tuning table), then solve the matrices whose factorization succeeded
    const int rc = batch_spotrf_interleaved_ex(n, batch, chunk, A, info, nfailed, nullptr, stream);
    if (rc != 0 || nrhs == 0) return rc;
    return potrs_groups(a, n, chunk);
}
