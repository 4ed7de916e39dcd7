// api.cu -- host side of libbulkgcd: the C ABI of include/bulkgcd.h.
//
// Validation, stream-ordered device buffers, layout transforms, kernel
// launches (persistent grids sized to the SM count), hit-buffer overflow
// retry and the final (i, j) sort.  No compute happens on the host.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <numeric>
#include <vector>

#include "../../include/bulkgcd.h"
#include "factor.cuh"
#include "kernels.cuh"

using namespace bulkgcd;

namespace {

thread_local char g_err[512] = "";

int set_err(int code, const char *fmt, ...) {
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(g_err, sizeof g_err, fmt, ap);
    va_end(ap);
    return code;
}

#define CK(call)                                                                                   \
    do {                                                                                           \
        cudaError_t e_ = (call);                                                                   \
        if (e_ != cudaSuccess) {                                                                   \
            int code_ = (e_ == cudaErrorMemoryAllocation) ? BULKGCD_ENOMEM : BULKGCD_ECUDA;        \
            return set_err(code_, "%s:%d %s: %s", __FILE__, __LINE__, #call, cudaGetErrorString(e_)); \
        }                                                                                          \
    } while (0)

int words_for(uint32_t bits) {
    switch (bits) {
        case 512: return 16;
        case 1024: return 32;
        case 2048: return 64;
        case 4096: return 128;
        default: return 0;
    }
}

// Per-device one-time set-up (B5: the only global state is a lazily created per-device
// context).  One instance per call site: `run` executes f() once per device, under a
// mutex, and only records success -- a failed attempt is retried by the next call.
// Thread-safe; a process that drives several GPUs gets the set-up on every device.
struct PerDeviceOnce {
    std::mutex mu;
    bool done[64] = {};
    template <class F>
    int run(F f) {
        int dev = 0;
        if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) return f();
        std::lock_guard<std::mutex> lock(mu);
        if (done[dev]) return 0;
        int rc = f();
        if (rc == 0) done[dev] = true;
        return rc;
    }
};

int sm_count() {
    int dev = 0, n = 148;
    if (cudaGetDevice(&dev) == cudaSuccess) cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
    return n > 0 ? n : 148;
}

int device_check() {
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return set_err(BULKGCD_ENODEV, "no CUDA device: %s", cudaGetErrorString(e));
    int major = 0, minor = 0;
    cudaDeviceGetAttribute(&major, cudaDevAttrComputeCapabilityMajor, dev);
    cudaDeviceGetAttribute(&minor, cudaDevAttrComputeCapabilityMinor, dev);
    if (major != 10 || minor != 0)
        return set_err(BULKGCD_ENODEV, "device %d is sm_%d%d; libbulkgcd is built for sm_100a only", dev, major,
                       minor);
    // The host-buffer entry points allocate stream-ordered (cudaMallocAsync) per call; by
    // default the pool unmaps everything at each synchronisation, so a repeated call
    // re-maps its buffers (hundreds of MB for bulkgcd_pairs).  Keep up to 4 GiB cached
    // in the device's default pool (the per-device context of include/bulkgcd.h B5).
    static PerDeviceOnce pool_once;
    return pool_once.run([&]() -> int {
        cudaMemPool_t pool;
        if (cudaDeviceGetDefaultMemPool(&pool, dev) == cudaSuccess) {
            uint64_t keep = 4ull << 30;
            cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &keep);
        }
        return 0;
    });
}

// RAII stream-ordered device buffer.
struct DBuf {
    void *p = nullptr;
    cudaStream_t s = nullptr;
    DBuf() = default;
    DBuf(const DBuf &) = delete;
    ~DBuf() {
        if (p) cudaFreeAsync(p, s);
    }
    cudaError_t alloc(size_t bytes, cudaStream_t st) {
        s = st;
        return cudaMallocAsync(&p, bytes ? bytes : 16, st);
    }
    template <class T>
    T *as() const { return (T *)p; }
};

size_t pad32(size_t m) { return (m + 31) / 32 * 32; }

// Shared-memory-resident kernels: W = 128 always, other widths with BULKGCD_FLAG_SMEM,
// and the comparison algorithms (BULKGCD_FLAG_ALGO_*).
template <int W, int ALG>
int launch_pairs_smem_alg(const PairsArgs &a, int mode, bool stats, cudaStream_t st) {
    constexpr size_t smem = smem_operand_bytes<W>();
    static PerDeviceOnce attr_once;  // dynamic shared memory opt-in, per device
    if (int rc = attr_once.run([]() -> int {
            CK(cudaFuncSetAttribute(pairs_smem_kernel<W, true, true, ALG>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
            CK(cudaFuncSetAttribute(pairs_smem_kernel<W, true, true, ALG>, cudaFuncAttributePreferredSharedMemoryCarveout, 100));
            CK(cudaFuncSetAttribute(pairs_smem_kernel<W, true, false, ALG>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
            CK(cudaFuncSetAttribute(pairs_smem_kernel<W, true, false, ALG>, cudaFuncAttributePreferredSharedMemoryCarveout, 100));
            CK(cudaFuncSetAttribute(pairs_smem_kernel<W, false, true, ALG>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
            CK(cudaFuncSetAttribute(pairs_smem_kernel<W, false, true, ALG>, cudaFuncAttributePreferredSharedMemoryCarveout, 100));
            CK(cudaFuncSetAttribute(pairs_smem_kernel<W, false, false, ALG>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
            CK(cudaFuncSetAttribute(pairs_smem_kernel<W, false, false, ALG>, cudaFuncAttributePreferredSharedMemoryCarveout, 100));
            return 0;
        }))
        return rc;
    uint64_t cohorts = (a.m + 31) / 32;
    uint64_t grid = std::min<uint64_t>((uint64_t)sm_count() * smem_blocks<W>(), (cohorts + 1) / 2);
    if (grid == 0) return 0;
    if (mode == BULKGCD_MODE_RSA) {
        if (stats) pairs_smem_kernel<W, true, true, ALG><<<(unsigned)grid, SM_THREADS, smem, st>>>(a);
        else pairs_smem_kernel<W, true, false, ALG><<<(unsigned)grid, SM_THREADS, smem, st>>>(a);
    } else {
        if (stats) pairs_smem_kernel<W, false, true, ALG><<<(unsigned)grid, SM_THREADS, smem, st>>>(a);
        else pairs_smem_kernel<W, false, false, ALG><<<(unsigned)grid, SM_THREADS, smem, st>>>(a);
    }
    CK(cudaGetLastError());
    return 0;
}

template <int W>
int launch_pairs_smem(const PairsArgs &a, int mode, bool stats, unsigned flags, cudaStream_t st) {
    switch (flags & BULKGCD_FLAG_ALGO_MASK) {
        case BULKGCD_FLAG_ALGO_FAST_BINARY: return launch_pairs_smem_alg<W, ALG_FAST_BINARY>(a, mode, stats, st);
        case BULKGCD_FLAG_ALGO_BINARY: return launch_pairs_smem_alg<W, ALG_BINARY>(a, mode, stats, st);
        default: return launch_pairs_smem_alg<W, ALG_APPROX>(a, mode, stats, st);
    }
}

template <int W>
int launch_pairs(const uint32_t *dA, const uint32_t *dB, uint32_t *dG, size_t m, size_t m_pad, int mode,
                 uint32_t *d_iters, unsigned long long *scratch, unsigned flags, cudaStream_t st) {
    CK(cudaMemsetAsync(scratch, 0, 8 * sizeof(unsigned long long), st));
    PairsArgs a{dA, dB, dG, m, m_pad, scratch + 1, d_iters, scratch + 2, W * 16};
    bool stats_ = (flags & BULKGCD_FLAG_STATS) || d_iters;
    if constexpr (W >= 128) {
        return launch_pairs_smem<W>(a, mode, stats_, flags, st);
    } else {
    if (flags & (BULKGCD_FLAG_SMEM | BULKGCD_FLAG_ALGO_MASK)) return launch_pairs_smem<W>(a, mode, stats_, flags, st);
    uint64_t cohorts = (m + 31) / 32;
    uint64_t grid = std::min<uint64_t>((uint64_t)sm_count() * Occ<W, true>::blocks, (cohorts + WARPS_PER_CTA - 1) / WARPS_PER_CTA);
    if (grid == 0) return 0;
    bool stats = (flags & BULKGCD_FLAG_STATS) || d_iters;
    if (mode == BULKGCD_MODE_RSA) {
        if (stats) pairs_kernel<W, true, true><<<(unsigned)grid, THREADS, 0, st>>>(a);
        else pairs_kernel<W, true, false><<<(unsigned)grid, THREADS, 0, st>>>(a);
    } else {
        if (stats) pairs_kernel<W, false, true><<<(unsigned)grid, THREADS, 0, st>>>(a);
        else pairs_kernel<W, false, false><<<(unsigned)grid, THREADS, 0, st>>>(a);
    }
    CK(cudaGetLastError());
    return 0;
    }
}

template <int W, int ALG>
int launch_allpairs_smem_alg(const AllPairsArgs &a, bool stats, cudaStream_t st) {
    constexpr size_t smem = smem_operand_bytes<W>();
    static PerDeviceOnce attr_once;  // dynamic shared memory opt-in, per device
    if (int rc = attr_once.run([]() -> int {
            CK(cudaFuncSetAttribute(allpairs_smem_kernel<W, true, ALG>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
            CK(cudaFuncSetAttribute(allpairs_smem_kernel<W, true, ALG>, cudaFuncAttributePreferredSharedMemoryCarveout, 100));
            CK(cudaFuncSetAttribute(allpairs_smem_kernel<W, false, ALG>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
            CK(cudaFuncSetAttribute(allpairs_smem_kernel<W, false, ALG>, cudaFuncAttributePreferredSharedMemoryCarveout, 100));
            return 0;
        }))
        return rc;
    uint64_t warps = a.c_end - a.c_begin;
    uint64_t grid = std::min<uint64_t>((uint64_t)sm_count() * smem_blocks<W>(), (warps + 1) / 2);
    if (stats) allpairs_smem_kernel<W, true, ALG><<<(unsigned)grid, SM_THREADS, smem, st>>>(a);
    else allpairs_smem_kernel<W, false, ALG><<<(unsigned)grid, SM_THREADS, smem, st>>>(a);
    CK(cudaGetLastError());
    return 0;
}

template <int W>
int launch_allpairs_smem(const AllPairsArgs &a, bool stats, unsigned flags, cudaStream_t st) {
    switch (flags & BULKGCD_FLAG_ALGO_MASK) {
        case BULKGCD_FLAG_ALGO_FAST_BINARY: return launch_allpairs_smem_alg<W, ALG_FAST_BINARY>(a, stats, st);
        case BULKGCD_FLAG_ALGO_BINARY: return launch_allpairs_smem_alg<W, ALG_BINARY>(a, stats, st);
        default: return launch_allpairs_smem_alg<W, ALG_APPROX>(a, stats, st);
    }
}

template <int W>
int launch_allpairs(const uint32_t *dN, const uint32_t *dBlk, size_t n, uint64_t c0, uint64_t c1, uint32_t *dHits,
                    uint64_t cap, unsigned long long *counters, unsigned flags, cudaStream_t st) {
    CK(cudaMemsetAsync(counters, 0, 8 * sizeof(unsigned long long), st));
    if (c1 <= c0) return 0;
    AllPairsArgs a{dBlk, dN, n, c0, c1, counters + 1, dHits, cap, counters, counters + 2, W * 16, nullptr};
    if constexpr (W >= 128) {
        // the 4096-bit product path: the hybrid kernel (A in registers, B in shared memory);
        // BULKGCD_FLAG_SMEM and the comparison algorithms keep the shared-memory kernels
        if ((flags & BULKGCD_FLAG_SMEM) || (flags & BULKGCD_FLAG_ALGO_MASK))
            return launch_allpairs_smem<W>(a, (flags & BULKGCD_FLAG_STATS) != 0, flags, st);
        constexpr size_t smem = hybrid_smem_bytes<W>();
        static PerDeviceOnce attr_once;
        if (int rc = attr_once.run([]() -> int {
                CK(cudaFuncSetAttribute(allpairs_hybrid_kernel<W, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
                CK(cudaFuncSetAttribute(allpairs_hybrid_kernel<W, true>, cudaFuncAttributePreferredSharedMemoryCarveout, 100));
                CK(cudaFuncSetAttribute(allpairs_hybrid_kernel<W, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
                CK(cudaFuncSetAttribute(allpairs_hybrid_kernel<W, false>, cudaFuncAttributePreferredSharedMemoryCarveout, 100));
                return 0;
            }))
            return rc;
        uint64_t warps = c1 - c0;
        constexpr int wpc = HY_THREADS / 32;
        uint64_t grid = std::min<uint64_t>((uint64_t)sm_count() * HY_BLOCKS, (warps + wpc - 1) / wpc);
        if (flags & BULKGCD_FLAG_STATS) allpairs_hybrid_kernel<W, true><<<(unsigned)grid, HY_THREADS, smem, st>>>(a);
        else allpairs_hybrid_kernel<W, false><<<(unsigned)grid, HY_THREADS, smem, st>>>(a);
        CK(cudaGetLastError());
        return 0;
    } else {
    // the comparison algorithms run on the shared-memory kernels (per-lane pointer swap,
    // the paper's own design): (D) there measures 661 ms on cfg3 against 1,235 ms on
    // the register harness, where its frequent no-swap iterations leave the hot loop
    if ((flags & BULKGCD_FLAG_SMEM) || (flags & BULKGCD_FLAG_ALGO_MASK))
        return launch_allpairs_smem<W>(a, (flags & BULKGCD_FLAG_STATS) != 0, flags, st);
    uint64_t warps = c1 - c0;
    constexpr int wpc = ApCfg<W>::warps_per_cta;
    uint64_t grid = std::min<uint64_t>((uint64_t)sm_count() * ApCfg<W>::blocks, (warps + wpc - 1) / wpc);
    constexpr size_t smem = allpairs_smem_bytes<W>();
    // dynamic shared memory opt-in and the largest shared-memory carveout, per device: the
    // residency of these kernels is set by their per-warp staging buffers, and with small
    // CTAs the driver's default carveout can leave room for fewer of them than the
    // register budget allows
    static PerDeviceOnce attr_once;
    if (int rc = attr_once.run([]() -> int {
            CK(cudaFuncSetAttribute(allpairs_kernel<W, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
            CK(cudaFuncSetAttribute(allpairs_kernel<W, true>, cudaFuncAttributePreferredSharedMemoryCarveout, 100));
            CK(cudaFuncSetAttribute(allpairs_kernel<W, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
            CK(cudaFuncSetAttribute(allpairs_kernel<W, false>, cudaFuncAttributePreferredSharedMemoryCarveout, 100));
            return 0;
        }))
        return rc;
    // straggler buffers (allpairs_cutk): one per resident warp, from the device's default pool
    DBuf strag;
    if constexpr (allpairs_cutk<W>() > 0) {
        CK(strag.alloc(grid * ApCfg<W>::warps_per_cta * strag_words<W>() * STRAG_CAP * sizeof(uint32_t), st));
        a.strag = strag.as<uint32_t>();
    }
    if (flags & BULKGCD_FLAG_STATS) allpairs_kernel<W, true><<<(unsigned)grid, ApCfg<W>::threads, smem, st>>>(a);
    else allpairs_kernel<W, false><<<(unsigned)grid, ApCfg<W>::threads, smem, st>>>(a);
    CK(cudaGetLastError());
    return 0;
    }
}

int check_moduli(const uint32_t *N, size_t n, int W) {
    for (size_t i = 0; i < n; ++i) {
        const uint32_t *x = N + i * W;
        if ((x[0] & 1u) == 0)
            return set_err(BULKGCD_EINVAL, "modulus %zu is even (RSA mode needs odd moduli > 1)", i);
        bool gt1 = x[0] > 1;
        for (int k = 1; k < W && !gt1; ++k) gt1 = x[k] != 0;
        if (!gt1) return set_err(BULKGCD_EINVAL, "modulus %zu is 1 (RSA mode needs odd moduli > 1)", i);
    }
    return 0;
}

}  // namespace

extern "C" {

const char *bulkgcd_strerror(int code) {
    switch (code) {
        case BULKGCD_OK: return "ok";
        case BULKGCD_EINVAL: return "invalid argument";
        case BULKGCD_ENOMEM: return "out of memory";
        case BULKGCD_ECUDA: return "CUDA error";
        case BULKGCD_ENODEV: return "no sm_100 device";
        default: return "unknown error";
    }
}

const char *bulkgcd_last_error(void) { return g_err; }

int bulkgcd_device_check(void) { return device_check(); }

size_t bulkgcd_blocked_words(size_t n, uint32_t bits) { return pad32(n) * (size_t)words_for(bits); }

uint64_t bulkgcd_cohort_count(size_t n) { return cohort_total(n); }

int bulkgcd_interleave(const uint32_t *d_in, uint32_t *d_out, size_t m, size_t m_pad, uint32_t bits,
                       int to_interleaved, void *stream) {
    int W = words_for(bits);
    if (!W) return set_err(BULKGCD_EINVAL, "unsupported bits %u", bits);
    if (m_pad < m || m_pad % 32) return set_err(BULKGCD_EINVAL, "m_pad must be >= m and a multiple of 32");
    if (m_pad == 0) return 0;
    if (!d_in || !d_out) return set_err(BULKGCD_EINVAL, "null pointer");
    dim3 grid((unsigned)(m_pad / 32), (unsigned)((W + 31) / 32)), block(32, 8);
    interleave_kernel<<<grid, block, 0, (cudaStream_t)stream>>>(d_in, d_out, m, m_pad, W, to_interleaved);
    CK(cudaGetLastError());
    return 0;
}

int bulkgcd_layout_blocked(const uint32_t *d_N, uint32_t *d_N_blk, size_t n, uint32_t bits, void *stream) {
    int W = words_for(bits);
    if (!W) return set_err(BULKGCD_EINVAL, "unsupported bits %u", bits);
    if (n == 0) return 0;
    if (!d_N || !d_N_blk) return set_err(BULKGCD_EINVAL, "null pointer");
    dim3 grid((unsigned)(pad32(n) / 32), (unsigned)((W + 31) / 32)), block(32, 8);
    blocked_kernel<<<grid, block, 0, (cudaStream_t)stream>>>(d_N, d_N_blk, n, W);
    CK(cudaGetLastError());
    return 0;
}

int bulkgcd_pairs_device(const uint32_t *d_A, const uint32_t *d_B, uint32_t *d_G, size_t m, size_t m_pad,
                         uint32_t bits, int mode, uint32_t *d_iters, unsigned long long *d_scratch, unsigned flags,
                         void *stream) {
    int W = words_for(bits);
    if (!W) return set_err(BULKGCD_EINVAL, "unsupported bits %u", bits);
    if (mode != BULKGCD_MODE_EXACT && mode != BULKGCD_MODE_RSA) return set_err(BULKGCD_EINVAL, "bad mode %d", mode);
    if (m == 0) return 0;
    if (!d_A || !d_B || !d_G || !d_scratch) return set_err(BULKGCD_EINVAL, "null pointer");
    if (m_pad < m || m_pad % 32) return set_err(BULKGCD_EINVAL, "m_pad must be >= m and a multiple of 32");
    cudaStream_t st = (cudaStream_t)stream;
    switch (W) {
        case 16: return launch_pairs<16>(d_A, d_B, d_G, m, m_pad, mode, d_iters, d_scratch, flags, st);
        case 32: return launch_pairs<32>(d_A, d_B, d_G, m, m_pad, mode, d_iters, d_scratch, flags, st);
        case 64: return launch_pairs<64>(d_A, d_B, d_G, m, m_pad, mode, d_iters, d_scratch, flags, st);
        default: return launch_pairs<128>(d_A, d_B, d_G, m, m_pad, mode, d_iters, d_scratch, flags, st);
    }
}

int bulkgcd_all_pairs_band(const uint32_t *d_N, const uint32_t *d_N_blk, size_t n, uint32_t bits,
                           uint64_t cohort_begin, uint64_t cohort_end, uint32_t *d_hits, uint64_t hit_cap,
                           unsigned long long *d_counters, unsigned flags, void *stream) {
    int W = words_for(bits);
    if (!W) return set_err(BULKGCD_EINVAL, "unsupported bits %u", bits);
    if (!d_counters) return set_err(BULKGCD_EINVAL, "null counters");
    uint64_t total = cohort_total(n);
    if (cohort_end > total) cohort_end = total;
    if (cohort_begin > cohort_end) cohort_begin = cohort_end;
    if (cohort_end > cohort_begin && (!d_N || !d_N_blk)) return set_err(BULKGCD_EINVAL, "null pointer");
    if (hit_cap && !d_hits) return set_err(BULKGCD_EINVAL, "null hit buffer with hit_cap > 0");
    cudaStream_t st = (cudaStream_t)stream;
    switch (W) {
        case 16: return launch_allpairs<16>(d_N, d_N_blk, n, cohort_begin, cohort_end, d_hits, hit_cap, d_counters, flags, st);
        case 32: return launch_allpairs<32>(d_N, d_N_blk, n, cohort_begin, cohort_end, d_hits, hit_cap, d_counters, flags, st);
        case 64: return launch_allpairs<64>(d_N, d_N_blk, n, cohort_begin, cohort_end, d_hits, hit_cap, d_counters, flags, st);
        default: return launch_allpairs<128>(d_N, d_N_blk, n, cohort_begin, cohort_end, d_hits, hit_cap, d_counters, flags, st);
    }
}

// Large host-buffer batches run in chunks on PAIRS_STREAMS streams, so the copy engines move
// chunk c+1 in (and chunk c-1 out) while chunk c computes: H2D, layout, kernel, layout back
// and D2H of one chunk are ordered on its stream, and a stream's buffers are reused by
// its next chunk only after its D2H (stream order).  Overlap needs pinned host buffers;
// with pageable ones the driver stages the copies synchronously and the result is the same.
// 2^17-pair chunks on three streams: 2^20 pairs through the C ABI with pinned buffers 7.77 -> 6.91 ms
// (134.9 -> 151.8 M GCD/s) against 2^18 on two; four streams 7.16 ms (tools/e2e_pairs.py)
constexpr size_t PAIRS_CHUNK = size_t(1) << 17;
constexpr int PAIRS_STREAMS = 3;

// Scope guard of the chunked path: on every exit -- including an error return in the
// middle of the chunk loop -- both streams are drained before they are destroyed, so no
// copy into the caller's G / iters is still in flight when the call returns.
struct StreamPair {
    cudaStream_t s[PAIRS_STREAMS] = {};
    ~StreamPair() {
        for (auto &x : s)
            if (x) cudaStreamSynchronize(x);
        for (auto &x : s)
            if (x) cudaStreamDestroy(x);
    }
};

static int pairs_chunked(const uint32_t *A, const uint32_t *B, size_t m, int W, uint32_t bits, int mode, uint32_t *G,
                         uint32_t *iters) {
    StreamPair sp;
    for (auto &x : sp.s) CK(cudaStreamCreateWithFlags(&x, cudaStreamNonBlocking));
    const size_t rm = PAIRS_CHUNK * W * 4, cm = pad32(PAIRS_CHUNK) * W * 4;
    struct Bufs {
        DBuf a, b, ac, bc, gc, it, sc;
    } buf[PAIRS_STREAMS];
    for (int k = 0; k < PAIRS_STREAMS; ++k) {
        cudaStream_t st = sp.s[k];
        CK(buf[k].a.alloc(rm, st));
        CK(buf[k].b.alloc(rm, st));
        CK(buf[k].ac.alloc(cm, st));
        CK(buf[k].bc.alloc(cm, st));
        CK(buf[k].gc.alloc(cm, st));
        CK(buf[k].sc.alloc(8 * sizeof(unsigned long long), st));
        if (iters) CK(buf[k].it.alloc(PAIRS_CHUNK * 4, st));
    }
    int rc;
    for (size_t c = 0, off = 0; off < m; ++c, off += PAIRS_CHUNK) {
        Bufs &b = buf[c % PAIRS_STREAMS];
        cudaStream_t st = sp.s[c % PAIRS_STREAMS];
        size_t mc = std::min(PAIRS_CHUNK, m - off), mp = pad32(mc), bytes = mc * W * 4;
        CK(cudaMemcpyAsync(b.a.p, A + off * W, bytes, cudaMemcpyHostToDevice, st));
        CK(cudaMemcpyAsync(b.b.p, B + off * W, bytes, cudaMemcpyHostToDevice, st));
        if ((rc = bulkgcd_interleave(b.a.as<uint32_t>(), b.ac.as<uint32_t>(), mc, mp, bits, 1, st))) return rc;
        if ((rc = bulkgcd_interleave(b.b.as<uint32_t>(), b.bc.as<uint32_t>(), mc, mp, bits, 1, st))) return rc;
        if ((rc = bulkgcd_pairs_device(b.ac.as<uint32_t>(), b.bc.as<uint32_t>(), b.gc.as<uint32_t>(), mc, mp, bits,
                                       mode, iters ? b.it.as<uint32_t>() : nullptr, b.sc.as<unsigned long long>(),
                                       0, st)))
            return rc;
        if ((rc = bulkgcd_interleave(b.gc.as<uint32_t>(), b.a.as<uint32_t>(), mc, mp, bits, 0, st))) return rc;
        CK(cudaMemcpyAsync(G + off * W, b.a.p, bytes, cudaMemcpyDeviceToHost, st));
        if (iters) CK(cudaMemcpyAsync(iters + off, b.it.p, mc * 4, cudaMemcpyDeviceToHost, st));
    }
    for (auto &x : sp.s) CK(cudaStreamSynchronize(x));
    return 0;
}

int bulkgcd_pairs_ex(const uint32_t *A, const uint32_t *B, size_t m, uint32_t bits, int mode, uint32_t *G,
                     uint32_t *iters) {
    int W = words_for(bits);
    if (!W) return set_err(BULKGCD_EINVAL, "unsupported bits %u (supported: 512, 1024, 2048, 4096)", bits);
    if (mode != BULKGCD_MODE_EXACT && mode != BULKGCD_MODE_RSA) return set_err(BULKGCD_EINVAL, "bad mode %d", mode);
    if (m == 0) return 0;
    if (!A || !B || !G) return set_err(BULKGCD_EINVAL, "null pointer with m > 0");
    if (mode == BULKGCD_MODE_RSA) {
        int rc = check_moduli(A, m, W);
        if (!rc) rc = check_moduli(B, m, W);
        if (rc) return rc;
    }
    int rc = device_check();
    if (rc) return rc;
    if (m > PAIRS_CHUNK) return pairs_chunked(A, B, m, W, bits, mode, G, iters);
    cudaStream_t st = cudaStreamPerThread;
    size_t m_pad = pad32(m), rm = m * W * 4, cm = m_pad * W * 4;
    DBuf dA, dB, dAc, dBc, dGc, dIt, dS;
    CK(dA.alloc(rm, st));
    CK(dB.alloc(rm, st));
    CK(dAc.alloc(cm, st));
    CK(dBc.alloc(cm, st));
    CK(dGc.alloc(cm, st));
    CK(dS.alloc(8 * sizeof(unsigned long long), st));
    if (iters) CK(dIt.alloc(m * 4, st));
    CK(cudaMemcpyAsync(dA.p, A, rm, cudaMemcpyHostToDevice, st));
    CK(cudaMemcpyAsync(dB.p, B, rm, cudaMemcpyHostToDevice, st));
    if ((rc = bulkgcd_interleave(dA.as<uint32_t>(), dAc.as<uint32_t>(), m, m_pad, bits, 1, st))) return rc;
    if ((rc = bulkgcd_interleave(dB.as<uint32_t>(), dBc.as<uint32_t>(), m, m_pad, bits, 1, st))) return rc;
    if ((rc = bulkgcd_pairs_device(dAc.as<uint32_t>(), dBc.as<uint32_t>(), dGc.as<uint32_t>(), m, m_pad, bits, mode,
                                   iters ? dIt.as<uint32_t>() : nullptr, dS.as<unsigned long long>(), 0, st)))
        return rc;
    // de-interleave into dA (reused as the row-major result buffer)
    if ((rc = bulkgcd_interleave(dGc.as<uint32_t>(), dA.as<uint32_t>(), m, m_pad, bits, 0, st))) return rc;
    CK(cudaMemcpyAsync(G, dA.p, rm, cudaMemcpyDeviceToHost, st));
    if (iters) CK(cudaMemcpyAsync(iters, dIt.p, m * 4, cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    return 0;
}

int bulkgcd_pairs(const uint32_t *A, const uint32_t *B, size_t m, uint32_t bits, uint32_t *G) {
    return bulkgcd_pairs_ex(A, B, m, bits, BULKGCD_MODE_EXACT, G, nullptr);
}

void bulkgcd_hits_free(bulkgcd_hits_t *h) {
    if (!h) return;
    free(h->ij);
    free(h->gcd);
    h->ij = nullptr;
    h->gcd = nullptr;
    h->count = 0;
}

int bulkgcd_all_pairs(const uint32_t *N, size_t n, uint32_t bits, bulkgcd_hits_t *out) {
    int W = words_for(bits);
    if (!out) return set_err(BULKGCD_EINVAL, "null hits_out");
    memset(out, 0, sizeof *out);
    out->bits = bits;
    if (!W) return set_err(BULKGCD_EINVAL, "unsupported bits %u (supported: 512, 1024, 2048, 4096)", bits);
    if (n > 0 && !N) return set_err(BULKGCD_EINVAL, "null moduli with n > 0");
    if (n > 0xFFFFFFFFull) return set_err(BULKGCD_EINVAL, "n too large");
    int rc = check_moduli(N, n, W);
    if (rc) return rc;
    if (n < 2) return 0;
    if ((rc = device_check())) return rc;
    cudaStream_t st = cudaStreamPerThread;
    DBuf dN, dBlk, dC, dH;
    CK(dN.alloc(n * W * 4, st));
    CK(dBlk.alloc(bulkgcd_blocked_words(n, bits) * 4, st));
    CK(dC.alloc(8 * sizeof(unsigned long long), st));
    CK(cudaMemcpyAsync(dN.p, N, n * W * 4, cudaMemcpyHostToDevice, st));
    if ((rc = bulkgcd_layout_blocked(dN.as<uint32_t>(), dBlk.as<uint32_t>(), n, bits, st))) return rc;
    uint64_t cap = 1024;
    uint64_t total = cohort_total(n);
    unsigned long long count = 0;
    for (int attempt = 0; attempt < 3; ++attempt) {
        if (dH.p) {
            cudaFreeAsync(dH.p, st);
            dH.p = nullptr;
        }
        CK(dH.alloc(cap * (2 + W) * 4, st));
        if ((rc = bulkgcd_all_pairs_band(dN.as<uint32_t>(), dBlk.as<uint32_t>(), n, bits, 0, total,
                                         dH.as<uint32_t>(), cap, dC.as<unsigned long long>(), 0, st)))
            return rc;
        CK(cudaMemcpyAsync(&count, dC.p, sizeof count, cudaMemcpyDeviceToHost, st));
        CK(cudaStreamSynchronize(st));
        if (count <= cap) break;
        cap = count;  // overflow: rerun with room for every hit
    }
    if (count > cap) return set_err(BULKGCD_ECUDA, "hit buffer overflow persisted");
    std::vector<uint32_t> rec(count * (2 + W));
    if (count) CK(cudaMemcpyAsync(rec.data(), dH.p, rec.size() * 4, cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    std::vector<size_t> order(count);
    std::iota(order.begin(), order.end(), 0);
    std::sort(order.begin(), order.end(), [&](size_t a, size_t b) {
        const uint32_t *ra = &rec[a * (2 + W)], *rb = &rec[b * (2 + W)];
        return ra[0] != rb[0] ? ra[0] < rb[0] : ra[1] < rb[1];
    });
    if (count) {
        out->ij = (uint32_t(*)[2])malloc(count * sizeof(uint32_t[2]));
        out->gcd = (uint32_t *)malloc(count * W * sizeof(uint32_t));
        if (!out->ij || !out->gcd) {
            bulkgcd_hits_free(out);
            return set_err(BULKGCD_ENOMEM, "host allocation of %llu hits failed", count);
        }
        for (size_t h = 0; h < count; ++h) {
            const uint32_t *r = &rec[order[h] * (2 + W)];
            out->ij[h][0] = r[0];
            out->ij[h][1] = r[1];
            memcpy(out->gcd + h * W, r + 2, W * 4);
        }
    }
    out->count = count;
    out->bits = bits;
    return 0;
}

int bulkgcd_cofactors_device(const uint32_t *d_N, size_t n, uint32_t bits, const uint32_t *d_hits, uint64_t count,
                             uint32_t *d_F, unsigned long long *d_bad, void *stream) {
    int W = words_for(bits);
    if (!W) return set_err(BULKGCD_EINVAL, "unsupported bits %u", bits);
    if (count == 0) return 0;
    if (!d_N || !d_hits || !d_F || !d_bad) return set_err(BULKGCD_EINVAL, "null pointer with count > 0");
    cudaStream_t st = (cudaStream_t)stream;
    uint64_t threads = 2 * count, block = 128, grid = (threads + block - 1) / block;
    switch (W) {
        case 16: cofactor_kernel<16><<<(unsigned)grid, (unsigned)block, 0, st>>>(d_N, n, d_hits, count, d_F, d_bad); break;
        case 32: cofactor_kernel<32><<<(unsigned)grid, (unsigned)block, 0, st>>>(d_N, n, d_hits, count, d_F, d_bad); break;
        case 64: cofactor_kernel<64><<<(unsigned)grid, (unsigned)block, 0, st>>>(d_N, n, d_hits, count, d_F, d_bad); break;
        default: cofactor_kernel<128><<<(unsigned)grid, (unsigned)block, 0, st>>>(d_N, n, d_hits, count, d_F, d_bad); break;
    }
    CK(cudaGetLastError());
    return 0;
}

int bulkgcd_cofactors(const uint32_t *N, size_t n, uint32_t bits, const bulkgcd_hits_t *hits, uint32_t *F) {
    int W = words_for(bits);
    if (!W) return set_err(BULKGCD_EINVAL, "unsupported bits %u (supported: 512, 1024, 2048, 4096)", bits);
    if (!hits) return set_err(BULKGCD_EINVAL, "null hits");
    if (hits->bits != bits) return set_err(BULKGCD_EINVAL, "hits were computed for %u bits, not %u", hits->bits, bits);
    size_t count = hits->count;
    if (count == 0) return 0;
    if (!N || !F || !hits->ij || !hits->gcd) return set_err(BULKGCD_EINVAL, "null pointer with count > 0");
    for (size_t h = 0; h < count; ++h)
        if (hits->ij[h][0] >= n || hits->ij[h][1] >= n)
            return set_err(BULKGCD_EINVAL, "hit %zu indexes a modulus >= n = %zu", h, n);
    int rc = device_check();
    if (rc) return rc;
    cudaStream_t st = cudaStreamPerThread;
    std::vector<uint32_t> rec(count * (2 + W));
    for (size_t h = 0; h < count; ++h) {
        rec[h * (2 + W)] = hits->ij[h][0];
        rec[h * (2 + W) + 1] = hits->ij[h][1];
        memcpy(&rec[h * (2 + W) + 2], hits->gcd + h * W, W * 4);
    }
    DBuf dN, dH, dF, dBad;
    CK(dN.alloc(n * W * 4, st));
    CK(dH.alloc(rec.size() * 4, st));
    CK(dF.alloc(2 * count * W * 4, st));
    CK(dBad.alloc(sizeof(unsigned long long), st));
    CK(cudaMemcpyAsync(dN.p, N, n * W * 4, cudaMemcpyHostToDevice, st));
    CK(cudaMemcpyAsync(dH.p, rec.data(), rec.size() * 4, cudaMemcpyHostToDevice, st));
    CK(cudaMemsetAsync(dBad.p, 0, sizeof(unsigned long long), st));
    if ((rc = bulkgcd_cofactors_device(dN.as<uint32_t>(), n, bits, dH.as<uint32_t>(), count, dF.as<uint32_t>(),
                                       dBad.as<unsigned long long>(), st)))
        return rc;
    unsigned long long bad = 0;
    CK(cudaMemcpyAsync(F, dF.p, 2 * count * W * 4, cudaMemcpyDeviceToHost, st));
    CK(cudaMemcpyAsync(&bad, dBad.p, sizeof bad, cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    if (bad) return set_err(BULKGCD_EINVAL, "%llu cofactor(s): gcd is zero, even, or does not divide the modulus", bad);
    return 0;
}

}  // extern "C"
