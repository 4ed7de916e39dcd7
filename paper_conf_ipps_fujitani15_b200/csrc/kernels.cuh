// kernels.cuh -- the bulk GCD kernels (sm_100a): layout transforms, the
// independent-pairs kernel (bulkgcd_pairs) and the all-pairs kernel
// (bulkgcd_all_pairs / bulkgcd_all_pairs_band).
#pragma once
#include <cstdint>
#include <type_traits>

#include "euclid.cuh"
#include "smem_euclid.cuh"

namespace bulkgcd {

#ifndef BULKGCD_THREADS
#define BULKGCD_THREADS 128  // 4 warps per CTA
#endif
constexpr int THREADS = BULKGCD_THREADS;
constexpr int WARPS_PER_CTA = THREADS / 32;
#ifndef MIN_WARPS
// resident warps per SM for W <= 32: 20 -> <= 96 registers per thread.  ptxas
// spills cold-section state only; more warps keep the ALU pipe busier across the
// fixed-latency dependency chains (cfg3: 12 -> 16 warps 292 -> 266 ms, 16 -> 20
// 253 -> 251 ms).
#define MIN_WARPS 20
#endif
#ifndef MIN_WARPS_W16
#define MIN_WARPS_W16 32  // 512-bit all-pairs: 64 registers (cfg6 86.4 -> 84.8 ms against 20 warps)
#endif
#ifndef MIN_WARPS_PAIRS
// the pairs kernel (1024-bit, 2^20 pairs): 16 -> 20 warps exact 4.22 -> 4.19 ms, RSA 3.65 -> 3.32 ms;
// 24 warps 4.32 / 3.47 ms
#define MIN_WARPS_PAIRS 20
#endif
#ifndef MIN_WARPS_W16_PAIRS
#define MIN_WARPS_W16_PAIRS 32  // 512-bit pairs: 2^20 exact 1.49 -> 1.46 ms, RSA 0.85 -> 0.83 ms against 20
#endif
#ifndef MIN_WARPS_W64
// W = 64 all-pairs: 12 warps/SM (168 registers; ptxas spills ~4 KB of cold and window state)
// beat 8 warps (255 registers, spill-free): cfg4 1,034 -> 943 ms; 16 warps spill the
// operands themselves (1,708 ms).
#define MIN_WARPS_W64 12
#endif
#ifndef MIN_WARPS_W64_PAIRS
#define MIN_WARPS_W64_PAIRS 12  // 2048-bit pairs: 2^18 exact 7.67 -> 7.23 ms, RSA 3.58 -> 3.29 ms against 8
#endif
// CTAs per SM by width: the operands take 2W registers per thread; W = 64
// (2048-bit) needs ~200+ registers, i.e. 8 warps per SM.
// Register cap: __launch_bounds__(THREADS, blocks) by default; -DBULKGCD_MAXNREG=N
// instead caps every kernel at N registers per thread (__maxnreg__).
#ifdef BULKGCD_MAXNREG
#define BULKGCD_BOUNDS(W, PAIRS) __maxnreg__(BULKGCD_MAXNREG)
#else
#define BULKGCD_BOUNDS(W, PAIRS) __launch_bounds__(THREADS, (Occ<W, PAIRS>::blocks))
#endif
template <int W, bool PAIRS = false>
struct Occ {
    static constexpr int warps = W >= 64 ? (PAIRS ? MIN_WARPS_W64_PAIRS : MIN_WARPS_W64)
                                         : (PAIRS ? (W <= 16 ? MIN_WARPS_W16_PAIRS : MIN_WARPS_PAIRS)
                                                  : (W <= 16 ? MIN_WARPS_W16 : MIN_WARPS));
    static constexpr int blocks = warps / WARPS_PER_CTA > 0 ? warps / WARPS_PER_CTA : 1;
};

// ------------------------------------------------------------------ layouts
// Word-interleaved ("column-wise", PAPER.md L361 and Fig. 3) layouts: lane t of
// a warp reads word k of its operand at consecutive addresses, so every limb
// load is one coalesced 128-byte transaction.
//   interleaved: X_cm[k * m_pad + i]
//   blocked    : X_blk[(b * W + k) * 32 + t] for i = 32 b + t  (one cohort's 32
//                operands are a contiguous W*128-byte block)

// row-major [m][W] -> interleaved [W][m_pad] (to_cm) or back.
__global__ void interleave_kernel(const uint32_t *__restrict__ in, uint32_t *__restrict__ out, uint64_t m,
                                  uint64_t m_pad, int W, int to_cm) {
    __shared__ uint32_t tile[32][33];
    uint64_t i0 = (uint64_t)blockIdx.x * 32;
    int k0 = blockIdx.y * 32;
    int tx = threadIdx.x, ty = threadIdx.y;  // 32 x 8
    for (int r = ty; r < 32; r += 8) {
        if (to_cm) {  // read row-major: row i0+r, word k0+tx
            uint64_t i = i0 + r;
            int k = k0 + tx;
            tile[r][tx] = (i < m && k < W) ? in[i * W + k] : 0u;
        } else {  // read interleaved: word k0+r, item i0+tx
            uint64_t i = i0 + tx;
            int k = k0 + r;
            tile[tx][r] = (i < m && k < W) ? in[(uint64_t)k * m_pad + i] : 0u;  // padding items are never read
        }
    }
    __syncthreads();
    for (int r = ty; r < 32; r += 8) {
        if (to_cm) {  // write interleaved: word k0+r, item i0+tx
            uint64_t i = i0 + tx;
            int k = k0 + r;
            if (i < m_pad && k < W) out[(uint64_t)k * m_pad + i] = tile[tx][r];
        } else {  // write row-major
            uint64_t i = i0 + r;
            int k = k0 + tx;
            if (i < m && k < W) out[i * W + k] = tile[r][tx];
        }
    }
}

// row-major [n][W] -> blocked [nb][W][32] (zero padded).
__global__ void blocked_kernel(const uint32_t *__restrict__ in, uint32_t *__restrict__ out, uint64_t n, int W) {
    __shared__ uint32_t tile[32][33];
    uint64_t b = blockIdx.x;
    int k0 = blockIdx.y * 32;
    int tx = threadIdx.x, ty = threadIdx.y;
    for (int r = ty; r < 32; r += 8) {
        uint64_t i = b * 32 + r;
        int k = k0 + tx;
        tile[r][tx] = (i < n && k < W) ? in[i * W + k] : 0u;
    }
    __syncthreads();
    for (int r = ty; r < 32; r += 8) {
        int k = k0 + r;
        if (k < W) out[(b * W + k) * 32 + tx] = tile[tx][r];
    }
}

// ------------------------------------------------------------ lane helpers
__device__ __forceinline__ uint64_t small_value(int l, uint64_t t) {
    return l >= 2 ? t : (l == 1 ? (t >> 32) : 0ull);
}

__device__ __forceinline__ int bitlen_top(int l, uint64_t t) {
    return l == 0 ? 0 : 32 * (l - 1) + (32 - __clz(hi32(t)));
}

// Order a lane's fresh operands so that A >= B, and compute lengths and tops.
template <int W>
__device__ __forceinline__ void setup_pair(uint32_t (&A)[W], uint32_t (&B)[W], int &lA, uint64_t &tA, int &lB,
                                           uint64_t &tB) {
    lA = scan_full<W>(A, tA) + 1;
    lB = scan_full<W>(B, tB) + 1;
    int c = lA != lB ? (lA < lB ? -1 : 1) : (tA != tB ? (tA < tB ? -1 : 1) : 0);
    if (c == 0) {  // equal lengths and tops: full compare, most significant first
#pragma unroll
        for (int k = W - 1; k >= 0; --k)
            if (c == 0 && A[k] != B[k]) c = A[k] < B[k] ? -1 : 1;
    }
    if (c < 0) {
        swap_regs<W>(A, B);
        int tl = lA; lA = lB; lB = tl;
        uint64_t tt = tA; tA = tB; tB = tt;
    }
}

// The per-cohort Euclid loop.  A >= B on entry (registers least-significant
// first, s = 0).  cond(lX, tX, lY, tY) is the do-while condition of a lane.
//
// Structure: a hot loop (two iterations per trip with exchanged roles) that
// touches the operand registers only through the fused pass, and a cold
// section that handles everything rare -- fix-ups (no swap, slow path),
// finished lanes whose result needs the operand registers (sink), and the
// realign when the warp length L dropped.  Keeping every conditional write of
// the register arrays out of the hot loop stops ptxas from materialising
// whole-array copies at merge points.  Each hot iteration ends with the loop
// test of the next one, and all warp-level decisions of an iteration are two
// votes: "some lane needs the cold section" and "some running
// lane still reaches the top register" (if none, the warp length L dropped and
// the cold section realigns; this also covers "no lane running") -- two ballots.
//
// Sink API: quick(fin, lX, tX, lY, tY) runs in the hot loop for every lane
// and returns true if a finished lane needs cold(...) (warp-converged, with
// the operand registers); scalar-only finishes are handled by quick itself.
//
// CMPL: complement form (gen_duff.py emit_cmpl) -- A is kept bit-complemented in its
// registers for the whole loop and B plain, so every update is a multiply-accumulate:
// hot(A, B) runs the A-type pass (A~ + alpha*B, ones shifted in), hot(B, A) the B-type
// pass (B + alpha*A~ + alpha).  The roles alternate strictly, which keeps A complemented;
// the rare cold-section code that reads the operand registers (fix-ups, the hit sink)
// sees plain values (A is complemented around it).
// HOIST: approx() for the next iteration is computed at the end of the current one, ahead of
// its votes and branches (measured: cfg4 851.5 -> 834.6 ms; cfg3 233.3 -> 235.1, 2^20 RSA pairs
// 2.47 -> 3.07, exact 3.74 -> 3.84 ms: the W = 64 all-pairs kernel only).
// CUTK > 0: straggler cut (all-pairs, split/mix forms only).  Every second iteration the warp counts
// its running lanes; once at most CUTK remain, sink.cut() stores their operands (and pair ids) in the
// warp's straggler buffer and the cohort ends; the kernel runs the stored lanes later, 32 at a time
// (allpairs_kernel), so the end of a cohort no longer runs a nearly empty warp.
template <int W, bool STATS, bool EXACT, bool ONE_ENTRY, class Cond, class Sink, bool CMPL = false, bool HOIST = false,
          bool SWAP_RESUME = false, int PG = 0, int CUTK = 0>
__device__ __forceinline__ void euclid_loop(uint32_t (&A)[W], uint32_t (&B)[W], int &lA, uint64_t &tA, int &lB,
                                            uint64_t &tB, bool live, Cond cond, Sink &sink, int s0,
                                            uint32_t &iters, uint32_t &nslow, uint32_t &limbs, uint32_t &slots,
                                            uint32_t &passw) {
    using CmA = std::integral_constant<int, CMPL ? 1 : 0>;  // hot_iter pass form with A updated
    using CmB = std::integral_constant<int, CMPL ? 2 : 0>;  // ... with B updated
    int s = s0;
    int fix = 0;     // pending fix-up of the last iteration (hot_iter's code)
    Approx ap;       // approx() for the coming hot iteration
    int resume = 0;  // roles of the next iteration: 0 -> (X, Y) = (A, B), 1 -> (B, A)
    if (CMPL) cmpl_regs<W>(A);

    // Cold section for the next roles (X, Y); the last iteration ran on (Y, X).
    // Applies fix-ups, runs the loop test, serves finished lanes, realigns.
    auto cold = [&](uint32_t(&X)[W], uint32_t(&Y)[W], int &lX, uint64_t &tX, int &lY, uint64_t &tY) -> bool {
        if (__any_sync(FULL, fix != 0)) {
            if (STATS && fix >= 2) ++nslow;
            if (CMPL) cmpl_regs<W>(A);
            apply_fix<W>(fix, Y, X, lY, tY, lX, tX, s);
            if (CMPL) cmpl_regs<W>(A);
            fix = 0;
        }
        bool run = live & cond(lX, tX, lY, tY);
        bool fin = live & !run;
        if (__any_sync(FULL, fin)) {
            bool need = sink.quick(fin, lX, tX, lY, tY);
            if (__any_sync(FULL, need)) {
                if (CMPL) cmpl_regs<W>(A);
                sink.cold(need, X, Y, lX, tX, lY, tY, s);
                if (CMPL) cmpl_regs<W>(A);
            }
        }
        live = run;
        unsigned brun = __ballot_sync(FULL, run);
        if (brun == 0u) return false;
        int L = __reduce_max_sync(FULL, (unsigned)(run ? lX : 0));
        while (W - s > L) {
            shift_up_1<W>(A);
            shift_up_1<W>(B);
            ++s;
        }
        return true;
    };
    // One hot iteration on roles (X, Y) (its loop test already passed: the
    // live lanes are the running ones), then the loop test of the next
    // iteration (roles (Y, X)).  Returns true to go cold.
    bool cut = false;
    auto hot = [&](auto cm, uint32_t(&X)[W], uint32_t(&Y)[W], int &lX, uint64_t &tX, int &lY, uint64_t &tY) -> bool {
        if (STATS) {
            ++slots;
            passw += W - s;  // words the warp's pass covers this iteration
            if (live) {
                ++iters;
                limbs += lX;  // limb-steps: words of X the update pass covers
            }
        }
        bool full, post, lt;
        if (!HOIST) ap = approx_pre<EXACT>(lX, tX, lY, tY);
        hot_iter<W, EXACT, decltype(cm)::value, PG>(X, Y, lX, tX, lY, tY, s, live, ap, full, post, lt);
        bool bad = live & (full | post | !lt);
        bool run = live & cond(lY, tY, lX, tX);
        bool fin = live & !run & !bad;
        bool need = sink.quick_hot(fin, lY, tY, lX, tX) | bad;
        bool top = run & (lY == W - s);
        if (HOIST) ap = approx_pre<EXACT>(lY, tY, lX, tX);  // the next iteration's roles (Y, X), ahead of the votes
        // vote.any with a predicate result: no mask compare on the ALU pipe
        bool any_need = __any_sync(FULL, need), any_top = __any_sync(FULL, top);
        if (any_need) {
            fix = fix_code(live, full, post, lt);
            return true;
        }
        if constexpr (CUTK > 0) {
            if (decltype(cm)::value == 0 && &X == &B) {  // after the B-updating iteration only
                if (__popc(__ballot_sync(FULL, run)) <= sink.cutk) {
                    live = run;
                    cut = true;
                    return true;
                }
            }
        }
        if (!any_top) {  // the warp length dropped (lanes finished or shrank): realign one word in place
            unsigned brun = __ballot_sync(FULL, run);
            if (brun == 0u) {  // nobody runs: go cold (the cohort ends there)
                fix = fix_code(live, full, post, lt);
                return true;
            }
            shift_up_1<W>(A);
            shift_up_1<W>(B);
            ++s;
        }
        live = run;
        return false;
    };

    for (;;) {
        bool more = resume == 0 ? cold(A, B, lA, tA, lB, tB) : cold(B, A, lB, tB, lA, tA);
        if (!more) return;
        // SWAP_RESUME: resuming on roles (B, A) exchanges the register arrays (and their lengths
        // and tops) instead, so the loop is entered at its first hot iteration only and the pass
        // is inlined twice, with no irreducible entry: 64-128 moves on a cold exit (~1 % of the
        // iterations) for a third less hot code (instruction cache).  In the complement form both
        // arrays are complemented too, so that A stays the complemented one.
        if (SWAP_RESUME && resume == 1) {
            if (CMPL) cmpl_regs<W>(A);  // plain A0, B0
            swap_regs<W>(A, B);
            if (CMPL) cmpl_regs<W>(A);  // A = ~B0 (the complemented one again), B = A0
            int tl = lA; lA = lB; lB = tl;
            uint64_t tt = tA; tA = tB; tB = tt;
            resume = 0;
        }
        if (HOIST) ap = resume == 0 ? approx_pre<EXACT>(lA, tA, lB, tB) : approx_pre<EXACT>(lB, tB, lA, tA);
        // ONE_ENTRY: resuming on roles (B, A) enters the loop at its second hot
        // iteration, so the pass is inlined twice (once per role assignment) instead of
        // three times.  Measured: RSA pairs 3.30 -> 2.72 ms per 2^20
        // (1024-bit) and 3.29 -> 2.87 ms per 2^18 (2048-bit), but all-pairs cfg3
        // 246.7 -> 256.0 ms and exact pairs 4.19 -> 4.38 ms, so only the RSA pairs
        // kernel uses it.
        if (ONE_ENTRY) {
            if (resume == 1) goto roles_ba;
        } else if (!SWAP_RESUME && resume == 1) {
            if (hot(CmB{}, B, A, lB, tB, lA, tA)) {
                resume = 0;
                continue;
            }
        }
        for (;;) {
            if (hot(CmA{}, A, B, lA, tA, lB, tB)) {
                resume = 1;
                break;
            }
        roles_ba:
            if (hot(CmB{}, B, A, lB, tB, lA, tA)) {
                resume = 0;
                break;
            }
        }
        if constexpr (CUTK > 0) {
            if (cut) {  // the last iteration updated B and went through no fix-up: A >= B
                sink.cut(live, A, B, s, lA);
                return;
            }
        }
    }
}

// RSA-mode loop condition (early-terminate, L243/L251/L255): continue while Y
// has at least s/2 bits.
struct RsaCond {
    int half;
    __device__ __forceinline__ bool operator()(int lX, uint64_t tX, int lY, uint64_t tY) const {
        // bitlen(Y) >= half (half a multiple of 32): lY > half/32, or lY == half/32 with y1's top bit set
        return 2 * lY + (int)(hi32(tY) >> 31) > half / 16;
    }
};

// Exact-mode condition: continue while Y != 0 and X has >= 3 words (Case 1,
// lX <= 2, finishes in the 64-bit tail).
struct ExactCond {
    __device__ __forceinline__ bool operator()(int lX, uint64_t tX, int lY, uint64_t tY) const {
        return (lY >= 1) & (lX >= 3);
    }
};

// -------------------------------------------------------------- generic I/O
// Write g << k2 (g: n words in local memory) as W output words.
template <int W>
__device__ __noinline__ void write_shifted(uint32_t *out, uint64_t stride, const uint32_t *g, int n, int k2) {
    int q = k2 >> 5, b = k2 & 31;
    for (int w = 0; w < W; ++w) {
        int src = w - q;
        uint32_t lo = (src >= 0 && src < n) ? g[src] : 0u;
        uint32_t lo1 = (src - 1 >= 0 && src - 1 < n) ? g[src - 1] : 0u;
        uint32_t v = b ? ((lo << b) | (lo1 >> (32 - b))) : lo;
        out[(uint64_t)w * stride] = v;
    }
}

// Exact-mode normalisation: gcd(x, 0) = x; strip the common
// power of two k2 = min(ctz a, ctz b) and all other trailing zeros.
// Returns 1 if the result is already known (a zero operand).
template <int W>
__device__ __forceinline__ int normalize_exact(uint32_t (&A)[W], uint32_t (&B)[W], int &k2) {
    uint32_t a[W], b[W];
#pragma unroll
    for (int k = 0; k < W; ++k) {
        a[k] = A[k];
        b[k] = B[k];
    }
    int za = 0, zb = 0;
    while (za < W && a[za] == 0) ++za;
    while (zb < W && b[zb] == 0) ++zb;
    if (za == W || zb == W) {  // gcd(x, 0) = x: leave x | 0 in A
#pragma unroll
        for (int k = 0; k < W; ++k) A[k] = a[k] | b[k];
        k2 = 0;
        return 1;
    }
    int ca = 32 * za + ctz32(a[za]);
    int cb = 32 * zb + ctz32(b[zb]);
    k2 = ca < cb ? ca : cb;
    n_rshift(a, W);
    n_rshift(b, W);
#pragma unroll
    for (int k = 0; k < W; ++k) {
        A[k] = a[k];
        B[k] = b[k];
    }
    return 0;
}

// ------------------------------------------------------------ pairs kernel
// G[i] = gcd(A[i], B[i]), i < m; operands and results word-interleaved.
// EXACT: full gcd of any operands (L41 + Approximate Euclid to Y = 0).
// RSA  : early-terminate; G = g if bitlen(g) >= bits/2 else 1.
struct PairsArgs {
    const uint32_t *A;
    const uint32_t *B;
    uint32_t *G;
    uint64_t m, m_pad;
    unsigned long long *work;  // cohort cursor, zeroed by the host
    uint32_t *iters;           // optional per-pair iteration counts
    unsigned long long *stats; // optional [sum iterations, slow steps, limb-steps]
    int half;
};

template <int W>
struct PairsSinkExact {
    uint32_t *G;
    uint64_t i, stride;
    int k2;
    bool tail;
    uint64_t x64, y64;
    // lX <= 2 (Y != 0): Case 1 from here on, in 64-bit scalars (no registers needed)
    __device__ __forceinline__ bool quick(bool fin, int lX, uint64_t tX, int lY, uint64_t tY) {
        if (fin && lY != 0) {
            tail = true;
            x64 = small_value(lX, tX);
            y64 = small_value(lY, tY);
        }
        return fin && lY == 0;
    }
    __device__ __forceinline__ bool quick_hot(bool fin, int lX, uint64_t tX, int lY, uint64_t tY) {
        return quick(fin, lX, tX, lY, tY);
    }
    // Y = 0: g = X (possibly long), written with the common power of two restored
    __device__ __forceinline__ void cold(bool need, uint32_t (&X)[W], uint32_t (&Y)[W], int lX, uint64_t tX, int lY,
                                         uint64_t tY, int s) {
        if (!need) return;
        uint32_t g[W];
#pragma unroll
        for (int k = 0; k < W; ++k) g[k] = X[k];
        write_shifted<W>(G + i, stride, g + s, W - s, k2);
    }
};

template <int W>
struct PairsSinkRsa {
    uint32_t *G;
    uint64_t i, stride;
    __device__ __forceinline__ bool quick(bool fin, int, uint64_t, int, uint64_t) { return fin; }
    __device__ __forceinline__ bool quick_hot(bool fin, int, uint64_t, int, uint64_t) { return fin; }
    __device__ __forceinline__ void cold(bool need, uint32_t (&X)[W], uint32_t (&Y)[W], int lX, uint64_t tX, int lY,
                                         uint64_t tY, int s) {
        if (!need) return;
        if (lY == 0) {
            uint32_t g[W];
#pragma unroll
            for (int k = 0; k < W; ++k) g[k] = X[k];
            write_shifted<W>(G + i, stride, g + s, W - s, 0);
        } else {
            for (int w = 0; w < W; ++w) G[i + (uint64_t)w * stride] = w == 0 ? 1u : 0u;
        }
    }
};

template <int W, bool RSA, bool STATS>
__global__ void BULKGCD_BOUNDS(W, true) pairs_kernel(PairsArgs a) {
    const int lane = threadIdx.x & 31;
    uint32_t iters = 0, nslow = 0, limbs = 0, slots = 0, passw = 0;
    // Cohort loop in claim / while (have) form: with a mid-loop `break` on the claimed id
    // instead, ptxas no longer proves the pass start s warp-uniform and emits a per-thread
    // BRX inside BSSY/BSYNC reconvergence for every pass (the all-pairs kernel's shape gets
    // the uniform BRXU).
    auto claim = [&](uint64_t &c) -> bool {
        unsigned long long cc = 0;
        if (lane == 0) cc = atomicAdd(a.work, 1ull);
        c = __shfl_sync(FULL, cc, 0);
        return c * 32 < a.m;
    };
    uint64_t c;
    bool have = claim(c);
    for (; have; have = claim(c)) {
        uint64_t i = c * 32 + lane;
        bool valid = i < a.m;
        uint32_t A[W], B[W];
#pragma unroll
        for (int k = 0; k < W; ++k) {
            A[k] = valid ? a.A[(uint64_t)k * a.m_pad + i] : 0u;
            B[k] = valid ? a.B[(uint64_t)k * a.m_pad + i] : 0u;
        }
        uint32_t it0 = iters;
        int lA, lB;
        uint64_t tA, tB;
        if (RSA) {
            bool live = valid;
            setup_pair<W>(A, B, lA, tA, lB, tB);
            PairsSinkRsa<W> sink{a.G, i, a.m_pad};
            // ONE_ENTRY (irreducible loop entry: the pass entry stays a per-thread BRX) beats the
            // two-entry loop with a uniform BRXU here: 2^20 RSA pairs 2.47 against 3.05 ms
            euclid_loop<W, STATS, false, true, RsaCond, PairsSinkRsa<W>, false, false, false, PASS_G_RSA<W>>(
                A, B, lA, tA, lB, tB, live, RsaCond{a.half}, sink, 0, iters, nslow, limbs, slots, passw);
        } else {
            int k2 = 0;
            bool known = false;
            if (valid) known = normalize_exact<W>(A, B, k2) != 0;
            if (valid && known) {
#pragma unroll
                for (int k = 0; k < W; ++k) a.G[i + (uint64_t)k * a.m_pad] = A[k];
            }
            bool live = valid && !known;
            if (!live) {
#pragma unroll
                for (int k = 0; k < W; ++k) A[k] = B[k] = 0;
            }
            setup_pair<W>(A, B, lA, tA, lB, tB);
            PairsSinkExact<W> sink{a.G, i, a.m_pad, k2, false, 0, 0};
            euclid_loop<W, STATS, true, false>(A, B, lA, tA, lB, tB, live, ExactCond{}, sink, 0, iters, nslow, limbs, slots,
                                               passw);
            // 64-bit tail: Case 1 of approx (lX <= 2): alpha = X div Y, exactly (L127).
            if (sink.tail) {
                uint64_t x = sink.x64, y = sink.y64;
                while (y != 0) {
                    uint64_t q = x / y;
                    if ((q & 1) == 0) q -= 1;
                    x = x - y * q;
                    if (x) x >>= __ffsll((long long)x) - 1;
                    if (x < y) { uint64_t t = x; x = y; y = t; }
                    if (STATS) {
                        ++iters;
                        limbs += (x >> 32) ? 2 : 1;
                    }
                }
                uint32_t g[2] = {lo32(x), hi32(x)};
                write_shifted<W>(a.G + i, a.m_pad, g, 2, sink.k2);
            }
        }
        if (a.iters && valid) a.iters[i] = iters - it0;
    }
    if (STATS && a.stats) {
        atomicAdd(&a.stats[0], (unsigned long long)iters);
        atomicAdd(&a.stats[1], (unsigned long long)nslow);
        atomicAdd(&a.stats[2], (unsigned long long)limbs);
        atomicAdd(&a.stats[3], (unsigned long long)slots);  // lane-slots: warp-iterations x 32
        atomicAdd(&a.stats[4], (unsigned long long)passw);  // lane-words of pass issued
    }
}

// --------------------------------------------------------- all-pairs kernel
// Work unit = cohort = (row block b of 32 consecutive moduli, column j), j >
// 32 b; lane t takes the pair (32 b + t, j) if 32 b + t < j.  Cohorts are
// numbered row block by row block: P(b) = b (n - 1) - 16 b (b - 1) cohorts
// precede row block b.  Every pair i < j is in exactly one cohort, and a
// contiguous range of cohort ids is a balanced share of the triangle (the
// multi-GPU band partition).
__host__ __device__ __forceinline__ uint64_t cohorts_before(uint64_t b, uint64_t n) {
    return b * (n - 1) - 16 * b * (b - 1);
}

__host__ __device__ __forceinline__ uint64_t cohort_total(uint64_t n) {
    if (n < 2) return 0;
    uint64_t nb = (n + 31) / 32;
    return cohorts_before(nb, n);
}

struct AllPairsArgs {
    const uint32_t *N_blk;  // blocked [nb][W][32]
    const uint32_t *N_rm;   // row-major [n][W]
    uint64_t n;
    uint64_t c_begin, c_end;
    unsigned long long *work;      // cursor, zeroed by the host
    uint32_t *hits;                // hit records [i, j, g[W]]
    uint64_t hit_cap;
    unsigned long long *hit_count;
    unsigned long long *stats;     // optional [sum iterations, slow steps, limb-steps]
    int half;
    uint32_t *strag;               // straggler buffers, one per resident warp (W <= 32)
};

// Straggler buffer of one warp (euclid_loop's CUTK): STRAG_CAP records of (i, j, length, A[W], B[W])
// with the numbers least significant word first (not top-aligned), word-major: record r's word k at
// rec[k * STRAG_CAP + r], so the lanes of a warp store and load consecutive words.
constexpr int STRAG_CAP = 64;
template <int W>
__host__ __device__ constexpr int strag_words() { return 3 + 2 * W; }

template <int W>
struct HitSink {
    uint32_t *hits;
    uint64_t cap;
    unsigned long long *count;
    uint32_t i, j;
    uint32_t *strag = nullptr;  // this warp's straggler buffer (CUTK)
    int *nstrag = nullptr;      // its fill level (warp-uniform)
    int cutk = -1;              // cut when at most cutk lanes still run (-1: never)
    // Store the running lanes' pairs (registers top-aligned at the warp-uniform s; word k of a
    // number in register s + k) least significant word first, with A's length lA (A >= B).
    __device__ __forceinline__ void cut(bool run, const uint32_t (&A)[W], const uint32_t (&B)[W], int s, int lA) {
        const int lane = threadIdx.x & 31;
        unsigned b = __ballot_sync(FULL, run);
        int slot = *nstrag + __popc(b & ((1u << lane) - 1u));
        if (run) {
            uint32_t *r = strag + slot;
            r[0] = i;
            r[STRAG_CAP] = j;
            r[2 * STRAG_CAP] = (uint32_t)lA;
#pragma unroll
            for (int k = 0; k < W; ++k) {
                if (k >= s) {
                    r[(3 + k - s) * STRAG_CAP] = A[k];
                    r[(3 + W + k - s) * STRAG_CAP] = B[k];
                }
            }
        }
        *nstrag += __popc(b);
    }
    // a lane that stops with Y != 0 is coprime-mode ("return 1", L243/L251): nothing to report
    __device__ __forceinline__ bool quick(bool fin, int, uint64_t, int lY, uint64_t) { return fin && lY == 0; }
    // In the hot loop a lane only finishes with Y = X' != 0 (a zero X' sets `post` and goes cold):
    // it is coprime-mode, nothing to report.
    __device__ __forceinline__ bool quick_hot(bool, int, uint64_t, int, uint64_t) { return false; }
    // Compacting hit writer: warp ballot + one atomic per warp (north_star (4)).
    __device__ __forceinline__ void cold(bool hit, uint32_t (&X)[W], uint32_t (&Y)[W], int lX, uint64_t tX, int lY,
                                         uint64_t tY, int s) {
        unsigned mask = __ballot_sync(FULL, hit);
        const int lane = threadIdx.x & 31;
        const int leader = __ffs(mask) - 1;
        unsigned long long base = 0;
        if (lane == leader) base = atomicAdd(count, (unsigned long long)__popc(mask));
        base = __shfl_sync(FULL, base, leader);
        if (!hit) return;
        uint64_t slot = base + __popc(mask & ((1u << lane) - 1));
        if (slot >= cap) return;  // counted, not written: the host retries with more room
        uint32_t *rec = hits + slot * (2 + W);
        rec[0] = i;
        rec[1] = j;
#pragma unroll
        for (int k = 0; k < W; ++k) {
            if (k >= s) rec[2 + k - s] = X[k];
            if (k >= W - s) rec[2 + k] = 0u;
        }
    }
};

// ---- TMA (bulk async copy) staging of a cohort's operands into shared memory
// Per warp, a double buffer: while the warp runs cohort c, the copy engine
// brings cohort c+1's row block (W x 32 words, one contiguous W*128-byte
// block of the blocked layout) and column modulus (W words) into the other
// buffer, completing on an mbarrier (cp.async.bulk ... mbarrier::complete_tx).
template <int W>
struct StageBuf {
    uint32_t row[W * 32];
    uint32_t col[W];
};

// CTA shape of the all-pairs kernel, by width: warps are independent (each claims its
// own cohorts from the atomic cursor), so the CTA size only decides how the resident
// warps are grouped.  W <= 32: one warp per CTA, 20 CTAs/SM (cfg3 246.7 -> 240.9 ms against
// 4-warp CTAs at the same 20 warps/SM, 96 registers; 19: 242.5, 21 (80 registers): 244.6).
// W = 64: 4-warp CTAs (one-warp CTAs: cfg4 851 -> 1,592 ms).
#ifndef BULKGCD_AP_THREADS_NARROW
#define BULKGCD_AP_THREADS_NARROW 32
#endif
#ifndef BULKGCD_AP_THREADS_W64
#define BULKGCD_AP_THREADS_W64 128
#endif
template <int W>
struct ApCfg {
    static constexpr int threads = W <= 32 ? BULKGCD_AP_THREADS_NARROW : BULKGCD_AP_THREADS_W64;
    static constexpr int warps_per_cta = threads / 32;
    static constexpr int warps = Occ<W>::warps;  // resident warps per SM (register budget)
    static constexpr int blocks = warps / warps_per_cta > 0 ? warps / warps_per_cta : 1;
};

template <int W>
constexpr size_t allpairs_smem_bytes() {
    return ApCfg<W>::warps_per_cta * (2 * sizeof(StageBuf<W>) + 2 * sizeof(unsigned long long));
}

__device__ __forceinline__ uint32_t smem_addr(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void mbar_init(unsigned long long *bar, unsigned count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_addr(bar)), "r"(count) : "memory");
}

__device__ __forceinline__ void mbar_expect_tx(unsigned long long *bar, unsigned bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_addr(bar)), "r"(bytes)
                 : "memory");
}

__device__ __forceinline__ void mbar_wait(unsigned long long *bar, unsigned phase) {
    asm volatile(
        "{\n\t.reg .pred p;\n"
        "WAIT_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
        "@!p bra WAIT_%=;\n}" ::"r"(smem_addr(bar)),
        "r"(phase)
        : "memory");
}

__device__ __forceinline__ void tma_bulk_g2s(void *dst, const void *src, unsigned bytes, unsigned long long *bar) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(smem_addr(dst)),
        "l"(src), "r"(bytes), "r"(smem_addr(bar))
        : "memory");
}

// cohort id -> (row block b, column j): largest b with P(b) <= c
__device__ __forceinline__ void cohort_coords(uint64_t c, uint64_t n, uint64_t &b, uint64_t &j) {
    uint64_t nb = (n + 31) / 32;
    uint64_t lo = 0, hi = nb;  // P(lo) <= c < P(hi)
    while (hi - lo > 1) {
        uint64_t mid = (lo + hi) / 2;
        if (cohorts_before(mid, n) <= c) lo = mid; else hi = mid;
    }
    b = lo;
    j = 32 * b + 1 + (c - cohorts_before(b, n));
}

// Complement-form pass (gen_duff.py emit_cmpl) in the all-pairs kernel, by width:
// measured on B200, cfg4 (2048-bit) 899.7 -> 852.1 ms, but cfg3 (1024-bit) 246.8 -> 255.1 ms
// and cfg6 (512-bit) 82.6 -> 83.9 ms (more spills at 96 / 64 registers): W = 64 only.
#ifndef BULKGCD_ALLPAIRS_CMPL_MIN_W
#define BULKGCD_ALLPAIRS_CMPL_MIN_W 64
#endif
template <int W>
__host__ __device__ constexpr bool allpairs_cmpl() { return W >= BULKGCD_ALLPAIRS_CMPL_MIN_W; }

// Straggler cut threshold of the all-pairs kernel by width (0: off; never with the complement form).
// Measured (cfg6 / cfg3): W = 16 79.2 -> 77.5 ms at 8, 77.3 ms at 12 (lane efficiency 0.870 -> 0.951);
// W = 32 229.5 -> 240.9 / 255.2 / 270.1 ms at 4 / 8 / 12 although warp-iterations drop 5 %: a batch
// mixes lanes of different cohorts and lengths, whose tops fall below the 5-register window (slow
// steps and window misses per pair 0.020 -> 0.063 at 8), and every such cold exit spills the state.
template <int W>
__host__ __device__ constexpr int allpairs_cutk() { return W <= 16 ? 12 : 0; }

#ifdef BULKGCD_MAXNREG
#define BULKGCD_AP_BOUNDS(W) __maxnreg__(BULKGCD_MAXNREG)
#else
#define BULKGCD_AP_BOUNDS(W) __launch_bounds__(ApCfg<W>::threads, ApCfg<W>::blocks)
#endif

template <int W, bool STATS>
__global__ void BULKGCD_AP_BOUNDS(W) allpairs_kernel(AllPairsArgs a) {
    extern __shared__ __align__(128) unsigned char smem_raw[];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    StageBuf<W> *buf = reinterpret_cast<StageBuf<W> *>(smem_raw) + 2 * warp;
    unsigned long long *bar =
        reinterpret_cast<unsigned long long *>(smem_raw + ApCfg<W>::warps_per_cta * 2 * sizeof(StageBuf<W>)) + 2 * warp;
    if (lane == 0) {
        mbar_init(&bar[0], 1);
        mbar_init(&bar[1], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncwarp();
    uint32_t iters = 0, nslow = 0, limbs = 0, slots = 0, passw = 0;
    unsigned phase[2] = {0, 0};
    constexpr unsigned kBytes = (W * 32 + W) * 4;

    // claim a cohort and (lane 0) start its copy into buffer `slot`
    auto claim = [&](int slot, uint64_t &c, uint64_t &b, uint64_t &j) -> bool {
        unsigned long long cc = 0;
        if (lane == 0) cc = atomicAdd(a.work, 1ull);
        c = __shfl_sync(FULL, cc, 0) + a.c_begin;
        if (c >= a.c_end) return false;
        cohort_coords(c, a.n, b, j);
        if (lane == 0) {
            mbar_expect_tx(&bar[slot], kBytes);
            tma_bulk_g2s(buf[slot].row, a.N_blk + b * W * 32, W * 32 * 4, &bar[slot]);
            tma_bulk_g2s(buf[slot].col, a.N_rm + j * W, W * 4, &bar[slot]);
        }
        return true;
    };

    // Straggler cut (euclid_loop's CUTK), W <= 32: this warp's buffer and fill level
    constexpr int kCutMax = allpairs_cutk<W>();
    const int kCut = a.strag ? kCutMax : -1;
    uint32_t *my_strag =
        a.strag ? a.strag + ((uint64_t)blockIdx.x * ApCfg<W>::warps_per_cta + warp) * strag_words<W>() * STRAG_CAP
                : nullptr;
    int nstrag = 0;

    // One work item per trip -- a cohort, or 32 stored stragglers once the buffer holds a full warp
    // of them (and at the end, whatever is left, run to completion) -- through a single inlined
    // euclid_loop (instruction cache).
    int slot = 0;
    uint64_t c, b, j;
    bool have = claim(0, c, b, j);
    for (;;) {
        int cnt = 0, cutk = kCut;
        if (kCutMax > 0 && nstrag >= 32) {
            cnt = 32;
        } else if (!have) {
            if (nstrag == 0) break;
            cnt = nstrag;  // < 32: the last batch, no further cut
            cutk = -1;
        }
        uint32_t A[W], B[W];
        bool live;
        uint32_t ri, rj;
        int s0 = 0;
        uint64_t c2 = 0, b2 = 0, j2 = 0;
        bool have2 = false;
        if (cnt == 0) {  // the next cohort: its operands were staged by TMA
            have2 = claim(slot ^ 1, c2, b2, j2);  // prefetch the one after
            mbar_wait(&bar[slot], phase[slot]);
            phase[slot] ^= 1;
            uint64_t i = 32 * b + lane;
            live = i < j;
            ri = (uint32_t)i;
            rj = (uint32_t)j;
#pragma unroll
            for (int k = 0; k < W; ++k) {
                A[k] = buf[slot].row[k * 32 + lane];  // conflict-free: one bank per lane
                B[k] = buf[slot].col[k];              // broadcast
            }
            __syncwarp();  // the buffer is refilled only after the next claim, i.e. after this read
        } else {  // stored stragglers (the top of the buffer), loaded top-aligned at their longest length
            nstrag -= cnt;
            const uint32_t *r = my_strag + nstrag + lane;
            live = lane < cnt;
            ri = live ? r[0] : 0u;
            rj = live ? r[STRAG_CAP] : 0u;
            int rl = live ? (int)r[2 * STRAG_CAP] : 0;
            s0 = W - (int)__reduce_max_sync(FULL, (unsigned)rl);
#pragma unroll
            for (int k = 0; k < W; ++k) {
                int q = k - s0;  // word q of the numbers sits in register s0 + q
                bool in = (q >= 0) & (q < rl);
                A[k] = in ? r[(3 + q) * STRAG_CAP] : 0u;
                B[k] = in ? r[(3 + W + q) * STRAG_CAP] : 0u;
            }
        }
        int lA, lB;
        uint64_t tA, tB;
        setup_pair<W>(A, B, lA, tA, lB, tB);
        lA = lA > 0 ? lA - s0 : 0;  // lengths count from the start register s0
        lB = lB > 0 ? lB - s0 : 0;
        HitSink<W> sink{a.hits, a.hit_cap, a.hit_count, ri, rj, my_strag, &nstrag, cutk};
        // SWAP_RESUME: cfg3 233.3 -> 232.0 ms, cfg6 80.7 -> 79.2 ms, cfg4 834.8 -> 832.4 ms (the exact
        // pairs kernel keeps three pass copies: with two, ptxas loses the uniform BRXU there, 3.74 -> 3.81 ms)
        euclid_loop<W, STATS, false, false, RsaCond, HitSink<W>, allpairs_cmpl<W>(), (W >= 64), true, 0, kCutMax>(
            A, B, lA, tA, lB, tB, live, RsaCond{a.half}, sink, s0, iters, nslow, limbs, slots, passw);
        if (cnt == 0) {
            slot ^= 1;
            have = have2;
            c = c2;
            b = b2;
            j = j2;
        }
    }
    if (STATS && a.stats) {
        atomicAdd(&a.stats[0], (unsigned long long)iters);
        atomicAdd(&a.stats[1], (unsigned long long)nslow);
        atomicAdd(&a.stats[2], (unsigned long long)limbs);
        atomicAdd(&a.stats[3], (unsigned long long)slots);  // lane-slots: warp-iterations x 32
        atomicAdd(&a.stats[4], (unsigned long long)passw);  // lane-words of pass issued
    }
}

// ------------------------------------------------- shared-memory-resident kernels
// 4096-bit (W = 128) bulk and all-pairs GCD with the operands in shared memory
// (smem_euclid.cuh); also reachable at W <= 64 through BULKGCD_FLAG_SMEM.
template <int W, bool RSA, bool STATS, int ALG>
__global__ void __launch_bounds__(SM_THREADS) pairs_smem_kernel(PairsArgs a) {
    extern __shared__ __align__(16) uint32_t sbuf[];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    constexpr int SW = smem_stride_words<W>();
    uint32_t *wb = sbuf + (size_t)warp * 2 * SW * 32;
    for (int k = W; k < SW; ++k) wb[k * 32 + lane] = wb[(SW + k) * 32 + lane] = 0u;  // zero pad (s_update_ls)
    uint32_t iters = 0, rare = 0, limbs = 0, betapos = 0;
    for (;;) {
        unsigned long long c = 0;
        if (lane == 0) c = atomicAdd(a.work, 1ull);
        c = __shfl_sync(FULL, c, 0);
        if (c * 32 >= a.m) break;
        uint64_t i = c * 32 + lane;
        bool valid = i < a.m;
        SOp X{wb + lane}, Y{wb + SW * 32 + lane};
        for (int k = 0; k < W; ++k) {
            X[k] = valid ? a.A[(uint64_t)k * a.m_pad + i] : 0u;
            Y[k] = valid ? a.B[(uint64_t)k * a.m_pad + i] : 0u;
        }
        uint32_t it0 = iters;
        if (ALG == ALG_APPROX) {  // lockstep loop: every lane of the warp takes part
            int lX = 0, lY = 0, k2 = 0;
            uint64_t tX = 0, tY = 0;
            bool go = valid;
            if (!RSA && valid) {
                int la = s_len(X, W), lb = s_len(Y, W);
                if (la == 0 || lb == 0) {  // gcd(x, 0) = x
                    SOp Z = la ? X : Y;
                    s_write_shifted(a.G + i, a.m_pad, Z, la ? la : lb, 0, W);
                    go = false;
                } else {  // L41: strip the common power of two k2 and every other factor 2
                    int ca = s_ctz(X, la), cb = s_ctz(Y, lb);
                    k2 = ca < cb ? ca : cb;
                    s_rshift(X, la);
                    s_rshift(Y, lb);
                }
            }
            if (go) s_setup(X, Y, lX, tX, lY, tY, W);
            s_euclid_ls<!RSA, STATS>(X, Y, lX, tX, lY, tY, a.half, go, iters, rare, limbs, betapos);
            if (go) {
                if (RSA) {
                    if (lY == 0) s_write_shifted(a.G + i, a.m_pad, X, lX, 0, W);  // g = X (L251)
                    else for (int w = 0; w < W; ++w) a.G[i + (uint64_t)w * a.m_pad] = w == 0 ? 1u : 0u;
                } else {
                    if (lY != 0) {  // Case 1 tail (lX <= 2)
                        uint64_t g = s_tail64<STATS>(s_value64(X, lX), s_value64(Y, lY), iters, limbs);
                        X[0] = (uint32_t)g;
                        X[1] = (uint32_t)(g >> 32);
                        lX = g >> 32 ? 2 : (g ? 1 : 0);
                    }
                    s_write_shifted(a.G + i, a.m_pad, X, lX, k2, W);
                }
            }
        } else if (valid) {
            int lX, lY;
            uint64_t tX, tY;
            if (RSA) {
                s_setup(X, Y, lX, tX, lY, tY, W);
                s_euclid<false, STATS, ALG>(X, Y, lX, tX, lY, tY, a.half, iters, rare, limbs, betapos);
                if (lY == 0) s_write_shifted(a.G + i, a.m_pad, X, lX, 0, W);  // g = X (L251)
                else for (int w = 0; w < W; ++w) a.G[i + (uint64_t)w * a.m_pad] = w == 0 ? 1u : 0u;
            } else {
                int la = s_len(X, W), lb = s_len(Y, W);
                if (la == 0 || lb == 0) {  // gcd(x, 0) = x
                    SOp Z = la ? X : Y;
                    s_write_shifted(a.G + i, a.m_pad, Z, la ? la : lb, 0, W);
                } else {  // L41: strip the common power of two k2 and every other factor 2
                    int ca = s_ctz(X, la), cb = s_ctz(Y, lb);
                    int k2 = ca < cb ? ca : cb;
                    s_rshift(X, la);
                    s_rshift(Y, lb);
                    s_setup(X, Y, lX, tX, lY, tY, W);
                    s_euclid<true, STATS, ALG>(X, Y, lX, tX, lY, tY, 0, iters, rare, limbs, betapos);
                    if (ALG == ALG_APPROX && lY != 0) {  // Case 1 tail (lX <= 2)
                        uint64_t g = s_tail64<STATS>(s_value64(X, lX), s_value64(Y, lY), iters, limbs);
                        X[0] = (uint32_t)g;
                        X[1] = (uint32_t)(g >> 32);
                        lX = g >> 32 ? 2 : (g ? 1 : 0);
                    }
                    s_write_shifted(a.G + i, a.m_pad, X, lX, k2, W);
                }
            }
        }
        if (a.iters && valid) a.iters[i] = iters - it0;
        __syncwarp();
    }
    if (STATS && a.stats) {
        atomicAdd(&a.stats[0], (unsigned long long)iters);
        atomicAdd(&a.stats[1], (unsigned long long)rare);
        atomicAdd(&a.stats[2], (unsigned long long)limbs);
        atomicAdd(&a.stats[3], (unsigned long long)iters);  // no lockstep accounting: lane-slots = iterations
        atomicAdd(&a.stats[4], (unsigned long long)limbs);
        atomicAdd(&a.stats[5], (unsigned long long)betapos);
    }
}

template <int W, bool STATS, int ALG>
__global__ void __launch_bounds__(SM_THREADS) allpairs_smem_kernel(AllPairsArgs a) {
    extern __shared__ __align__(16) uint32_t sbuf[];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    constexpr int SW = smem_stride_words<W>();
    uint32_t *wb = sbuf + (size_t)warp * 2 * SW * 32;
    for (int k = W; k < SW; ++k) wb[k * 32 + lane] = wb[(SW + k) * 32 + lane] = 0u;  // zero pad (s_update_ls)
    uint32_t iters = 0, rare = 0, limbs = 0, betapos = 0;
    for (;;) {
        unsigned long long cc = 0;
        if (lane == 0) cc = atomicAdd(a.work, 1ull);
        uint64_t c = __shfl_sync(FULL, cc, 0) + a.c_begin;
        if (c >= a.c_end) break;
        uint64_t b, j;
        cohort_coords(c, a.n, b, j);
        uint64_t i = 32 * b + lane;
        bool live = i < j;
        SOp X{wb + lane}, Y{wb + SW * 32 + lane};
        for (int k = 0; k < W; ++k) {
            X[k] = a.N_blk[(b * W + k) * 32 + lane];  // one coalesced 128-byte row per word
            Y[k] = a.N_rm[j * W + k];                 // the column modulus (broadcast)
        }
        int lX = 0, lY = 0;
        uint64_t tX = 0, tY = 0;
        if (ALG == ALG_APPROX) {  // lockstep loop: every lane of the warp takes part
            if (live) s_setup(X, Y, lX, tX, lY, tY, W);
            s_euclid_ls<false, STATS>(X, Y, lX, tX, lY, tY, a.half, live, iters, rare, limbs, betapos);
        } else if (live) {
            s_setup(X, Y, lX, tX, lY, tY, W);
            s_euclid<false, STATS, ALG>(X, Y, lX, tX, lY, tY, a.half, iters, rare, limbs, betapos);
        }
        bool hit = live && lY == 0;  // Y = 0: g = X has >= bits/2 bits (L251)
        unsigned mask = __ballot_sync(FULL, hit);
        if (mask) {  // compacting hit writer: ballot + one atomic per warp
            const int leader = __ffs(mask) - 1;
            unsigned long long base = 0;
            if (lane == leader) base = atomicAdd(a.hit_count, (unsigned long long)__popc(mask));
            base = __shfl_sync(FULL, base, leader);
            if (hit) {
                uint64_t slot = base + __popc(mask & ((1u << lane) - 1));
                if (slot < a.hit_cap) {
                    uint32_t *rec = a.hits + slot * (2 + W);
                    rec[0] = (uint32_t)i;
                    rec[1] = (uint32_t)j;
                    s_write_shifted(rec + 2, 1, X, lX, 0, W);
                }
            }
        }
        __syncwarp();
    }
    if (STATS && a.stats) {
        atomicAdd(&a.stats[0], (unsigned long long)iters);
        atomicAdd(&a.stats[1], (unsigned long long)rare);
        atomicAdd(&a.stats[2], (unsigned long long)limbs);
        atomicAdd(&a.stats[3], (unsigned long long)iters);
        atomicAdd(&a.stats[4], (unsigned long long)limbs);
        atomicAdd(&a.stats[5], (unsigned long long)betapos);
    }
}

}  // namespace bulkgcd

#include "hybrid_euclid.cuh"  // the 4096-bit all-pairs kernel (one operand in registers, one in shared memory)
