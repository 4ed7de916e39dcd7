// hybrid_euclid.cuh -- the 4096-bit all-pairs kernel: one operand in registers, one in
// shared memory (DESIGN.md §6 "hybrid").
//
// At W = 128 words the two operands of a lane (256 words) fit neither in registers nor,
// at a useful residency, in shared memory (both operands: 32 KiB per warp -> 6 warps/SM,
// latency-bound).  Here operand A stays in registers -- top-aligned like the 1024/2048-bit
// kernels (word i at register s + i, the warp-uniform pass start s, realigned when the warp
// length drops) -- and operand B in shared memory, least significant word first, one
// 32-lane row per word (the paper's column-wise arrangement, L361/Fig. 3, at warp
// granularity).  The roles alternate exactly as in euclid_loop: hot(A) updates A reading B
// (one LDS per limb), hot(B) updates B in place reading A (LDS + STS per limb).  B's word at
// register position k lives at [base + 128 k] with base = &B[0] - 128 s, so every access
// is a static immediate, and a realign (s += 1) only moves A's registers and the base.
// 16 KiB of shared memory per warp and 255 registers per thread: 8 warps/SM (at 168 registers,
// 12 warps/SM, ptxas spills operand words inside the passes: cfg7 11.0 ms against 5.9 ms).
//
// RSA mode (early terminate, L243/L251/L255) only: every running operand keeps >= W/2
// words, so the static windows and rows stay in range (the exact-mode 4096-bit bulk pairs
// keep the shared-memory kernels of smem_euclid.cuh).  Same approx() (exact floor), same
// fix-up codes and slow path as hot_iter / apply_fix, so per-pair iteration counts and
// results equal the model's and the other kernels'.
#pragma once
#include <cstdint>
#include <type_traits>

#include "euclid.cuh"

namespace bulkgcd {

__device__ __forceinline__ uint32_t h_lds(uint32_t addr) {
    uint32_t v;
    asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(addr) : "memory");
    return v;
}
__device__ __forceinline__ void h_sts(uint32_t addr, uint32_t v) {
    asm volatile("st.shared.u32 [%0], %1;" ::"r"(addr), "r"(v) : "memory");
}

constexpr int HWIN = 12;  // top window of the 4096-bit operands (the wider spread of long runs)

// One hot iteration of the hybrid loop: SIDE 'A' updates A (registers) with multiplicand B
// (shared memory), SIDE 'B' updates B with multiplicand A.  (lX, tX) are the updated
// operand's cached length and top pair, (lY, tY) the multiplicand's; as hot_iter<W, false>.
// `ap` = approx_pre<false>(lX, tX, lY, tY) (euclid.cuh: L127 Case 4, the exact floor, the odd alpha of
// L107), computed by the loop at the end of the previous iteration (hoisted ahead of its votes).
template <int W, char SIDE>
__device__ __forceinline__ void hot_iter_h(uint32_t (&A)[W], uint32_t base, int &lX, uint64_t &tX, int lY,
                                           uint64_t tY, int s, bool run, const Approx &ap, bool &full, bool &post,
                                           bool &lt) {
    full = ap.full;
    uint32_t alpha = (run & !full) ? ap.a : 0u;           // the pass is a no-op for every other lane
    uint32_t r;
    uint32_t zs = duff_hpass<W, PASS_G_HYBRID, SIDE>(A, alpha, s, base, r);
    uint64_t t;
    int p;
    if (SIDE == 'A') {
        p = scan_window<W, HWIN>(A, t);
    } else {
        uint32_t w[W];
#pragma unroll
        for (int k = W - HWIN - 1; k < W; ++k) w[k] = h_lds(base + 128u * k);
        p = scan_window<W, HWIN>(w, t);
    }
    int ln = p - s + 1;
    uint32_t d0, d1;
    int d2;
    asm("sub.cc.u32 %0, %3, %4;\n\tsubc.cc.u32 %1, %5, %6;\n\tsubc.s32 %2, %7, %8;"
        : "=r"(d0), "=r"(d1), "=r"(d2)
        : "r"(lo32(t)), "r"(lo32(tY)), "r"(hi32(t)), "r"(hi32(tY)), "r"(ln), "r"(lY));
    lt = d2 < 0;
    post = (zs == 0) | (hi32(t) == 0u) | ((d0 | d1 | (uint32_t)d2) == 0);
    lX = ln;
    tX = t;
}

// Per-lane exchange of A (registers) and B (shared memory), words at positions >= s.
template <int W>
__device__ __forceinline__ void h_swap(uint32_t (&A)[W], uint32_t base, int s) {
#pragma unroll
    for (int k = 0; k < W; ++k) {
        if (k >= s) {
            uint32_t b = h_lds(base + 128u * k);
            h_sts(base + 128u * k, A[k]);
            A[k] = b;
        }
    }
}

// Slow path (rare): both operands to local memory, one exact step (n_iterate / n_rshift of
// euclid.cuh), the order, back.  updB: B is the operand the last iteration updated.
template <int W>
__device__ __forceinline__ void h_slow_step(uint32_t (&A)[W], uint32_t base, int s, int mode, bool updB, int &lX,
                                            uint64_t &tX, int &lY, uint64_t &tY) {
    uint32_t x[W], y[W];
#pragma unroll
    for (int k = 0; k < W; ++k) {
        uint32_t b = k >= s ? h_lds(base + 128u * k) : 0u;
        x[k] = updB ? b : A[k];
        y[k] = updB ? A[k] : b;
    }
    int n = W - s;
    if (mode == 2)
        n_iterate(x + s, y + s, n);
    else
        n_rshift(x + s, n);
    n_order(x + s, y + s, n);
    lX = nlen(x + s, n);
    lY = nlen(y + s, n);
    tX = top_pair(x + s, lX);
    tY = top_pair(y + s, lY);
#pragma unroll
    for (int k = 0; k < W; ++k) {
        A[k] = updB ? y[k] : x[k];
        if (k >= s) h_sts(base + 128u * k, updB ? x[k] : y[k]);
    }
}

// The hybrid Euclid loop (RSA mode): euclid_loop's structure -- hot iterations with
// alternating roles, all warp decisions by vote, a cold section for fix-ups, finished
// lanes and realigns -- over A (registers) and B (shared memory, row 0 at bbase).
// lA/tA, lB/tB: lengths and tops; A >= B on entry (setup by the caller).
template <int W, bool STATS, class Sink>
__device__ __forceinline__ void hybrid_loop(uint32_t (&A)[W], uint32_t bbase, int &lA, uint64_t &tA, int &lB,
                                            uint64_t &tB, bool live, RsaCond cond, Sink &sink, uint32_t &iters,
                                            uint32_t &nslow, uint32_t &limbs, uint32_t &slots, uint32_t &passw) {
    int s = 0;
    int fix = 0;     // pending fix-up of the last iteration (fix_code)
    int resume = 0;  // roles of the next iteration: 0 -> A updated (X = A), 1 -> B updated
    Approx ap;       // approx() for the coming hot iteration
    auto base = [&]() { return bbase - 128u * (uint32_t)s; };

    // Cold section for the next roles; xb: X (the operand updated next) is B.
    auto cold = [&](bool xb, int &lX, uint64_t &tX, int &lY, uint64_t &tY) -> bool {
        if (__any_sync(FULL, fix != 0)) {
            if (STATS && fix >= 2) ++nslow;
            // the last iteration updated Y of these roles (the other operand)
            if (fix == 1) {
                h_swap<W>(A, base(), s);  // X' >= Y: "if (X < Y) swap" did not fire
                int tl = lX; lX = lY; lY = tl;
                uint64_t tt = tX; tX = tY; tY = tt;
            } else if (fix >= 2) {
                h_slow_step<W>(A, base(), s, fix, !xb, lY, tY, lX, tX);
            }
            fix = 0;
        }
        bool run = live & cond(lX, tX, lY, tY);
        bool fin = live & !run;
        if (__any_sync(FULL, fin)) {
            bool need = sink.quick(fin, lX, tX, lY, tY);
            if (__any_sync(FULL, need)) {
                if (xb && need) h_swap<W>(A, base(), s);  // the result X = g is in B: bring it to A
                sink.cold(need, A, A, lX, tX, lY, tY, s);
            }
        }
        live = run;
        unsigned brun = __ballot_sync(FULL, run);
        if (brun == 0u) return false;
        int L = __reduce_max_sync(FULL, (unsigned)(run ? lX : 0));
        while (W - s > L) {
            shift_up_1<W>(A);
            ++s;
        }
        return true;
    };
    // One hot iteration updating X (xb: X = B), then the next iteration's loop test.
    auto hot = [&](auto side, int &lX, uint64_t &tX, int &lY, uint64_t &tY) -> bool {
        constexpr char SIDE = decltype(side)::value;
        if (STATS) {
            ++slots;
            passw += W - s;
            if (live) {
                ++iters;
                limbs += lX;
            }
        }
        bool full, post, lt;
        hot_iter_h<W, SIDE>(A, base(), lX, tX, lY, tY, s, live, ap, full, post, lt);
        bool bad = live & (full | post | !lt);
        bool run = live & cond(lY, tY, lX, tX);
        bool fin = live & !run & !bad;
        bool need = sink.quick_hot(fin, lY, tY, lX, tX) | bad;
        bool top = run & (lY == W - s);
        ap = approx_pre<false>(lY, tY, lX, tX);  // the next iteration's roles, ahead of the votes
        bool any_need = __any_sync(FULL, need), any_top = __any_sync(FULL, top);
        if (any_need) {
            fix = fix_code(live, full, post, lt);
            return true;
        }
        if (!any_top) {  // the warp length dropped: realign one word in place (B: the base moves)
            unsigned brun = __ballot_sync(FULL, run);
            if (brun == 0u) {
                fix = fix_code(live, full, post, lt);
                return true;
            }
            shift_up_1<W>(A);
            ++s;
        }
        live = run;
        return false;
    };
    using SA = std::integral_constant<char, 'A'>;
    using SB = std::integral_constant<char, 'B'>;
    for (;;) {
        bool more = resume == 0 ? cold(false, lA, tA, lB, tB) : cold(true, lB, tB, lA, tA);
        if (!more) return;
        // Resuming with B updated next: exchange the operands (registers <-> shared memory) instead
        // of entering the loop at its second iteration, so the pass is inlined twice, not three
        // times (instruction cache; as euclid_loop's SWAP_RESUME).
        if (resume == 1) {
            h_swap<W>(A, base(), s);
            int tl = lA; lA = lB; lB = tl;
            uint64_t tt = tA; tA = tB; tB = tt;
            resume = 0;
        }
        ap = approx_pre<false>(lA, tA, lB, tB);
        for (;;) {
            if (hot(SA{}, lA, tA, lB, tB)) {
                resume = 1;
                break;
            }
            if (hot(SB{}, lB, tB, lA, tA)) {
                resume = 0;
                break;
            }
        }
    }
}

// ------------------------------------------------------------------ the kernel
#ifndef BULKGCD_HY_THREADS
#define BULKGCD_HY_THREADS 128
#endif
#ifndef BULKGCD_HY_BLOCKS
#define BULKGCD_HY_BLOCKS 2
#endif
constexpr int HY_THREADS = BULKGCD_HY_THREADS;  // 4 warps per CTA
constexpr int HY_BLOCKS = BULKGCD_HY_BLOCKS;    // 8 warps per SM: 255 registers (no spills in the hot loop), 16 KiB of B per warp

template <int W>
constexpr size_t hybrid_smem_bytes() {
    return (size_t)(HY_THREADS / 32) * W * 32 * sizeof(uint32_t);
}

#ifdef BULKGCD_HY_MAXNREG
#define BULKGCD_HY_BOUNDS __maxnreg__(BULKGCD_HY_MAXNREG)
#else
#define BULKGCD_HY_BOUNDS __launch_bounds__(HY_THREADS, HY_BLOCKS)
#endif
template <int W, bool STATS>
__global__ void BULKGCD_HY_BOUNDS allpairs_hybrid_kernel(AllPairsArgs a) {
    extern __shared__ __align__(16) uint32_t hbuf[];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const uint32_t bbase = (uint32_t)__cvta_generic_to_shared(hbuf + (size_t)warp * W * 32 + lane);
    uint32_t iters = 0, nslow = 0, limbs = 0, slots = 0, passw = 0;
    for (;;) {
        unsigned long long cc = 0;
        if (lane == 0) cc = atomicAdd(a.work, 1ull);
        uint64_t c = __shfl_sync(FULL, cc, 0) + a.c_begin;
        if (c >= a.c_end) break;
        uint64_t b, j;
        cohort_coords(c, a.n, b, j);
        uint64_t i = 32 * b + lane;
        bool live = i < j;
        uint32_t A[W];
        int lB = 0;
#pragma unroll
        for (int k = 0; k < W; ++k) {
            A[k] = a.N_blk[(b * W + k) * 32 + lane];  // the row modulus: one coalesced 128-byte row per word
            uint32_t v = a.N_rm[j * W + k];           // the column modulus (broadcast)
            h_sts(bbase + 128u * k, v);
            if (v != 0u) lB = k + 1;
        }
        uint64_t tB = lB ? (((uint64_t)h_lds(bbase + 128u * (lB - 1)) << 32) |
                            (lB >= 2 ? h_lds(bbase + 128u * (lB - 2)) : 0u))
                         : 0ull;
        uint64_t tA;
        int lA = scan_full<W>(A, tA) + 1;
        // order the pair so that A >= B (lengths, tops, then every word; duplicates compare equal)
        int cmp = lA != lB ? (lA < lB ? -1 : 1) : (tA != tB ? (tA < tB ? -1 : 1) : 0);
        if (cmp == 0) {
#pragma unroll
            for (int k = W - 1; k >= 0; --k) {
                uint32_t v = h_lds(bbase + 128u * k);
                if (cmp == 0 && A[k] != v) cmp = A[k] < v ? -1 : 1;
            }
        }
        if (cmp < 0) {
            h_swap<W>(A, bbase, 0);
            int tl = lA; lA = lB; lB = tl;
            uint64_t tt = tA; tA = tB; tB = tt;
        }
        HitSink<W> sink{a.hits, a.hit_cap, a.hit_count, (uint32_t)i, (uint32_t)j};
        hybrid_loop<W, STATS>(A, bbase, lA, tA, lB, tB, live, RsaCond{a.half}, sink, iters, nslow, limbs, slots,
                              passw);
        __syncwarp();
    }
    if (STATS && a.stats) {
        atomicAdd(&a.stats[0], (unsigned long long)iters);
        atomicAdd(&a.stats[1], (unsigned long long)nslow);
        atomicAdd(&a.stats[2], (unsigned long long)limbs);
        atomicAdd(&a.stats[3], (unsigned long long)slots);  // lane-slots: warp-iterations x 32
        atomicAdd(&a.stats[4], (unsigned long long)passw);
    }
}

}  // namespace bulkgcd
