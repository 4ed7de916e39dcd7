// smem_euclid.cuh -- shared-memory-resident Approximate Euclid (4096-bit and up).
//
// At 4096 bits (W = 128) the two operands of a lane are 256 words: they cannot
// live in registers (SURVEY.md §7 H-c, §8(f) N1).  Here every lane keeps X and
// Y in shared memory, word k of a lane's operand at buf[k * 32 + lane] -- the
// paper's column-wise arrangement (L361, Fig. 3) at warp granularity, so every
// access of a warp is one conflict-free 32-bank wavefront whatever k each lane
// is at.  This is the paper's own design (X, Y in per-thread memory with a
// pointer swap, L227, L447) moved from Kepler local memory (DRAM) into
// on-chip shared memory:
//
//  * operands are least-significant-word first with per-lane lengths lX, lY
//    (Fig. 1); words at and above a length are zero;
//  * swap(X, Y) is a swap of two per-lane pointers (W4, L227);
//  * approx() is the paper's full case analysis (L127: Cases 1-4), on the cached
//    top pairs <x1x2>, <y1y2> (L115-L123);
//  * the update X <- rshift(X - alpha*Y) (beta = 0, W1, L233) is one fused
//    least-to-most-significant pass over lX words; beta > 0 (W2, L241) and an
//    rshift by >= 32 bits take a plain two-pass route.
//
// The same code serves exact mode (bulkgcd_pairs: L41 reduction, Case 1 in a
// 64-bit tail) and RSA mode (early terminate, L243/L251/L255), and is
// instantiated for W = 128 (the width that needs it) and, behind
// BULKGCD_FLAG_SMEM, for W = 16/32/64 so the tests can compare it with the
// register-resident kernels pair for pair.
#pragma once
#include <cstdint>

#include "euclid.cuh"  // div_floor_est / div_floor_fix

namespace bulkgcd {

// Algorithms (the paper's comparison columns, same harness):
//   ALG_APPROX       (E) Approximate Euclid, L107 -- the product
//   ALG_FAST_BINARY  (D) Fast Binary Euclid, L43: X <- rshift(X - Y), i.e. (alpha, beta) = (1, 0) (L111)
//   ALG_BINARY       (C) Binary Euclid, L57: X <- X/2 | Y <- Y/2 | X <- (X - Y)/2
enum { ALG_APPROX = 0, ALG_FAST_BINARY = 1, ALG_BINARY = 2 };

constexpr int SM_THREADS = 64;  // 2 warps per CTA: 2 x 2 x (W + SM_PAD) x 32 x 4 bytes = 68 KiB at W = 128
// Zero words above each operand buffer: the lockstep pass (s_update_ls) runs in 4-limb chunks up to
// 3 words past the longest operand and prefetches the next chunk (up to 8 past), all reading zeros.
constexpr int SM_PAD = 8;

template <int W>
__host__ __device__ constexpr int smem_stride_words() { return W + SM_PAD; }  // words per operand buffer

template <int W>
constexpr size_t smem_operand_bytes() {
    return (size_t)(SM_THREADS / 32) * 2 * smem_stride_words<W>() * 32 * sizeof(uint32_t);
}

template <int W>
constexpr int smem_blocks() {  // CTAs per SM: 227 KiB usable shared memory per SM
    return (int)((220u * 1024u) / (smem_operand_bytes<W>() + 256)) > 8 ? 8
                                                                        : (int)((220u * 1024u) / (smem_operand_bytes<W>() + 256));
}

// One lane's operand: word k at p[32 k].
struct SOp {
    uint32_t *p;
    __device__ __forceinline__ uint32_t &operator[](int k) const { return p[k * 32]; }
};

__device__ __forceinline__ int s_len(SOp x, int from) {  // significant words, scanning down from `from`
    int l = from;
    while (l > 0 && x[l - 1] == 0u) --l;
    return l;
}

__device__ __forceinline__ uint64_t s_top(SOp x, int l) {  // <x1 x2> (L115): top two words, x1 non-zero
    if (l <= 0) return 0;
    return ((uint64_t)x[l - 1] << 32) | (l >= 2 ? x[l - 2] : 0u);
}

__device__ __forceinline__ int s_cmp(SOp x, int lx, uint64_t tx, SOp y, int ly, uint64_t ty) {
    if (lx != ly) return lx < ly ? -1 : 1;
    if (tx != ty) return tx < ty ? -1 : 1;
    for (int k = lx - 3; k >= 0; --k) {
        uint32_t a = x[k], b = y[k];
        if (a != b) return a < b ? -1 : 1;
    }
    return 0;
}

__device__ __forceinline__ uint64_t s_value64(SOp x, int l) {  // l <= 2
    return l == 0 ? 0ull : (l == 1 ? (uint64_t)x[0] : (((uint64_t)x[1] << 32) | x[0]));
}

// rshift (L37) of an n-word operand in place (any shift, including >= 32 bits).
__device__ __forceinline__ void s_rshift(SOp x, int n) {
    int q = 0;
    while (q < n && x[q] == 0u) ++q;
    if (q == n) return;
    uint32_t b = __clz(__brev(x[q]));
    for (int k = 0; k < n; ++k) {
        uint32_t lo = (k + q < n) ? x[k + q] : 0u;
        uint32_t hi = (k + q + 1 < n) ? x[k + q + 1] : 0u;
        x[k] = b ? ((lo >> b) | (hi << (32 - b))) : lo;
    }
}

// approx(X, Y) of L127 for lX >= 3 (Cases 2-4; Case 1 is the 64-bit tail).  Every case is
// one quotient num div den < 2^32 (L133); it is taken exactly as in the register kernels: an
// FP64 estimate (div_floor_est) and, for the rare estimates within 2^-16 of an integer, the
// exact 96-bit check (div_floor_fix) -- instead of a 64-bit integer division subroutine.
__device__ __forceinline__ void s_approx(int lX, uint64_t tX, int lY, uint64_t tY, uint32_t &alpha, int &beta) {
    uint32_t x1 = (uint32_t)(tX >> 32), y1 = (uint32_t)(tY >> 32);
    uint64_t num = tX, den;
    if (lY == 1) {
        if (x1 >= y1) { num = x1; den = y1; beta = lX - 1; }                  // Case 2-A
        else { den = y1; beta = lX - 2; }                                     // Case 2-B
    } else if (lY == 2) {
        if (tX >= tY) { den = tY; beta = lX - 2; }                            // Case 3-A
        else { den = (uint64_t)y1 + 1; beta = lX - 3; }                       // Case 3-B
    } else if (tX > tY) { den = tY + 1; beta = lX - lY; }                    // Case 4-A
    else if (lX > lY) { den = (uint64_t)y1 + 1; beta = lX - lY - 1; }        // Case 4-B
    else { num = 1; den = 1; beta = 0; }                                      // Case 4-C: (1, 0)
    if (den == 1) {
        alpha = (uint32_t)num;  // 4-C, or a divisor of 1 (then num < 2^32, L133)
        return;
    }
    bool near;
    uint32_t qhi;
    uint32_t q = div_floor_est(num, den, near, qhi);
    if (near) q = div_floor_fix(num, den, qhi);
    alpha = q;  // < 2^32 outside Case 1 (L133); the bound alpha*D^beta <= X div Y is L123's
}

// One iteration's update of X (X >= Y > 0 odd, lX >= 3): beta = 0 -> X <- rshift(X - alpha*Y) with alpha
// made odd (L107); beta > 0 -> X <- rshift(X - alpha*Y*D^beta + Y) (L107, W2).  Returns true if it was a
// rare route (beta > 0 or a shift by >= 32 bits).
__device__ __forceinline__ bool s_update(SOp X, int lX, SOp Y, uint32_t alpha, int beta) {
    if (beta == 0) {
        alpha -= ~alpha & 1u;  // alpha is odd
        uint64_t p = (uint64_t)alpha * Y[0];
        uint32_t h = (uint32_t)(p >> 32);
        uint32_t x0 = X[0];
        uint32_t zp = x0 - (uint32_t)p;
        uint32_t br = x0 < (uint32_t)p;
        if (zp != 0u) {  // fused rshift by r < 32 (W1, L233): X[k-1] = (z_k : z_{k-1}) >> r
            uint32_t r = __clz(__brev(zp));
#pragma unroll 4
            for (int k = 1; k < lX; ++k) {
                uint64_t q = (uint64_t)alpha * Y[k] + h;
                h = (uint32_t)(q >> 32);
                uint64_t d = (uint64_t)X[k] - (uint32_t)q - br;
                uint32_t z = (uint32_t)d;
                br = (uint32_t)(d >> 63);
                X[k - 1] = __funnelshift_r(zp, z, r);
                zp = z;
            }
            X[lX - 1] = zp >> r;
            return false;
        }
        X[0] = 0u;  // z_0 = 0: plain subtraction, then rshift by >= 32 bits
        for (int k = 1; k < lX; ++k) {
            uint64_t q = (uint64_t)alpha * Y[k] + h;
            h = (uint32_t)(q >> 32);
            uint64_t d = (uint64_t)X[k] - (uint32_t)q - br;
            X[k] = (uint32_t)d;
            br = (uint32_t)(d >> 63);
        }
        s_rshift(X, lX);
        return true;
    }
    // beta > 0: X - alpha*Y*D^beta + Y, modulo 2^(32 lX): the result lies in [0, X] (alpha*D^beta <= X div Y,
    // L123), so the wrapped intermediate carries/borrows cancel.
    uint32_t c = 0;
    for (int k = 0; k < lX; ++k) {
        uint64_t s = (uint64_t)X[k] + Y[k] + c;
        X[k] = (uint32_t)s;
        c = (uint32_t)(s >> 32);
    }
    uint32_t h = 0, br = 0;
    for (int k = beta; k < lX; ++k) {
        uint64_t q = (uint64_t)alpha * Y[k - beta] + h;
        h = (uint32_t)(q >> 32);
        uint64_t d = (uint64_t)X[k] - (uint32_t)q - br;
        X[k] = (uint32_t)d;
        br = (uint32_t)(d >> 63);
    }
    s_rshift(X, lX);
    return true;
}

// Four limbs k..k+3 of the fused pass X <- rshift(X - alpha*Y) (W1, L233) in one PTX block:
// the product carry h rides in the 64-bit addend of mad.wide (IMAD.WIDE + IADD3 + IMAD.X),
// the borrow in the CC flag of a subc.cc chain, saved between chunks in b (0 or ~0u: one
// sub.cc to restore it, one subc to save it), and the funnel shift produces the words k-1..k+2
// of the shifted result from (zp, z_k..z_{k+3}).  (A two-borrow-chain form -- independent
// products, a shorter dependency per limb -- measured 7.9 -> 8.3 ms on cfg7: not taken.)
__device__ __forceinline__ void s_chunk4(const uint32_t (&x)[4], const uint32_t (&y)[4], uint32_t alpha, uint32_t r,
                                         uint32_t &h, uint32_t &b, uint32_t &zp, uint32_t (&o)[4]) {
    asm("{\n\t.reg .u32 lo, hi, z0, z1, z2, z3, t;\n\t.reg .u64 p, q;\n\t"
        "sub.cc.u32 t, 0, %6;\n\t"
        "mov.b64 q, {%5, 0};\n\tmad.wide.u32 p, %15, %11, q;\n\tmov.b64 {lo, hi}, p;\n\tsubc.cc.u32 z0, %7, lo;\n\t"
        "mov.b64 q, {hi, 0};\n\tmad.wide.u32 p, %15, %12, q;\n\tmov.b64 {lo, hi}, p;\n\tsubc.cc.u32 z1, %8, lo;\n\t"
        "mov.b64 q, {hi, 0};\n\tmad.wide.u32 p, %15, %13, q;\n\tmov.b64 {lo, hi}, p;\n\tsubc.cc.u32 z2, %9, lo;\n\t"
        "mov.b64 q, {hi, 0};\n\tmad.wide.u32 p, %15, %14, q;\n\tmov.b64 {lo, hi}, p;\n\tsubc.cc.u32 z3, %10, lo;\n\t"
        "subc.u32 %6, 0, 0;\n\t"
        "mov.u32 %5, hi;\n\t"
        "shf.r.wrap.b32 %0, %4, z0, %16;\n\tshf.r.wrap.b32 %1, z0, z1, %16;\n\t"
        "shf.r.wrap.b32 %2, z1, z2, %16;\n\tshf.r.wrap.b32 %3, z2, z3, %16;\n\t"
        "mov.u32 %4, z3;\n\t}"
        : "=r"(o[0]), "=r"(o[1]), "=r"(o[2]), "=r"(o[3]), "+r"(zp), "+r"(h), "+r"(b)
        : "r"(x[0]), "r"(x[1]), "r"(x[2]), "r"(x[3]), "r"(y[0]), "r"(y[1]), "r"(y[2]), "r"(y[3]), "r"(alpha),
          "r"(r));
}

// The beta = 0 update of the lockstep loop (s_euclid_ls): the same X <- rshift(X - alpha*Y) as
// s_update, but the pass runs to the warp-uniform bound L (the longest running lane's lX; the
// words of a shorter lane at and above its lX are zero and stay zero, since X - alpha*Y >= 0
// leaves no borrow or carry out of word lX - 1), in chunks of 4 limbs, so every running lane
// executes the same straight-line code, and it is software-pipelined: chunk c + 1 is loaded
// before chunk c is computed and stored (X and Y are different buffers and a store only
// writes a word already read).  Chunks may run past L into the SM_PAD zero words that pad
// every operand buffer (they read zeros and write zeros).  The rare routes (beta > 0, rshift
// by >= 32 bits) fall back to s_update.
__device__ __forceinline__ bool s_update_ls(SOp X, int lX, SOp Y, uint32_t alpha, int beta, int L) {
    if (beta != 0) return s_update(X, lX, Y, alpha, beta);
    alpha -= ~alpha & 1u;  // alpha is odd (L107)
    const uint32_t x0 = X[0], y0 = Y[0];
    uint64_t p = (uint64_t)alpha * y0;
    uint32_t h = (uint32_t)(p >> 32);
    uint32_t zp = x0 - (uint32_t)p;
    uint32_t b = x0 < (uint32_t)p ? ~0u : 0u;
    if (zp == 0u) return s_update(X, lX, Y, alpha, 0);  // rshift by >= 32 bits: the plain route
    const uint32_t r = __clz(__brev(zp));
    uint32_t xa[4], ya[4], xb[4], yb[4], o[4];
    const uint32_t *px = X.p, *py = Y.p;
#pragma unroll
    for (int i = 0; i < 4; ++i) {
        xa[i] = px[(1 + i) * 32];
        ya[i] = py[(1 + i) * 32];
    }
    int k0 = 1;
    for (;;) {
#pragma unroll
        for (int i = 0; i < 4; ++i) {  // prefetch the next chunk
            xb[i] = px[(k0 + 4 + i) * 32];
            yb[i] = py[(k0 + 4 + i) * 32];
        }
        s_chunk4(xa, ya, alpha, r, h, b, zp, o);
#pragma unroll
        for (int i = 0; i < 4; ++i) X[k0 - 1 + i] = o[i];
        k0 += 4;
        if (k0 >= L) break;
#pragma unroll
        for (int i = 0; i < 4; ++i) {
            xa[i] = px[(k0 + 4 + i) * 32];
            ya[i] = py[(k0 + 4 + i) * 32];
        }
        s_chunk4(xb, yb, alpha, r, h, b, zp, o);
#pragma unroll
        for (int i = 0; i < 4; ++i) X[k0 - 1 + i] = o[i];
        k0 += 4;
        if (k0 >= L) break;
    }
    X[k0 - 1] = zp >> r;  // top word of the last chunk (k0 - 1 >= L - 1; a zero word if above L - 1)
    return false;
}

// Binary Euclid step on one operand T (L57): T <- (T - c*Y) / 2, c in {0, 1}, lT words.
__device__ __forceinline__ void s_half_update(SOp T, int lT, SOp Y, uint32_t c) {
    uint32_t br = 0, zp = 0;
    for (int k = 0; k < lT; ++k) {
        uint32_t y = c ? Y[k] : 0u;
        uint64_t d = (uint64_t)T[k] - y - br;
        uint32_t z = (uint32_t)d;
        br = (uint32_t)(d >> 63);
        if (k > 0) T[k - 1] = __funnelshift_r(zp, z, 1);
        zp = z;
    }
    T[lT - 1] = zp >> 1;
}

// RSA-mode loop condition (L243/L251/L255): Y has at least `half` bits (half a multiple of 32).
__device__ __forceinline__ bool s_rsa_run(int lY, uint64_t tY, int half) {
    return 2 * lY + (int)((uint32_t)(tY >> 32) >> 31) > half / 16;
}

// The Approximate Euclidean loop (L107) of one lane on shared-memory operands,
// X >= Y on entry.  EXACT: until Y = 0, with Case 1 (lX <= 2) left to the
// caller's 64-bit tail; RSA: while bitlen(Y) >= half.  Counters: iterations,
// rare-route updates (beta > 0 or rshift >= 32 bits), limb-steps (sum of lX).
template <bool EXACT, bool STATS, int ALG = ALG_APPROX>
__device__ __forceinline__ void s_euclid(SOp &X, SOp &Y, int &lX, uint64_t &tX, int &lY, uint64_t &tY, int half,
                                         uint32_t &iters, uint32_t &rare, uint32_t &limbs, uint32_t &betapos) {
    for (;;) {
        // exact mode: (E) leaves Case 1 (lX <= 2) to the 64-bit tail; (C), (D) run to Y = 0
        bool run = EXACT ? ((lY >= 1) & (ALG != ALG_APPROX || lX >= 3)) : s_rsa_run(lY, tY, half);
        if (!run) break;
        if (ALG == ALG_BINARY) {
            bool xe = (X[0] & 1u) == 0, ye = (Y[0] & 1u) == 0;
            if (STATS) {
                ++iters;
                limbs += (!xe && ye) ? lY : lX;
            }
            if (!xe && ye) {  // Y <- Y/2 (Y shrinks: still Y <= X)
                s_half_update(Y, lY, Y, 0u);
                lY = s_len(Y, lY);
                tY = s_top(Y, lY);
                continue;
            }
            s_half_update(X, lX, Y, xe ? 0u : 1u);  // X <- X/2 or (X - Y)/2
        } else {
            uint32_t alpha = 1;
            int beta = 0;
            if (ALG == ALG_APPROX) s_approx(lX, tX, lY, tY, alpha, beta);
            if (STATS) {
                ++iters;
                limbs += lX;
                betapos += beta > 0;
            }
            bool r = s_update(X, lX, Y, alpha, beta);
            if (STATS) rare += r;
        }
        lX = s_len(X, lX);
        tX = s_top(X, lX);
        if (s_cmp(X, lX, tX, Y, lY, tY) < 0) {  // "if (X < Y) swap(X, Y)": a pointer swap (L227)
            SOp t = X; X = Y; Y = t;
            int tl = lX; lX = lY; lY = tl;
            uint64_t tt = tX; tX = tY; tY = tt;
        }
    }
}

// The Approximate Euclidean loop (ALG_APPROX) in warp lockstep: every lane of the warp calls
// it (`live` = the lane has a pair to run); each trip is one iteration of every still-running
// lane, with the fused pass bounded by the longest running operand (s_update_ls).  Same
// arithmetic, counters and results as s_euclid, lane for lane.
template <bool EXACT, bool STATS>
__device__ __forceinline__ void s_euclid_ls(SOp &X, SOp &Y, int &lX, uint64_t &tX, int &lY, uint64_t &tY, int half,
                                            bool live, uint32_t &iters, uint32_t &rare, uint32_t &limbs,
                                            uint32_t &betapos) {
    for (;;) {
        bool run = live && (EXACT ? ((lY >= 1) & (lX >= 3)) : s_rsa_run(lY, tY, half));
        if (!__any_sync(0xffffffffu, run)) break;
        const int L = (int)__reduce_max_sync(0xffffffffu, run ? (unsigned)lX : 0u);
        live = run;
        if (run) {
            uint32_t alpha;
            int beta;
            s_approx(lX, tX, lY, tY, alpha, beta);
            if (STATS) {
                ++iters;
                limbs += lX;
                betapos += beta > 0;
            }
            bool rr = s_update_ls(X, lX, Y, alpha, beta, L);
            if (STATS) rare += rr;
            lX = s_len(X, lX);
            tX = s_top(X, lX);
            if (s_cmp(X, lX, tX, Y, lY, tY) < 0) {  // "if (X < Y) swap(X, Y)": a pointer swap (L227)
                SOp t = X; X = Y; Y = t;
                int tl = lX; lX = lY; lY = tl;
                uint64_t tt = tX; tX = tY; tY = tt;
            }
        }
    }
}

// Exact-mode Case 1 (lX <= 2, L127): alpha = X div Y in 64-bit, to Y = 0.  Returns the gcd.
template <bool STATS>
__device__ __forceinline__ uint64_t s_tail64(uint64_t x, uint64_t y, uint32_t &iters, uint32_t &limbs) {
    while (y != 0) {
        if (STATS) {
            ++iters;
            limbs += (x >> 32) ? 2 : 1;  // lX of this iteration (the model's limb-step count)
        }
        uint64_t q = x / y;
        if ((q & 1) == 0) q -= 1;
        x = x - y * q;
        if (x) x >>= __ffsll((long long)x) - 1;
        if (x < y) { uint64_t t = x; x = y; y = t; }
    }
    return x;
}

// Order a lane's fresh operands so that X >= Y; lengths and tops.
__device__ __forceinline__ void s_setup(SOp &X, SOp &Y, int &lX, uint64_t &tX, int &lY, uint64_t &tY, int W) {
    lX = s_len(X, W);
    lY = s_len(Y, W);
    tX = s_top(X, lX);
    tY = s_top(Y, lY);
    if (s_cmp(X, lX, tX, Y, lY, tY) < 0) {
        SOp t = X; X = Y; Y = t;
        int tl = lX; lX = lY; lY = tl;
        uint64_t tt = tX; tX = tY; tY = tt;
    }
}

__device__ __forceinline__ int s_ctz(SOp x, int n) {  // trailing zero bits of a non-zero operand
    int q = 0;
    while (x[q] == 0u) ++q;
    return 32 * q + (int)__clz(__brev(x[q]));
}

// out[w * stride] = word w of (x << k2), w < W (x: l words).
__device__ __forceinline__ void s_write_shifted(uint32_t *out, uint64_t stride, SOp x, int l, int k2, int W) {
    int q = k2 >> 5, b = k2 & 31;
    for (int w = 0; w < W; ++w) {
        int src = w - q;
        uint32_t lo = (src >= 0 && src < l) ? x[src] : 0u;
        uint32_t lo1 = (src - 1 >= 0 && src - 1 < l) ? x[src - 1] : 0u;
        out[(uint64_t)w * stride] = b ? ((lo << b) | (lo1 >> (32 - b))) : lo;
    }
}

}  // namespace bulkgcd
