// factor.cuh -- factor output for the all-pairs hits.
//
// "if gcd(n1, n2) = p != 1 then n1 = p * (n1 / p)": once the
// all-pairs search reports (i, j, g), both moduli are factored by one exact
// division each.  One thread per cofactor (two per hit); hits are few, so the
// kernel is latency-bound and tiny next to the search.
//
// Exact division by an odd g (Hensel / Jebelean right-to-left division): with
// v = g[0]^-1 mod 2^32, quotient word k is q_k = r_k * v mod 2^32, where r is
// the running remainder after subtracting q_0..q_{k-1} times g; this yields
// q = n * g^-1 mod 2^(32W), which is n / g whenever g divides n.  The kernel
// then checks q * g == n over all 2W product words and counts a failure
// otherwise (the host turns that into BULKGCD_EINVAL).
#pragma once
#include <cstdint>

namespace bulkgcd {

// Inverse of an odd x modulo 2^32 by Newton's iteration (3 -> 6 -> 12 -> 24 -> 48 bits).
__device__ __forceinline__ uint32_t inv32(uint32_t x) {
    uint32_t v = x;  // x * x == 1 mod 8 for odd x
#pragma unroll
    for (int i = 0; i < 4; ++i) v *= 2u - x * v;
    return v;
}

// hits: records {i, j, g[W]}; F[(2h + side) * W + k] = word k of N[side ? j : i] / g.
template <int W>
__global__ void cofactor_kernel(const uint32_t *__restrict__ N, uint64_t n, const uint32_t *__restrict__ hits,
                                uint64_t count, uint32_t *__restrict__ F, unsigned long long *bad) {
    uint64_t t = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= 2 * count) return;
    uint64_t h = t >> 1;
    int side = (int)(t & 1);
    const uint32_t *rec = hits + h * (2 + W);
    uint64_t row = rec[side];
    const uint32_t *g = rec + 2;
    uint32_t *q = F + t * W;
    int lg = W;
    while (lg > 0 && g[lg - 1] == 0) --lg;
    if (row >= n || lg == 0 || (g[0] & 1u) == 0) {  // not a valid hit record: report, write zeros
        for (int k = 0; k < W; ++k) q[k] = 0;
        atomicAdd(bad, 1ull);
        return;
    }
    const uint32_t *x = N + row * W;
    uint32_t r[W];
    for (int k = 0; k < W; ++k) r[k] = x[k];
    const uint32_t v = inv32(g[0]);
    for (int k = 0; k < W; ++k) {
        uint32_t qk = r[k] * v;
        q[k] = qk;
        // r -= qk * g * 2^(32k) over words k .. W-1 (words beyond W are dropped: mod 2^(32W))
        uint64_t carry = 0;   // product carry
        uint32_t borrow = 0;  // subtraction borrow
        for (int w = 0; k + w < W; ++w) {
            uint64_t p = (uint64_t)qk * (w < lg ? g[w] : 0u) + carry;
            carry = p >> 32;
            uint64_t d = (uint64_t)r[k + w] - (uint32_t)p - borrow;
            r[k + w] = (uint32_t)d;
            borrow = (uint32_t)(d >> 63);
            if (w >= lg && carry == 0 && borrow == 0) break;
        }
    }
    // check: q * g == n exactly (2W-word product; the upper W words must vanish)
    bool ok = true;
    {
        uint32_t prod[2 * W];
        for (int k = 0; k < 2 * W; ++k) prod[k] = 0;
        for (int a = 0; a < W; ++a) {
            uint64_t c = 0;
            uint32_t qa = q[a];
            for (int b = 0; b < lg; ++b) {
                uint64_t p = (uint64_t)qa * g[b] + prod[a + b] + c;
                prod[a + b] = (uint32_t)p;
                c = p >> 32;
            }
            for (int k = a + lg; k < 2 * W && c; ++k) {
                uint64_t s = (uint64_t)prod[k] + c;
                prod[k] = (uint32_t)s;
                c = s >> 32;
            }
        }
        for (int k = 0; k < W; ++k) ok &= prod[k] == x[k];
        for (int k = W; k < 2 * W; ++k) ok &= prod[k] == 0u;
    }
    if (!ok) atomicAdd(bad, 1ull);
}

}  // namespace bulkgcd
