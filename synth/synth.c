/*
 * synth.c -- seeded synthetic RSA-moduli generator (input generation only).
 *
 * Test/bench infrastructure shared by the CUDA path's tests and the oracle's
 * tests.  It holds NONE of the GCD method's arithmetic: it only draws
 * counter-based pseudo-random candidates and asks OpenSSL whether they are
 * (probable) primes, then multiplies two primes into a modulus n = p*q.
 *
 * Recipe (PAPER.md L239/L451
 * generate keys with the OpenSSL toolkit, which sets the top two bits of each
 * s/2-bit prime so that p*q has exactly s bits):
 *   prime #k of stream `seed`:  c0 = R(seed, k) mod 2^(pb) | 3 << (pb-2) | 1,
 *   then c0, c0+2, c0+4, ... until BN_check_prime() accepts it.
 *   R is SplitMix64 applied to a (seed, k, word) counter, so any prime can be
 *   regenerated independently of the others (and in parallel).
 *
 * Limbs are little-endian uint32 (limb 0 least significant), the layout of
 * include/bulkgcd.h.
 */
#include <openssl/bn.h>
#include <pthread.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

static uint64_t splitmix64(uint64_t x) {
    x += 0x9E3779B97F4A7C15ull;
    x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
    x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
    return x ^ (x >> 31);
}

/* 64 random bits for word `w` of candidate `k` in stream `seed`. */
static uint64_t counter_word(uint64_t seed, uint64_t k, uint64_t w) {
    uint64_t h = splitmix64(seed ^ 0x5EED5EED00000000ull);
    h = splitmix64(h ^ k);
    return splitmix64(h ^ (w * 0xD6E8FEB86659FD93ull));
}

static int bn_to_limbs(const BIGNUM *b, uint32_t *out, int nlimbs) {
    unsigned char buf[1024];
    int nbytes = nlimbs * 4;
    if (nbytes > (int)sizeof(buf)) return -1;
    if (BN_bn2lebinpad(b, buf, nbytes) != nbytes) return -1;
    for (int i = 0; i < nlimbs; ++i)
        out[i] = (uint32_t)buf[4 * i] | ((uint32_t)buf[4 * i + 1] << 8) |
                 ((uint32_t)buf[4 * i + 2] << 16) | ((uint32_t)buf[4 * i + 3] << 24);
    return 0;
}

static BIGNUM *limbs_to_bn(const uint32_t *in, int nlimbs) {
    unsigned char buf[1024];
    if (nlimbs * 4 > (int)sizeof(buf)) return NULL;
    for (int i = 0; i < nlimbs; ++i) {
        buf[4 * i] = (unsigned char)in[i];
        buf[4 * i + 1] = (unsigned char)(in[i] >> 8);
        buf[4 * i + 2] = (unsigned char)(in[i] >> 16);
        buf[4 * i + 3] = (unsigned char)(in[i] >> 24);
    }
    return BN_lebin2bn(buf, nlimbs * 4, NULL);
}

/* One prime of `pbits` bits (multiple of 32) -> out[pbits/32]. */
static int one_prime(uint32_t pbits, uint64_t seed, uint64_t k, uint32_t *out, BN_CTX *ctx) {
    int nl = (int)(pbits / 32);
    uint32_t limbs[256];
    for (int w = 0; w < (nl + 1) / 2; ++w) {
        uint64_t r = counter_word(seed, k, (uint64_t)w);
        limbs[2 * w] = (uint32_t)r;
        if (2 * w + 1 < nl) limbs[2 * w + 1] = (uint32_t)(r >> 32);
    }
    limbs[nl - 1] |= 0xC0000000u; /* top two bits set (OpenSSL-style) */
    limbs[0] |= 1u;               /* odd */
    BIGNUM *c = limbs_to_bn(limbs, nl);
    if (!c) return -1;
    int rc = -1;
    for (int step = 0; step < 1 << 20; ++step) {
        int p = BN_check_prime(c, ctx, NULL);
        if (p < 0) break;
        if (p == 1) {
            if (BN_num_bits(c) != (int)pbits) break; /* overflowed: cannot happen for sane pbits */
            rc = bn_to_limbs(c, out, nl);
            break;
        }
        if (!BN_add_word(c, 2)) break;
    }
    BN_free(c);
    return rc;
}

typedef struct {
    uint32_t pbits;
    uint64_t seed, first;
    size_t begin, end;
    uint32_t *out;
    int rc;
} job_t;

static void *worker(void *arg) {
    job_t *j = (job_t *)arg;
    BN_CTX *ctx = BN_CTX_new();
    j->rc = ctx ? 0 : -1;
    int nl = (int)(j->pbits / 32);
    for (size_t i = j->begin; i < j->end && j->rc == 0; ++i)
        j->rc = one_prime(j->pbits, j->seed, j->first + i, j->out + i * (size_t)nl, ctx);
    BN_CTX_free(ctx);
    return NULL;
}

/* Generate primes first..first+count-1 of stream `seed`, each `pbits` bits,
 * into out[count][pbits/32].  Returns 0 or -1. */
int synth_primes(uint32_t pbits, uint64_t seed, uint64_t first, size_t count, uint32_t *out,
                 int nthreads) {
    if (pbits < 64 || pbits % 32 || pbits > 8192 || !out) return -1;
    if (count == 0) return 0;
    if (nthreads < 1) nthreads = 1;
    if ((size_t)nthreads > count) nthreads = (int)count;
    pthread_t th[256];
    job_t jobs[256];
    if (nthreads > 256) nthreads = 256;
    size_t per = (count + nthreads - 1) / nthreads;
    for (int t = 0; t < nthreads; ++t) {
        size_t b = (size_t)t * per, e = b + per;
        if (b > count) b = count;
        if (e > count) e = count;
        jobs[t] = (job_t){pbits, seed, first, b, e, out, 0};
        if (pthread_create(&th[t], NULL, worker, &jobs[t])) jobs[t].rc = -1, th[t] = 0;
    }
    int rc = 0;
    for (int t = 0; t < nthreads; ++t) {
        if (th[t]) pthread_join(th[t], NULL);
        if (jobs[t].rc) rc = -1;
    }
    return rc;
}

/* out[i] = p[i] * q[i] (full product, 2*pl limbs); plain schoolbook, used only to
 * build the synthetic moduli. */
int synth_mul(const uint32_t *p, const uint32_t *q, size_t count, uint32_t pl, uint32_t *out) {
    for (size_t i = 0; i < count; ++i) {
        const uint32_t *a = p + i * pl, *b = q + i * pl;
        uint32_t *o = out + i * 2 * (size_t)pl;
        memset(o, 0, 8 * (size_t)pl);
        for (uint32_t x = 0; x < pl; ++x) {
            uint64_t c = 0;
            for (uint32_t y = 0; y < pl; ++y) {
                uint64_t t = (uint64_t)a[x] * b[y] + o[x + y] + c;
                o[x + y] = (uint32_t)t;
                c = t >> 32;
            }
            o[x + pl] = (uint32_t)c;
        }
    }
    return 0;
}
