/*
 * bulkgcd.h -- C ABI of libbulkgcd, a B200 (sm_100a) implementation of bulk
 * GCD computation with the Approximate Euclidean algorithm of
 *   T. Fujita, K. Nakano, Y. Ito, "Bulk GCD Computation Using a GPU to Break
 *   Weak RSA Keys", IPDPSW 2015  (cited as PAPER.md L<line>).
 *
 * Numbers.  A `bits`-bit number is W = bits/32 little-endian 32-bit words
 * ("d = 32", L251): word k (0 = least significant) of number i is at
 * X[i*W + k] ("row-major").  Supported bits: 512, 1024, 2048, 4096 (W = 16, 32,
 * 64, 128).  W <= 64 run register-resident kernels; W = 128 runs the
 * shared-memory-resident kernels (the operands do not fit in registers).
 *
 * Modes.
 *   EXACT (BULKGCD_MODE_EXACT): the exact gcd of any operands 0 <= a, b <
 *     2^bits, including even values and zero: gcd(x, 0) = x, gcd(0, 0) = 0,
 *     and the even-input reduction of L41; the Approximate Euclidean
 *     algorithm (L107, approx() of L127) runs until Y = 0 ("non-terminate").
 *   RSA (BULKGCD_MODE_RSA): the early-terminate algorithm (L243)
 *     for odd operands > 1: the loop stops once Y has fewer than bits/2 bits;
 *     the result is g = gcd(a, b) if g has at least bits/2 bits, else 1
 *     (reading of the garbled epilogue L243 with L251).
 *
 * Errors.  Every entry point returns 0 on success or a negative BULKGCD_E*
 * code; it never aborts.  bulkgcd_strerror() names a code and
 * bulkgcd_last_error() returns the calling thread's last detailed message.
 *
 * Threading.  Reentrant; host entry points use the calling thread's
 * per-thread default CUDA stream and stream-ordered allocations, inputs are
 * never modified, and there is no global state besides a thread-local error
 * message and, once per device, a release threshold of 4 GiB on the device's
 * default memory pool (stream-ordered buffers stay cached between calls
 * instead of being unmapped at every synchronisation).
 */
#ifndef BULKGCD_H
#define BULKGCD_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define BULKGCD_OK 0
#define BULKGCD_EINVAL (-1) /* bad argument (null pointer with count > 0, unsupported bits, bad modulus) */
#define BULKGCD_ENOMEM (-2) /* host or device allocation failed */
#define BULKGCD_ECUDA (-3)  /* CUDA runtime/launch error (see bulkgcd_last_error) */
#define BULKGCD_ENODEV (-4) /* no sm_100 (B200-class) device visible */

#define BULKGCD_MODE_EXACT 0
#define BULKGCD_MODE_RSA 1

#define BULKGCD_FLAG_STATS 1u /* device entry points: accumulate iteration/slow-step counters */
#define BULKGCD_FLAG_SMEM 2u  /* device entry points: use the shared-memory-resident kernels (the W = 128
                                 design) at any width -- a diagnostic/test route, same results */
/* Comparison algorithms of the paper's Tables IV/V, device entry points only;
 * same results (gcd / RSA-mode hits), different iteration counts.  Default: Approximate Euclid (E). */
#define BULKGCD_FLAG_ALGO_FAST_BINARY (1u << 8) /* (D) Fast Binary Euclid, L43: X <- rshift(X - Y) */
#define BULKGCD_FLAG_ALGO_BINARY (2u << 8)      /* (C) Binary Euclid, L57: X/2, Y/2 or (X - Y)/2 */
#define BULKGCD_FLAG_ALGO_MASK (3u << 8)

/* Hits of bulkgcd_all_pairs; arrays are allocated by the library. */
typedef struct {
    size_t count;      /* number of hits */
    uint32_t (*ij)[2]; /* ij[h] = {i, j}, i < j, sorted ascending by (i, j) */
    uint32_t *gcd;     /* gcd[h*W + k]: word k of gcd(N[i], N[j]) */
    uint32_t bits;     /* the call's bits (W = bits/32) */
} bulkgcd_hits_t;

/*
 * G[i] = gcd(A[i], B[i]) for i < m, exact mode.
 * A, B, G: host, row-major, m*W words each; G is caller-allocated.  m = 0 is a
 * no-op.  Errors: EINVAL (null pointer with m > 0, unsupported bits), ENOMEM,
 * ECUDA, ENODEV.
 */
int bulkgcd_pairs(const uint32_t *A, const uint32_t *B, size_t m, uint32_t bits, uint32_t *G);

/*
 * bulkgcd_pairs with a mode (BULKGCD_MODE_EXACT or BULKGCD_MODE_RSA) and an
 * optional iters[m] output (host, may be NULL): the number of do-while
 * iterations of the Approximate Euclidean algorithm each pair took (Table IV,
 * L239).  In RSA mode every operand must be odd and > 1 (else EINVAL) and
 * G[i] = g if bitlen(g) >= bits/2 else 1.
 */
int bulkgcd_pairs_ex(const uint32_t *A, const uint32_t *B, size_t m, uint32_t bits, int mode, uint32_t *G,
                     uint32_t *iters);

/*
 * All-pairs weak-key search (L431, L437, L453): for every i < j < n, RSA mode
 * on (N[i], N[j]); reports (i, j, g) iff g = gcd(N[i], N[j]) has at least
 * bits/2 bits, with g exact.  N: host, row-major, n*W words; every N[i] must
 * be odd and > 1 (else EINVAL).  n < 2 gives 0 hits.  *hits_out is filled
 * with library-allocated arrays (release with bulkgcd_hits_free); rows are
 * sorted by (i, j).  Duplicate moduli are reported with g = N[i].
 */
int bulkgcd_all_pairs(const uint32_t *N, size_t n, uint32_t bits, bulkgcd_hits_t *hits_out);

/* Release the arrays of a bulkgcd_hits_t (safe on a zeroed struct). */
void bulkgcd_hits_free(bulkgcd_hits_t *hits);

const char *bulkgcd_strerror(int code);
const char *bulkgcd_last_error(void);

/* 0 if the current CUDA device is an sm_100 part, else ENODEV/ECUDA. */
int bulkgcd_device_check(void);

/* ------------------------------------------------------------------------
 * Device-level entry points (pointers are CUDA device pointers owned by the
 * caller, e.g. torch tensors; calls are asynchronous on `stream`, a
 * cudaStream_t or NULL for the legacy default stream).  Used by the multi-GPU
 * driver (one process per GPU) and by benchmarks that keep data resident.
 * --------------------------------------------------------------------- */

/*
 * Word-interleaved ("column-wise", L361 and Fig. 3) layout: word k of item i
 * at X_cm[k*m_pad + i], m_pad >= m, multiple of 32.  to_interleaved = 1:
 * row-major d_in[m][W] -> d_out[W][m_pad] (padding zeroed); 0: the inverse.
 */
int bulkgcd_interleave(const uint32_t *d_in, uint32_t *d_out, size_t m, size_t m_pad, uint32_t bits,
                       int to_interleaved, void *stream);

/*
 * Blocked layout of the moduli for the all-pairs kernel: block b holds N[32b
 * .. 32b+31] interleaved, d_N_blk[(b*W + k)*32 + t] = word k of N[32b + t]
 * (zero padded).  d_N_blk needs bulkgcd_blocked_words(n, bits) words.
 */
int bulkgcd_layout_blocked(const uint32_t *d_N, uint32_t *d_N_blk, size_t n, uint32_t bits, void *stream);
size_t bulkgcd_blocked_words(size_t n, uint32_t bits);

/*
 * Number of all-pairs work units ("cohorts": 32 consecutive rows i x one
 * column j, i < j) for n moduli.  Cohort ids are ordered row block by row
 * block, so a contiguous id range is a balanced row band of the pair triangle.
 */
uint64_t bulkgcd_cohort_count(size_t n);

/*
 * bulkgcd_pairs on device data: d_A, d_B, d_G interleaved [W][m_pad];
 * d_iters (may be NULL): per-pair iteration counts; d_scratch: >= 8
 * unsigned long long of device memory, zeroed by the call ([2] = summed
 * iterations, [3] = slow-path steps, [4] = limb-steps = sum of lX over all
 * iterations, [5] = lane-slots, when flags has BULKGCD_FLAG_STATS or d_iters
 * is given; the shared-memory kernels (W = 128 or BULKGCD_FLAG_SMEM) count
 * beta > 0 updates and rshifts by >= 32 bits as [3], set [5] = [2], [6] = [4],
 * and add [7] = iterations with beta > 0, the statistic of L253).  No
 * validation of operand values.
 */
int bulkgcd_pairs_device(const uint32_t *d_A, const uint32_t *d_B, uint32_t *d_G, size_t m, size_t m_pad,
                         uint32_t bits, int mode, uint32_t *d_iters, unsigned long long *d_scratch,
                         unsigned flags, void *stream);

/*
 * One GPU's share of the all-pairs search: cohorts [cohort_begin, cohort_end)
 * over moduli d_N (row-major, n*W) and d_N_blk (bulkgcd_layout_blocked).  Hit
 * records go to d_hits[h*(2+W) ...] = {i, j, g[0..W-1]} in completion order;
 * d_counters (>= 8 unsigned long long, device) is zeroed by the call, then
 * [0] = number of hits found (records beyond hit_cap are counted but not
 * written: retry with a larger buffer); with BULKGCD_FLAG_STATS, [2] = summed
 * iterations, [3] = slow-path steps, [4] = limb-steps (sum of lX, the words
 * each update pass covers), [5] = lane-slots (32 x warp-iterations; [2]/[5]
 * is the SIMT lane efficiency), [6] = lane-words issued by the passes ([4]/[6]
 * is the pass-word efficiency); the shared-memory kernels as for
 * bulkgcd_pairs_device, with [7] = iterations with beta > 0 (L253).  Moduli
 * must be odd and > 1 (not checked here).  At 512 bits the call also takes a
 * stream-ordered scratch buffer from the device's default pool for the
 * kernel's straggler cut (~42 MiB, released on `stream` after the launch).
 */
int bulkgcd_all_pairs_band(const uint32_t *d_N, const uint32_t *d_N_blk, size_t n, uint32_t bits,
                           uint64_t cohort_begin, uint64_t cohort_end, uint32_t *d_hits, uint64_t hit_cap,
                           unsigned long long *d_counters, unsigned flags, void *stream);

/*
 * Factor output: "if gcd(n1, n2) = p != 1
 * then n1 = p * (n1/p)".  For every hit h of a bulkgcd_all_pairs result on the
 * same N and bits, F[(2h)*W + k] = word k of N[i] / g and F[(2h+1)*W + k] =
 * word k of N[j] / g (exact division by the odd g, on the GPU).
 * N: host row-major n*W words; F: host, caller-allocated, 2*count*W words.
 * Errors: EINVAL (null pointer with count > 0, bits mismatch, an index >= n, or
 * a g that is zero, even or does not divide its modulus), ENOMEM, ECUDA, ENODEV.
 */
int bulkgcd_cofactors(const uint32_t *N, size_t n, uint32_t bits, const bulkgcd_hits_t *hits, uint32_t *F);

/*
 * Device form: d_hits holds `count` records {i, j, g[W]} (the layout
 * bulkgcd_all_pairs_band writes), d_F receives 2*count*W words as above, and
 * *d_bad (device, zeroed by the caller) is incremented once per cofactor whose
 * record is invalid or whose g does not divide the modulus (that F row is then
 * meaningless).  Asynchronous on `stream`.
 */
int bulkgcd_cofactors_device(const uint32_t *d_N, size_t n, uint32_t bits, const uint32_t *d_hits, uint64_t count,
                             uint32_t *d_F, unsigned long long *d_bad, void *stream);

#ifdef __cplusplus
}
#endif

#endif /* BULKGCD_H */
