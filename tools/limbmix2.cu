// limbmix2.cu -- cost of candidate fused-limb formulations of X <- rshift(X - alpha*Y)
//
// Round-2 question: can the limb drop below the 5-instruction split form
// (IMAD.WIDE, IADD3 carry-add, IMAD.X, IADD3.X borrow, SHF.R.W)?
// The "complement" form keeps one operand bit-complemented: with X~ = D^n-1-X,
//   T = alpha*Y + X~  (mod D^n)  is the complement of Z = X - alpha*Y,
// so the subtract-with-borrow chain disappears and each limb is one
// multiply-accumulate  t_k + D c_k = alpha*m_k + a_k + c_{k-1}  (fits 64 bits).
// Variants (each over W = 32 register-resident words per lane, full passes):
//   S   current split form (gen_duff.py body)
//   Mu  MAC as two 64-bit adds  (mad.wide addend a_k, add.u64 carry)      + funnel
//   Mc  MAC with explicit add.cc/addc chains (lo+a, then +c)              + funnel
//   Ma  MAC: u = a_k + c (64-bit), mad.wide with 64-bit addend u          + funnel
//   *n  the same without the funnel shift
// Prints SMSP-cycles per warp-limb at 16 and 24 resident warps/SM.
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o build/limbmix2 tools/limbmix2.cu && build/limbmix2
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>

constexpr int W = 32;

enum { S, MU, MC, MA, SN, MUN, MCN, MAN, NV };
static const char *NAMES[] = {"S_split", "Mu_mac64", "Mc_mac_cc", "Ma_mac_addend", "S_noshift", "Mu_noshift",
                              "Mc_noshift", "Ma_noshift"};

template <int V>
__device__ __forceinline__ void mac(uint32_t a, uint32_t m, uint32_t al, uint32_t &c, uint32_t &t) {
    if (V == MU || V == MUN) {
        asm volatile(
            "{.reg .u64 p, q, w; cvt.u64.u32 q, %2; mad.wide.u32 p, %3, %4, q; cvt.u64.u32 w, %5; add.u64 p, p, w;"
            " mov.b64 {%0, %1}, p;}"
            : "=r"(t), "=r"(c) : "r"(a), "r"(al), "r"(m), "r"(c));
    }
    if (V == MC || V == MCN) {
        asm volatile(
            "{.reg .u64 p; .reg .u32 lo, hi; mul.wide.u32 p, %2, %3; mov.b64 {lo, hi}, p;"
            " add.cc.u32 lo, lo, %4; addc.u32 hi, hi, 0; add.cc.u32 %0, lo, %5; addc.u32 %1, hi, 0;}"
            : "=r"(t), "=r"(c) : "r"(al), "r"(m), "r"(a), "r"(c));
    }
    if (V == MA || V == MAN) {
        asm volatile(
            "{.reg .u64 p, u; .reg .u32 ul, uh; add.cc.u32 ul, %2, %5; addc.u32 uh, 0, 0; mov.b64 u, {ul, uh};"
            " mad.wide.u32 p, %3, %4, u; mov.b64 {%0, %1}, p;}"
            : "=r"(t), "=r"(c) : "r"(a), "r"(al), "r"(m), "r"(c));
    }
}

template <int V>
__device__ __forceinline__ void pass(uint32_t (&X)[W], const uint32_t (&Y)[W], uint32_t al, uint32_t r) {
    if (V == S || V == SN) {
        uint32_t lo, hi = 0, z, zp = 0;
        asm volatile("{.reg .u64 p; mul.wide.u32 p, %2, %3; mov.b64 {%0, %1}, p;}" : "=r"(lo), "=r"(hi) : "r"(al), "r"(Y[0]));
        asm volatile("sub.cc.u32 %0, %1, %2;" : "=r"(zp) : "r"(X[0]), "r"(lo));
        if (V == SN) X[0] = zp;
#pragma unroll
        for (int k = 1; k < W; ++k) {
            asm volatile("{.reg .u64 p, q; mov.b64 q, {%2, 0}; mad.wide.u32 p, %3, %4, q; mov.b64 {%0, %1}, p;}"
                         : "=r"(lo), "=r"(hi) : "r"(hi), "r"(al), "r"(Y[k]));
            asm volatile("subc.cc.u32 %0, %1, %2;" : "=r"(z) : "r"(X[k]), "r"(lo));
            if (V == S) X[k - 1] = __funnelshift_r(zp, z, r);
            else X[k] = z;
            zp = z;
        }
        if (V == S) X[W - 1] = __funnelshift_r(zp, 0xffffffffu, r);
        return;
    }
    // complement MAC: X <- (alpha*Y + X) >> r, ones shifted in at the top
    uint32_t c = 0, t, tp;
    mac<V>(X[0], Y[0], al, c, tp);
    if (V >= SN) X[0] = tp;
#pragma unroll
    for (int k = 1; k < W; ++k) {
        mac<V>(X[k], Y[k], al, c, t);
        if (V < SN) X[k - 1] = __funnelshift_r(tp, t, r);
        else X[k] = t;
        tp = t;
    }
    if (V < SN) X[W - 1] = __funnelshift_r(tp, 0xffffffffu, r);
}

template <int V>
__global__ void __launch_bounds__(128) kern(uint32_t *out, uint32_t seed, int iters) {
    uint32_t X[W], Y[W];
    const uint32_t *src = out + 64 + (blockIdx.x * 128 + threadIdx.x) % 1024;  // opaque operands
#pragma unroll
    for (int k = 0; k < W; ++k) {
        X[k] = src[k * 1024] * (threadIdx.x + 3);
        Y[k] = src[k * 1024 + 7] ^ seed;
    }
    uint32_t a = (seed + threadIdx.x) | 1, r = ((seed + threadIdx.x) & 7) + 1;
    for (int it = 0; it < iters; ++it) {
        pass<V>(X, Y, a, r);
        a += X[W - 1] & 2;  // loop-carried dependency through the result
    }
    uint32_t acc = 0;
#pragma unroll
    for (int k = 0; k < W; ++k) acc ^= X[k];
    if (acc == 0x12345678u) out[0] = acc;
}

template <int V>
static double run(int sms, double f, uint32_t *out, int warps) {
    const int blocks = sms * warps / 4, iters = 2000;
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    kern<V><<<blocks, 128>>>(out, 7, iters);
    cudaDeviceSynchronize();
    float best = 1e30f;
    for (int rep = 0; rep < 3; ++rep) {
        cudaEventRecord(e0);
        kern<V><<<blocks, 128>>>(out, 7, iters);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms;
        cudaEventElapsedTime(&ms, e0, e1);
        if (ms < best) best = ms;
    }
    double limbs = (double)blocks * 4 * iters * W;  // warp-limbs
    return best * 1e-3 * f * sms * 4 / limbs;       // SMSP-cycles per warp-limb
}

template <int V>
static void row(int sms, double f, uint32_t *out, bool &first) {
    for (int w : {16, 24}) {
        double c = run<V>(sms, f, out, w);
        printf("%s\"%s_w%d\": %.3f", first ? "" : ", ", NAMES[V], w, c);
        first = false;
    }
}

int main() {
    int sms = 0, clk_khz = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    cudaDeviceGetAttribute(&clk_khz, cudaDevAttrClockRate, 0);
    uint32_t *out;
    cudaMalloc(&out, (64 + 64 * 1024 + 64) * 4);
    cudaMemset(out, 0x5a, (64 + 64 * 1024 + 64) * 4);
    double f = clk_khz * 1e3;
    bool first = true;
    printf("{\"unit\": \"SMSP-cycles per warp-limb (attribute clock %d kHz)\", \"variants\": {", clk_khz);
    row<S>(sms, f, out, first);
    row<MU>(sms, f, out, first);
    row<MC>(sms, f, out, first);
    row<MA>(sms, f, out, first);
    row<SN>(sms, f, out, first);
    row<MUN>(sms, f, out, first);
    row<MCN>(sms, f, out, first);
    row<MAN>(sms, f, out, first);
    printf("}, \"cuda\": \"%s\"}\n", cudaGetErrorString(cudaGetLastError()));
    return 0;
}
