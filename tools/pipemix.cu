// pipemix.cu -- which sm_100a integer instructions share an issue pipe?
//
// Each thread runs CH independent chains of op A and CH of op B, interleaved
// 1:1 (B = none for the single-op rows), at full occupancy, so the rate is the
// pipe throughput, not latency.  Two ops that sit on different pipes reach
// ~the sum of their single rates; two on the same pipe stay at the single
// rate.  Prints one JSON object: warp-instructions / clock / SM (at the
// attribute clock; the loaded clock of this pool is the same 1965 MHz).
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o build/pipemix tools/pipemix.cu && build/pipemix
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>

#define REP 32
#define CH 6

enum { NONE, SHF, IMAD, IADD3, LOP3, IMADW, FFMA, SEL, IMADHI, IADDX, NOPS };
static const char *NAMES[] = {"none", "SHF", "IMAD", "IADD3", "LOP3", "IMAD.WIDE(addend)", "FFMA", "SEL", "IMAD.HI",
                              "IADD3.X-chain"};

template <int OP>
__device__ __forceinline__ void step(uint32_t (&v)[CH], uint64_t (&w)[CH], float (&f)[CH], uint32_t k, bool p) {
#pragma unroll
    for (int c = 0; c < CH; ++c) {
        const int n = (c + 1) % CH;
        if (OP == SHF) asm volatile("shf.r.wrap.b32 %0, %0, %1, %2;" : "+r"(v[c]) : "r"(v[n]), "r"(k));
        if (OP == IMAD) asm volatile("mad.lo.u32 %0, %0, %1, %2;" : "+r"(v[c]) : "r"(k), "r"(v[n]));
        if (OP == IADD3) asm volatile("add.u32 %0, %0, %1;" : "+r"(v[c]) : "r"(v[n]));
        if (OP == LOP3) asm volatile("xor.b32 %0, %0, %1;" : "+r"(v[c]) : "r"(v[n]));
        if (OP == IMADW) asm volatile("mad.wide.u32 %0, %1, %2, %0;" : "+l"(w[c]) : "r"((uint32_t)w[n]), "r"(k));
        if (OP == FFMA) asm volatile("fma.rn.f32 %0, %0, %1, %2;" : "+f"(f[c]) : "f"(f[n]), "f"(1.0001f));
        if (OP == SEL) asm volatile("{.reg .pred q; setp.ne.u32 q, %2, 0; selp.b32 %0, %0, %1, q;}" : "+r"(v[c]) : "r"(v[n]), "r"((uint32_t)p));
        if (OP == IMADHI) asm volatile("mad.hi.u32 %0, %0, %1, %2;" : "+r"(v[c]) : "r"(k), "r"(v[n]));
    }
    if (OP == IADDX) {  // CH carry chains of length CH: add.cc + addc.cc...
        asm volatile("add.cc.u32 %0, %0, %1;" : "+r"(v[0]) : "r"(v[1]));
#pragma unroll
        for (int c = 1; c < CH; ++c) asm volatile("addc.cc.u32 %0, %0, %1;" : "+r"(v[c]) : "r"(v[(c + 1) % CH]));
    }
}

template <int A, int B>
__global__ void __launch_bounds__(256) kern(uint32_t *out, uint32_t seed, int iters) {
    uint32_t a[CH], b[CH];
    uint64_t wa[CH], wb[CH];
    float fa[CH], fb[CH];
#pragma unroll
    for (int c = 0; c < CH; ++c) {
        a[c] = seed * (threadIdx.x + 1) + c;
        b[c] = seed ^ (c * 0x9E3779B9u) ^ threadIdx.x;
        wa[c] = a[c] * 0x100000001ull;
        wb[c] = b[c] * 0x100000001ull;
        fa[c] = (float)a[c];
        fb[c] = (float)b[c];
    }
    uint32_t k = (seed & 7) | 1;
    bool p = (threadIdx.x & 1) != 0;
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int r = 0; r < REP; ++r) {
            step<A>(a, wa, fa, k, p);
            step<B>(b, wb, fb, k, p);
        }
    }
    uint32_t acc = 0;
#pragma unroll
    for (int c = 0; c < CH; ++c) acc ^= a[c] ^ b[c] ^ (uint32_t)wa[c] ^ (uint32_t)wb[c] ^ __float_as_uint(fa[c] + fb[c]);
    if (acc == 0x12345678u) out[0] = acc;
}

template <int A, int B>
static double run(int sms, double f, uint32_t *out) {
    const int blocks = sms * 8, threads = 256, iters = 400;
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    kern<A, B><<<blocks, threads>>>(out, 7, iters);
    cudaDeviceSynchronize();
    cudaEventRecord(e0);
    kern<A, B><<<blocks, threads>>>(out, 7, iters);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    double ninst = (double)blocks * (threads / 32) * iters * REP * CH * ((A != NONE) + (B != NONE));
    double r = ninst / (ms * 1e-3) / f / sms;
    printf("%s\"%s%s%s\": %.3f", (A == SHF && B == NONE) ? "" : ", ", NAMES[A], B == NONE ? "" : "+", B == NONE ? "" : NAMES[B], r);
    return r;
}

int main() {
    int sms = 0, clk_khz = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    cudaDeviceGetAttribute(&clk_khz, cudaDevAttrClockRate, 0);
    uint32_t *out;
    cudaMalloc(&out, 64);
    double f = clk_khz * 1e3;
    printf("{\"sms\": %d, \"clock_khz_attr\": %d, \"unit\": \"warp-instructions/clk/SM\", \"rates\": {", sms, clk_khz);
    run<SHF, NONE>(sms, f, out);
    run<IMAD, NONE>(sms, f, out);
    run<IADD3, NONE>(sms, f, out);
    run<LOP3, NONE>(sms, f, out);
    run<IMADW, NONE>(sms, f, out);
    run<FFMA, NONE>(sms, f, out);
    run<SEL, NONE>(sms, f, out);
    run<IMADHI, NONE>(sms, f, out);
    run<IADDX, NONE>(sms, f, out);
    run<SHF, IMAD>(sms, f, out);
    run<IADD3, IMAD>(sms, f, out);
    run<LOP3, IMAD>(sms, f, out);
    run<SEL, IMAD>(sms, f, out);
    run<IADDX, IMAD>(sms, f, out);
    run<SHF, IMADW>(sms, f, out);
    run<IADDX, IMADW>(sms, f, out);
    run<SHF, IADD3>(sms, f, out);
    run<SHF, IADDX>(sms, f, out);
    run<IADD3, LOP3>(sms, f, out);
    run<SHF, FFMA>(sms, f, out);
    run<IADD3, FFMA>(sms, f, out);
    run<IMAD, FFMA>(sms, f, out);
    run<IMADW, FFMA>(sms, f, out);
    run<SHF, IMADHI>(sms, f, out);
    printf("}, \"cuda\": \"%s\"}\n", cudaGetErrorString(cudaGetLastError()));
    return 0;
}
