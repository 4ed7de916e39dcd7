// pipemix3.cu -- which pipe runs FSEL (selp.f32) on sm_100a, and at what rate?  If FSEL is not on the
// ALU pipe, the window scan's selects (SEL: ALU, half rate) could move off the all-pairs kernel's busiest
// pipe.  Rates in SMSP-cycles per warp per (A step + B step), CH independent chains, full occupancy.
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o build/pipemix3 tools/pipemix3.cu && build/pipemix3
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>

#define REP 32
#define CH 6

enum { NONE, SEL, FSEL, SHF, IMAD, LOP3, IMNMX, PRMT, NOPS };
static const char *NAMES[] = {"none", "SEL", "FSEL", "SHF", "IMAD", "LOP3", "IMNMX", "PRMT"};

template <int OP>
__device__ __forceinline__ void step(uint32_t (&v)[CH], uint32_t k, uint32_t z) {
#pragma unroll
    for (int c = 0; c < CH; ++c) {
        const int n = (c + 1) % CH;
        if (OP == SEL) asm volatile("{.reg .pred q; setp.ne.u32 q, %2, 0; selp.b32 %0, %0, %1, q;}" : "+r"(v[c]) : "r"(v[n]), "r"(z));
        if (OP == FSEL)
            asm volatile("{.reg .pred q; .reg .f32 a, b; setp.ne.u32 q, %2, 0; mov.b32 a, %0; mov.b32 b, %1;"
                         " selp.f32 a, a, b, q; mov.b32 %0, a;}" : "+r"(v[c]) : "r"(v[n]), "r"(z));
        if (OP == SHF) asm volatile("shf.r.wrap.b32 %0, %0, %1, %2;" : "+r"(v[c]) : "r"(v[n]), "r"(k));
        if (OP == IMAD) asm volatile("mad.lo.u32 %0, %0, %1, %2;" : "+r"(v[c]) : "r"(k), "r"(v[n]));
        if (OP == LOP3) asm volatile("xor.b32 %0, %0, %1;" : "+r"(v[c]) : "r"(v[n]));
        if (OP == IMNMX) asm volatile("min.u32 %0, %0, %1;" : "+r"(v[c]) : "r"(v[n]));
        if (OP == PRMT) asm volatile("prmt.b32 %0, %0, %1, %2;" : "+r"(v[c]) : "r"(v[n]), "r"(k));
    }
}

template <int A, int B>
__global__ void __launch_bounds__(256) kern(uint32_t *out, uint32_t seed, int iters) {
    uint32_t a[CH], b[CH];
#pragma unroll
    for (int c = 0; c < CH; ++c) {
        a[c] = seed * (threadIdx.x + 1) + c;
        b[c] = seed ^ (c * 0x9E3779B9u) ^ threadIdx.x;
    }
    uint32_t k = (seed & 7) | 1, z = threadIdx.x & 1;
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int r = 0; r < REP; ++r) {
            step<A>(a, k, z);
            step<B>(b, k, z);
        }
    }
    uint32_t acc = 0;
#pragma unroll
    for (int c = 0; c < CH; ++c) acc ^= a[c] ^ b[c];
    if (acc == 0x12345678u) out[0] = acc;
}

template <int A, int B>
static void run(int sms, double f, uint32_t *out, bool &first) {
    const int blocks = sms * 8, threads = 256, iters = 200;
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    kern<A, B><<<blocks, threads>>>(out, 7, 4);
    cudaEventRecord(e0);
    kern<A, B><<<blocks, threads>>>(out, 7, iters);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms = 0;
    cudaEventElapsedTime(&ms, e0, e1);
    double warps = (double)blocks * threads / 32;
    double steps = (double)iters * REP * CH;  // per warp, each of A and B
    double cyc = ms * 1e-3 * f * sms * 4 / (warps * steps);  // SMSP-cycles per warp per (A + B) step
    printf("%s\"%s%s%s\": %.3f", first ? "" : ", ", NAMES[A], B == NONE ? "" : "+", B == NONE ? "" : NAMES[B], cyc);
    first = false;
}

int main() {
    int dev = 0, sms = 0, khz = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    cudaDeviceGetAttribute(&khz, cudaDevAttrClockRate, dev);
    double f = khz * 1e3;
    uint32_t *out;
    cudaMalloc(&out, 4);
    bool first = true;
    printf("{\"unit\": \"SMSP-cycles per warp per (A step + B step)\", \"rates\": {");
    run<SEL, NONE>(sms, f, out, first);
    run<FSEL, NONE>(sms, f, out, first);
    run<SHF, NONE>(sms, f, out, first);
    run<IMAD, NONE>(sms, f, out, first);
    run<LOP3, NONE>(sms, f, out, first);
    run<IMNMX, NONE>(sms, f, out, first);
    run<PRMT, NONE>(sms, f, out, first);
    run<FSEL, SHF>(sms, f, out, first);
    run<FSEL, IMAD>(sms, f, out, first);
    run<SEL, SHF>(sms, f, out, first);
    run<SEL, IMAD>(sms, f, out, first);
    run<FSEL, SEL>(sms, f, out, first);
    printf("}, \"cuda\": \"%s\"}\n", cudaGetErrorString(cudaGetLastError()));
    return 0;
}
