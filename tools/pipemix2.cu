// pipemix2.cu -- which resource does IMAD.WIDE.U32 share on sm_100a?  (round-2 follow-up of pipemix.cu)
//
// pipemix.cu found SHF + IMAD.WIDE and IADD3.X + IMAD.WIDE serialise while SHF + IMAD
// overlap.  This probe pairs IMAD.WIDE (zero addend, as in the GCD pass) with every
// other opcode of the pass and of its per-iteration overhead, CH independent chains
// per op, full occupancy: rate = warp-instructions / clock / SM at the attribute clock.
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o build/pipemix2 tools/pipemix2.cu && build/pipemix2
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>

#define REP 32
#define CH 6

enum { NONE, WIDE, IMAD, IMADX, IADD3, IADD3CO, IADD3X2, SHF, SEL, ISETP, LOP3, IMADMOV, DFMA, NOPS };
static const char *NAMES[] = {"none", "IMAD.WIDE", "IMAD", "WIDE+IADD3+IMAD.X", "IADD3", "ADD64(IADD3co+IADD3.X)", "ADD3W(IADD3 2co+IADD3.X 2ci)",
                              "SHF", "SEL", "ISETP", "LOP3", "IMAD.MOV", "DFMA"};

template <int OP>
__device__ __forceinline__ void step(uint32_t (&v)[CH], uint32_t (&u)[CH], double (&d)[CH], uint32_t k, uint32_t z) {
#pragma unroll
    for (int c = 0; c < CH; ++c) {
        const int n = (c + 1) % CH;
        if (OP == WIDE) {  // IMAD.WIDE.U32 with RZ addend (the pass's product)
            asm volatile("{.reg .u64 p; mul.wide.u32 p, %2, %3; mov.b64 {%0, %1}, p;}" : "=r"(v[c]), "=r"(u[c]) : "r"(v[n]), "r"(u[n]));
        }
        if (OP == IMAD) asm volatile("mad.lo.u32 %0, %0, %1, %2;" : "+r"(v[c]) : "r"(k), "r"(v[n]));
        if (OP == IMADX)  // the split form's product step: IMAD.WIDE + IADD3 (carry-out) + IMAD.X
            asm volatile("{.reg .u64 p, q; mov.b64 q, {%1, 0}; mad.wide.u32 p, %2, %3, q; mov.b64 {%0, %1}, p;}"
                         : "=r"(v[c]), "+r"(u[c]) : "r"(v[n]), "r"(k));
        if (OP == IADD3) asm volatile("add.u32 %0, %0, %1;" : "+r"(v[c]) : "r"(v[n]));
        if (OP == IADD3CO)  // 64-bit add: IADD3 (carry-out) + IADD3.X (carry-in)
            asm volatile("{add.cc.u32 %0, %0, %2; addc.u32 %1, %1, %3;}" : "+r"(v[c]), "+r"(u[c]) : "r"(v[n]), "r"(u[n]));
        if (OP == IADD3X2) {  // 3-input 64-bit add: IADD3 (2 carry-out) + IADD3.X (2 carry-in)
            asm volatile("{.reg .u64 a, b, s; mov.b64 a, {%0, %1}; cvt.u64.u32 b, %2; add.u64 s, a, b; cvt.u64.u32 b, %3;"
                         " add.u64 s, s, b; mov.b64 {%0, %1}, s;}" : "+r"(v[c]), "+r"(u[c]) : "r"(v[n]), "r"(u[n]));
        }
        if (OP == SHF) asm volatile("shf.r.wrap.b32 %0, %0, %1, %2;" : "+r"(v[c]) : "r"(v[n]), "r"(k));
        if (OP == SEL) asm volatile("{.reg .pred q; setp.ne.u32 q, %2, 0; selp.b32 %0, %0, %1, q;}" : "+r"(v[c]) : "r"(v[n]), "r"(z));
        if (OP == ISETP) asm volatile("{.reg .pred q; setp.lt.u32 q, %0, %1; selp.u32 %0, 1, 0, q;}" : "+r"(v[c]) : "r"(v[n]));
        if (OP == LOP3) asm volatile("xor.b32 %0, %0, %1;" : "+r"(v[c]) : "r"(v[n]));
        if (OP == IMADMOV) asm volatile("mov.b32 %0, %1;" : "=r"(v[c]) : "r"(u[n]));
        if (OP == DFMA) asm volatile("fma.rn.f64 %0, %0, %1, %1;" : "+d"(d[c]) : "d"(d[n]));
    }
}

template <int A, int B>
__global__ void __launch_bounds__(256) kern(uint32_t *out, uint32_t seed, int iters) {
    uint32_t a[CH], b[CH], ua[CH], ub[CH];
    double da[CH], db[CH];
#pragma unroll
    for (int c = 0; c < CH; ++c) {
        a[c] = seed * (threadIdx.x + 1) + c;
        b[c] = seed ^ (c * 0x9E3779B9u) ^ threadIdx.x;
        ua[c] = a[c] * 3u;
        ub[c] = b[c] * 5u;
        da[c] = (double)a[c] * 1e-9;
        db[c] = (double)b[c] * 1e-9;
    }
    uint32_t k = (seed & 7) | 1, z = threadIdx.x & 1;
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int r = 0; r < REP; ++r) {
            step<A>(a, ua, da, k, z);
            step<B>(b, ub, db, k, z);
        }
    }
    uint32_t acc = 0;
#pragma unroll
    for (int c = 0; c < CH; ++c) acc ^= a[c] ^ b[c] ^ ua[c] ^ ub[c] ^ (uint32_t)(long long)(da[c] + db[c]);
    if (acc == 0x12345678u) out[0] = acc;
}

// SASS instructions per chain step of op X (counted here by hand from cuobjdump; IADD3CO = 3,
// IMADX = 2, IADD3X2 = 2 (+1 IMAD.MOV), WIDE = 1); the rate below counts PTX-level steps.
template <int A, int B>
static void run(int sms, double f, uint32_t *out, bool &first) {
    const int blocks = sms * 8, threads = 256, iters = 200;
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    kern<A, B><<<blocks, threads>>>(out, 7, iters);
    cudaDeviceSynchronize();
    float best = 1e30f;
    for (int rep = 0; rep < 3; ++rep) {
        cudaEventRecord(e0);
        kern<A, B><<<blocks, threads>>>(out, 7, iters);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms;
        cudaEventElapsedTime(&ms, e0, e1);
        if (ms < best) best = ms;
    }
    // SMSP-cycles per (step of A + step of B) per warp
    double steps = (double)blocks * (threads / 32) * iters * REP * CH;
    double cyc = best * 1e-3 * f * sms * 4 / steps;
    printf("%s\"%s%s%s\": %.3f", first ? "" : ", ", NAMES[A], B == NONE ? "" : "+", B == NONE ? "" : NAMES[B], cyc);
    first = false;
}

int main() {
    int sms = 0, clk_khz = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    cudaDeviceGetAttribute(&clk_khz, cudaDevAttrClockRate, 0);
    uint32_t *out;
    cudaMalloc(&out, 64);
    double f = clk_khz * 1e3;
    bool first = true;
    printf("{\"unit\": \"SMSP-cycles per warp per (A step + B step)\", \"rates\": {");
    run<WIDE, NONE>(sms, f, out, first);
    run<IMAD, NONE>(sms, f, out, first);
    run<IMADX, NONE>(sms, f, out, first);
    run<IADD3, NONE>(sms, f, out, first);
    run<IADD3CO, NONE>(sms, f, out, first);
    run<IADD3X2, NONE>(sms, f, out, first);
    run<SHF, NONE>(sms, f, out, first);
    run<SEL, NONE>(sms, f, out, first);
    run<ISETP, NONE>(sms, f, out, first);
    run<LOP3, NONE>(sms, f, out, first);
    run<DFMA, NONE>(sms, f, out, first);
    run<WIDE, IMAD>(sms, f, out, first);
    run<WIDE, IMADX>(sms, f, out, first);
    run<WIDE, IADD3>(sms, f, out, first);
    run<WIDE, IADD3CO>(sms, f, out, first);
    run<WIDE, IADD3X2>(sms, f, out, first);
    run<WIDE, SHF>(sms, f, out, first);
    run<WIDE, SEL>(sms, f, out, first);
    run<WIDE, ISETP>(sms, f, out, first);
    run<WIDE, LOP3>(sms, f, out, first);
    run<WIDE, DFMA>(sms, f, out, first);
    run<SHF, IMADX>(sms, f, out, first);
    run<SHF, IADD3X2>(sms, f, out, first);
    run<SHF, SEL>(sms, f, out, first);
    run<SHF, ISETP>(sms, f, out, first);
    run<SHF, DFMA>(sms, f, out, first);
    run<IADD3X2, IMADX>(sms, f, out, first);
    run<IADD3CO, SHF>(sms, f, out, first);
    run<IADD3X2, IMAD>(sms, f, out, first);
    run<IADD3CO, IMAD>(sms, f, out, first);
    run<SHF, IMAD>(sms, f, out, first);
    printf("}, \"cuda\": \"%s\"}\n", cudaGetErrorString(cudaGetLastError()));
    return 0;
}
