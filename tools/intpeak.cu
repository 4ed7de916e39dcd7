// intpeak.cu -- B200 integer-pipe microbenchmark ("C11").
//
// Measures sustained warp-instructions / clock / SM for the SASS the GCD pass
// is made of (IADD3, IADD3.X carry chains, SHF.R.W funnel shifts, IMAD,
// IMAD.WIDE, SEL, ISETP, LOP3) and for the pass's own limb step, with 8
// independent chains per thread and full occupancy, so the result is the
// pipe throughput, not latency.  Prints one JSON object.
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o build/intpeak tools/intpeak.cu && build/intpeak
#include <cstdio>
#include <cstdlib>
#include <cstdint>
#include <cuda_runtime.h>

#define REP 64
#define CHAINS 8

template <int OP>
__global__ void __launch_bounds__(256) kern(uint32_t *out, uint32_t seed, int iters) {
    uint32_t a[CHAINS], b[CHAINS];
#pragma unroll
    for (int c = 0; c < CHAINS; ++c) {
        a[c] = seed * (threadIdx.x + 1) + c;
        b[c] = seed ^ (c * 0x9E3779B9u);
    }
    uint32_t sh = seed & 7;
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int r = 0; r < REP; ++r) {
#pragma unroll
            for (int c = 0; c < CHAINS; ++c) {
                if (OP == 0) asm volatile("add.u32 %0, %0, %1;" : "+r"(a[c]) : "r"(b[c]));                 // IADD3
                if (OP == 1) asm volatile("shf.r.wrap.b32 %0, %0, %1, %2;" : "+r"(a[c]) : "r"(b[c]), "r"(sh));  // SHF
                if (OP == 2) asm volatile("mad.lo.u32 %0, %0, %1, %1;" : "+r"(a[c]) : "r"(b[c]));          // IMAD
                if (OP == 3) asm volatile("xor.b32 %0, %0, %1;" : "+r"(a[c]) : "r"(b[c]));                 // LOP3
                if (OP == 4) {                                                                          // IMAD.WIDE
                    uint64_t p;
                    asm volatile("mul.wide.u32 %0, %1, %2;" : "=l"(p) : "r"(a[c]), "r"(b[c]));
                    a[c] = (uint32_t)p ^ (uint32_t)(p >> 32);
                }
                if (OP == 7) {  // issue-rate probe: one ALU (SHF) + one FMA (IMAD) op per chain step
                    asm volatile("shf.l.wrap.b32 %0, %0, %1, %2;" : "+r"(a[c]) : "r"(b[c]), "r"(sh));
                    asm volatile("mad.lo.u32 %0, %0, %1, %2;" : "+r"(b[c]) : "r"(a[c]), "r"(sh));
                }
                if (OP == 8) {  // FFMA alone (fmaheavy + fmalite)
                    asm volatile("fma.rn.f32 %0, %0, %1, %1;" : "+f"(*(float *)&a[c]) : "f"(*(float *)&b[c]));
                }
                if (OP == 9) {  // SHF (alu) + FFMA
                    asm volatile("shf.l.wrap.b32 %0, %0, %1, %2;" : "+r"(a[c]) : "r"(b[c]), "r"(sh));
                    asm volatile("fma.rn.f32 %0, %0, %1, %1;" : "+f"(*(float *)&b[c]) : "f"(*(float *)&a[c]));
                }
                if (OP == 10) {  // SHF (alu) + DFMA (fp64)
                    double d = __hiloint2double(a[c], b[c]);
                    asm volatile("shf.l.wrap.b32 %0, %0, %1, %2;" : "+r"(a[c]) : "r"(b[c]), "r"(sh));
                    asm volatile("fma.rn.f64 %0, %0, %0, %0;" : "+d"(d));
                    b[c] ^= __double2loint(d);
                }
                if (OP == 11) {  // SHF (alu) + FSEL-style select on the fp32 path (fmnmx)
                    asm volatile("shf.l.wrap.b32 %0, %0, %1, %2;" : "+r"(a[c]) : "r"(b[c]), "r"(sh));
                    asm volatile("min.f32 %0, %0, %1;" : "+f"(*(float *)&b[c]) : "f"(*(float *)&a[c]));
                }
                if (OP == 5) asm volatile("{.reg .pred p; setp.lt.u32 p, %0, %1; selp.b32 %0, %0, %1, p;}" : "+r"(a[c]) : "r"(b[c]));  // ISETP+SEL
            }
        }
        if (OP == 6) {  // carry chains: 8 chains of REP add.cc/addc each
#pragma unroll
            for (int c = 0; c < CHAINS; ++c) {
                asm volatile("add.cc.u32 %0, %0, %1;" : "+r"(a[c]) : "r"(b[c]));
#pragma unroll
                for (int r = 1; r < REP; ++r) asm volatile("addc.cc.u32 %0, %0, %1;" : "+r"(a[(c + r) % CHAINS]) : "r"(b[c]));
            }
        }
    }
    uint32_t acc = 0;
#pragma unroll
    for (int c = 0; c < CHAINS; ++c) acc ^= a[c];
    if (acc == 0x12345678u) out[0] = acc;
}

// The GCD pass limb step, W-word operands in registers: X <- rshift(X - alpha*Y)
// FORM 0: as generated (IMAD.WIDE, IADD3, IMAD.X, IADD3.X, SHF)
// FORM 1: product split in two subtract chains (IMAD, IMAD.HI, IADD3.X, IADD3.X, SHF)
// FORM 2: FORM 0 with the funnel shift done on the FMA pipe (IMAD + IMAD.HI)
template <int W, int FORM>
__global__ void __launch_bounds__(128) limbk(uint32_t *out, uint32_t seed, int iters) {
    uint32_t X[W], Y[W];
    const uint32_t *src = out + 64 + (blockIdx.x * 128 + threadIdx.x) % 1024;  // opaque operands (no rematerialisation)
#pragma unroll
    for (int k = 0; k < W; ++k) {
        X[k] = src[k * 1024] * (threadIdx.x + 3);
        Y[k] = src[k * 1024 + 7] ^ seed;
    }
    uint32_t alpha = (seed + threadIdx.x) | 1, r = (seed + threadIdx.x) & 7;
    uint32_t m = 1u << (32 - (r + 1));
    for (int it = 0; it < iters; ++it) {
        if (FORM == 1) {
            uint32_t z[W];
            asm volatile("sub.cc.u32 %0, %1, %2;" : "=r"(z[0]) : "r"(X[0]), "r"(alpha * Y[0]));
#pragma unroll
            for (int k = 1; k < W; ++k)
                asm volatile("subc.cc.u32 %0, %1, %2;" : "=r"(z[k]) : "r"(X[k]), "r"(alpha * Y[k]));
            asm volatile("sub.cc.u32 %0, %0, %1;" : "+r"(z[1]) : "r"(__umulhi(alpha, Y[0])));
#pragma unroll
            for (int k = 2; k < W; ++k)
                asm volatile("subc.cc.u32 %0, %0, %1;" : "+r"(z[k]) : "r"(__umulhi(alpha, Y[k - 1])));
#pragma unroll
            for (int k = 0; k < W - 1; ++k) X[k] = __funnelshift_r(z[k], z[k + 1], r);
            X[W - 1] = z[W - 1] >> r;
        } else {
            uint32_t zp, z, lo, hi;
            asm volatile("{.reg .u64 p; mul.wide.u32 p, %2, %3; mov.b64 {%0, %1}, p;}" : "=r"(lo), "=r"(hi) : "r"(alpha), "r"(Y[0]));
            asm volatile("sub.cc.u32 %0, %1, %2;" : "=r"(zp) : "r"(X[0]), "r"(lo));
#pragma unroll
            for (int k = 1; k < W; ++k) {
                asm volatile("{.reg .u64 p, q; mov.b64 q, {%2, 0}; mad.wide.u32 p, %3, %4, q; mov.b64 {%0, %1}, p;}"
                             : "=r"(lo), "=r"(hi) : "r"(hi), "r"(alpha), "r"(Y[k]));
                asm volatile("subc.cc.u32 %0, %1, %2;" : "=r"(z) : "r"(X[k]), "r"(lo));
                if (FORM == 2) X[k - 1] = __umulhi(zp, m) + z * m;
                else X[k - 1] = __funnelshift_r(zp, z, r);
                zp = z;
            }
            X[W - 1] = __funnelshift_r(zp, 0u, r);
        }
        alpha += X[W - 1] & 2;
    }
    uint32_t acc = 0;
#pragma unroll
    for (int k = 0; k < W; ++k) acc ^= X[k];
    if (acc == 0x12345678u) out[0] = acc;
}

template <class F>
static double time_ms(F f) {
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    f();
    cudaDeviceSynchronize();
    cudaEventRecord(e0);
    f();
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    return ms;
}

int main(int argc, char **argv) {
    int dev = 0, sms = 0, clk_khz = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    cudaDeviceGetAttribute(&clk_khz, cudaDevAttrClockRate, dev);
    uint32_t *out;
    cudaMalloc(&out, (64 + 64 * 1024 + 64) * 4);
    cudaMemset(out, 0x5a, (64 + 64 * 1024 + 64) * 4);
    const int iters = 2000;
    if (argc > 2) {  // profiling mode: intpeak FORM WARPS_PER_SM -- one limbk launch
        int form = atoi(argv[1]), w = atoi(argv[2]);
        int blocks = sms * w / 4;
        if (form == 0) limbk<32, 0><<<blocks, 128>>>(out, 7, 200);
        if (form == 1) limbk<32, 1><<<blocks, 128>>>(out, 7, 200);
        if (form == 2) limbk<32, 2><<<blocks, 128>>>(out, 7, 200);
        cudaDeviceSynchronize();
        printf("%s\n", cudaGetErrorString(cudaGetLastError()));
        return 0;
    }
    const char *names[] = {"IADD3", "SHF.R.W", "IMAD", "LOP3", "IMAD.WIDE+LOP3", "ISETP+SEL", "IADD3.X-carry-chains",
                           "SHF+IMAD(alu+fma issue probe)", "FFMA", "SHF+FFMA", "SHF+DFMA+LOP3", "SHF+FMNMX"};
    printf("{\"sms\": %d, \"clock_khz_attr\": %d, \"ops\": {", sms, clk_khz);
    double f = clk_khz * 1e3;  // nominal max clock; the bench records the real one
    for (int op = 0; op < 12; ++op) {
        int blocks = sms * 8, threads = 256;
        double ms = 0;
        switch (op) {
            case 0: ms = time_ms([&] { kern<0><<<blocks, threads>>>(out, 7, iters); }); break;
            case 1: ms = time_ms([&] { kern<1><<<blocks, threads>>>(out, 7, iters); }); break;
            case 2: ms = time_ms([&] { kern<2><<<blocks, threads>>>(out, 7, iters); }); break;
            case 3: ms = time_ms([&] { kern<3><<<blocks, threads>>>(out, 7, iters); }); break;
            case 4: ms = time_ms([&] { kern<4><<<blocks, threads>>>(out, 7, iters); }); break;
            case 5: ms = time_ms([&] { kern<5><<<blocks, threads>>>(out, 7, iters); }); break;
            case 6: ms = time_ms([&] { kern<6><<<blocks, threads>>>(out, 7, iters); }); break;
            case 7: ms = time_ms([&] { kern<7><<<blocks, threads>>>(out, 7, iters); }); break;
            case 8: ms = time_ms([&] { kern<8><<<blocks, threads>>>(out, 7, iters); }); break;
            case 9: ms = time_ms([&] { kern<9><<<blocks, threads>>>(out, 7, iters); }); break;
            case 10: ms = time_ms([&] { kern<10><<<blocks, threads>>>(out, 7, iters); }); break;
            case 11: ms = time_ms([&] { kern<11><<<blocks, threads>>>(out, 7, iters); }); break;
        }
        double ninst = (double)blocks * (threads / 32) * iters * REP * CHAINS * (op == 10 ? 3 : (op == 4 || op == 5 || op == 7 || op == 9 || op == 11) ? 2 : 1);
        double per_clk_sm = ninst / (ms * 1e-3) / f / sms;
        printf("%s\"%s\": {\"ms\": %.3f, \"warp_inst_per_clk_per_sm_at_max_clock\": %.3f}", op ? ", " : "", names[op], ms,
               per_clk_sm);
    }
    // limb step at the pass's register footprint (W = 32): forms x warps per SM
    printf(", \"limb_step_W32\": {");
    const int wps[] = {8, 12, 16, 24, 32};
    for (int form = 0; form < 3; ++form) {
        for (int wi = 0; wi < 5; ++wi) {
            int blocks = sms * wps[wi] / 4, threads = 128;
            double ms = 0;
            if (form == 0) ms = time_ms([&] { limbk<32, 0><<<blocks, threads>>>(out, 7, iters * 4); });
            if (form == 1) ms = time_ms([&] { limbk<32, 1><<<blocks, threads>>>(out, 7, iters * 4); });
            if (form == 2) ms = time_ms([&] { limbk<32, 2><<<blocks, threads>>>(out, 7, iters * 4); });
            double limbs = (double)blocks * (threads / 32) * iters * 4 * 32;
            double per = limbs / (ms * 1e-3) / f / sms;
            printf("%s\"form%d_warps%d\": %.3f", (form || wi) ? ", " : "", form, wps[wi], 4.0 / per);
        }
    }
    printf("}");
    printf("}, \"cuda\": \"%s\"}\n", cudaGetErrorString(cudaGetLastError()));
    return 0;
}
