// limbmix.cu -- where does the fused limb step X <- rshift(X - alpha*Y) spend its cycles?
//
// Each thread keeps W = 32 words of X and Y in registers (as the all-pairs
// kernel does) and runs full 32-limb passes; variants drop parts of the limb:
//   A  full limb (the gen_duff.py body: mad.wide with carry addend, subc.cc borrow, shf.r.wrap funnel)
//   B  A without the funnel shift
//   C  A without the product (X - Y, borrow + funnel)
//   D  product chain only (IMAD.WIDE + carry add)
//   E  funnel shift only
//   F  borrow chain only
// Prints SMSP-cycles per limb (at the attribute clock) for 16 and 32 resident warps/SM.
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o build/limbmix tools/limbmix.cu && build/limbmix
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>

constexpr int W = 32;

template <int V>
__device__ __forceinline__ void pass(uint32_t (&X)[W], const uint32_t (&Y)[W], uint32_t a, uint32_t r) {
    uint32_t lo, hi = 0, z, zp = 0;
    if (V == 0 || V == 1 || V == 3) {
        asm volatile("{.reg .u64 p; mul.wide.u32 p, %2, %3; mov.b64 {%0, %1}, p;}" : "=r"(lo), "=r"(hi) : "r"(a), "r"(Y[0]));
        if (V == 3) X[0] = lo;
        else asm volatile("sub.cc.u32 %0, %1, %2;" : "=r"(zp) : "r"(X[0]), "r"(lo));
        if (V == 1) X[0] = zp;
#pragma unroll
        for (int k = 1; k < W; ++k) {
            asm volatile("{.reg .u64 p, q; mov.b64 q, {%2, 0}; mad.wide.u32 p, %3, %4, q; mov.b64 {%0, %1}, p;}"
                         : "=r"(lo), "=r"(hi) : "r"(hi), "r"(a), "r"(Y[k]));
            if (V == 3) {
                X[k] = lo;
                continue;
            }
            asm volatile("subc.cc.u32 %0, %1, %2;" : "=r"(z) : "r"(X[k]), "r"(lo));
            if (V == 0) X[k - 1] = __funnelshift_r(zp, z, r);
            else X[k] = z;
            zp = z;
        }
        if (V == 0) X[W - 1] = __funnelshift_r(zp, 0u, r);
        if (V == 3) X[W - 1] ^= hi;
    }
    if (V == 2) {
        asm volatile("sub.cc.u32 %0, %1, %2;" : "=r"(zp) : "r"(X[0]), "r"(Y[0]));
#pragma unroll
        for (int k = 1; k < W; ++k) {
            asm volatile("subc.cc.u32 %0, %1, %2;" : "=r"(z) : "r"(X[k]), "r"(Y[k]));
            X[k - 1] = __funnelshift_r(zp, z, r);
            zp = z;
        }
        X[W - 1] = __funnelshift_r(zp, 0u, r);
    }
    if (V == 4) {
#pragma unroll
        for (int k = 0; k < W - 1; ++k) X[k] = __funnelshift_r(X[k], X[k + 1], r);
        X[W - 1] = __funnelshift_r(X[W - 1], Y[0], r);
    }
    if (V == 6 || V == 7) {
        // two borrow chains per G-limb block: z = x - lo(aY) (chain 1), z -= hi(aY) one word up
        // (chain 2); borrows saved/restored between blocks; one IMAD.WIDE per limb, no carry add
        constexpr int G = V == 6 ? 4 : 8;
        uint32_t b1 = 0, b2 = 0, hprev = 0, zp = 0;
#pragma unroll
        for (int k0 = 0; k0 < W; k0 += G) {
            uint32_t lo[G], hi[G], z[G];
#pragma unroll
            for (int g = 0; g < G; ++g)
                asm volatile("{.reg .u64 p; mul.wide.u32 p, %2, %3; mov.b64 {%0, %1}, p;}" : "=r"(lo[g]), "=r"(hi[g]) : "r"(a), "r"(Y[k0 + g]));
            asm volatile("sub.cc.u32 %0, 0, %1;" : "=r"(z[0]) : "r"(b1));  // CF = (b1 != 0)
#pragma unroll
            for (int g = 0; g < G; ++g) asm volatile("subc.cc.u32 %0, %1, %2;" : "=r"(z[g]) : "r"(X[k0 + g]), "r"(lo[g]));
            asm volatile("subc.u32 %0, 0, 0;" : "=r"(b1));
            asm volatile("sub.cc.u32 %0, 0, %1;" : "=r"(b2) : "r"(b2));
            asm volatile("subc.cc.u32 %0, %0, %1;" : "+r"(z[0]) : "r"(hprev));
#pragma unroll
            for (int g = 1; g < G; ++g) asm volatile("subc.cc.u32 %0, %0, %1;" : "+r"(z[g]) : "r"(hi[g - 1]));
            asm volatile("subc.u32 %0, 0, 0;" : "=r"(b2));
            hprev = hi[G - 1];
#pragma unroll
            for (int g = 0; g < G; ++g) {
                if (k0 + g > 0) X[k0 + g - 1] = __funnelshift_r(zp, z[g], r);
                zp = z[g];
            }
        }
        X[W - 1] = __funnelshift_r(zp, 0u, r);
    }
    if (V == 8) {  // B then E: the product/borrow sweep, then a separate shift sweep
        pass<1>(X, Y, a, r);
        pass<4>(X, Y, a, r);
    }
    if (V == 5) {
        asm volatile("sub.cc.u32 %0, %0, %1;" : "+r"(X[0]) : "r"(Y[0]));
#pragma unroll
        for (int k = 1; k < W; ++k) asm volatile("subc.cc.u32 %0, %0, %1;" : "+r"(X[k]) : "r"(Y[k]));
    }
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
    cudaEventRecord(e0);
    kern<V><<<blocks, 128>>>(out, 7, iters);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    double limbs = (double)blocks * 4 * iters * W;  // warp-limbs
    return ms * 1e-3 * f * sms * 4 / limbs;          // SMSP-cycles per warp-limb
}

int main() {
    int sms = 0, clk_khz = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    cudaDeviceGetAttribute(&clk_khz, cudaDevAttrClockRate, 0);
    uint32_t *out;
    cudaMalloc(&out, (64 + 64 * 1024 + 64) * 4);
    cudaMemset(out, 0x5a, (64 + 64 * 1024 + 64) * 4);
    double f = clk_khz * 1e3;
    const char *names[] = {"A_full", "B_no_shift", "C_no_product", "D_product_only", "E_shift_only", "F_borrow_only",
                           "G_two_chains_G4", "H_two_chains_G8", "I_B_then_E"};
    printf("{\"unit\": \"SMSP-cycles per warp-limb\", \"variants\": {");
    for (int w : {16, 32}) {
        double c[9] = {run<0>(sms, f, out, w), run<1>(sms, f, out, w), run<2>(sms, f, out, w),
                       run<3>(sms, f, out, w), run<4>(sms, f, out, w), run<5>(sms, f, out, w),
                       run<6>(sms, f, out, w), run<7>(sms, f, out, w), run<8>(sms, f, out, w)};
        for (int v = 0; v < 9; ++v) printf("%s\"%s_w%d\": %.3f", (w == 16 && v == 0) ? "" : ", ", names[v], w, c[v]);
    }
    printf("}, \"cuda\": \"%s\"}\n", cudaGetErrorString(cudaGetLastError()));
    return 0;
}
