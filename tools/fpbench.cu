// fpbench.cu -- FP32 vs packed FP32x2 throughput on B200 (sm_100a).
// Each thread runs 8 independent chains for N iterations; reports warp
// instructions / clk / SM and FP32 lane-ops / clk / SM.
#include <cuda_runtime.h>
#include <stdio.h>

typedef unsigned long long u64;

__device__ __forceinline__ u64 fma2(u64 a, u64 b, u64 c) {
    u64 r;
    asm volatile("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(r) : "l"(a), "l"(b), "l"(c));
    return r;
}
__device__ __forceinline__ u64 add2(u64 a, u64 b) {
    u64 r;
    asm volatile("add.rn.f32x2 %0, %1, %2;" : "=l"(r) : "l"(a), "l"(b));
    return r;
}
__device__ __forceinline__ u64 fma2s(u64 a, float b, u64 c) {  // scalar broadcast coefficient
    u64 r, bb;
    asm("mov.b64 %0, {%1, %1};" : "=l"(bb) : "f"(b));
    asm volatile("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(r) : "l"(a), "l"(bb), "l"(c));
    return r;
}

template <int MODE>
__global__ void kern(float* out, int n, float c0, float c1) {
    float f[16];
    u64 p[8], q[8];
    double d[8];
    for (int i = 0; i < 16; ++i) f[i] = threadIdx.x * 0.001f + i;
    for (int i = 0; i < 8; ++i) d[i] = threadIdx.x * 0.001 + i;
    for (int i = 0; i < 8; ++i) {
        p[i] = ((u64)__float_as_uint(f[i]) << 32) | __float_as_uint(f[i + 8]);
        q[i] = p[i] ^ 0x1234;
    }
    for (int it = 0; it < n; ++it) {
#pragma unroll
        for (int i = 0; i < 8; ++i) {
            if (MODE == 0) {  // scalar FFMA, coefficient in register
                f[i] = __fmaf_rn(f[i], c0, f[i + 8]);
                f[i + 8] = __fmaf_rn(f[i + 8], c1, f[i]);
            } else if (MODE == 1) {  // scalar FADD
                f[i] = __fadd_rn(f[i], f[(i + 3) & 15]);
                f[i + 8] = __fadd_rn(f[i + 8], f[(i + 5) & 15]);
            } else if (MODE == 2) {  // FFMA2, three 64-bit operands
                p[i] = fma2(p[i], q[i], p[(i + 1) & 7]);
            } else if (MODE == 3) {  // FFMA2 with a broadcast scalar coefficient
                p[i] = fma2s(q[i], c0, p[i]);
            } else if (MODE == 4) {  // FADD2
                p[i] = add2(p[i], q[(i + 3) & 7]);
            } else if (MODE == 5) {  // DFMA
                d[i] = __fma_rn(d[i], (double)c0, d[(i + 1) & 7]);
            } else if (MODE == 6) {  // DADD
                d[i] = __dadd_rn(d[i], d[(i + 3) & 7]);
            }
        }
    }
    float s = 0;
    for (int i = 0; i < 16; ++i) s += f[i];
    for (int i = 0; i < 8; ++i) s += __uint_as_float((unsigned)p[i]) + (float)d[i];
    if (s == 1.2345f) out[threadIdx.x] = s;
}

int main() {
    float* o;
    cudaMalloc(&o, 4096);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    int clk_khz;
    cudaDeviceGetAttribute(&clk_khz, cudaDevAttrClockRate, 0);
    const int n = 20000;
    const char* names[] = {"FFMA (scalar)", "FADD (scalar)", "FFMA2 (3x64-bit)", "FFMA2 (bcast scalar)", "FADD2", "DFMA", "DADD"};
    for (int mode = 0; mode < 7; ++mode)
        for (int warps : {4, 8, 16, 32}) {
            auto k = mode == 0 ? kern<0> : mode == 1 ? kern<1> : mode == 2 ? kern<2> : mode == 3 ? kern<3>
                   : mode == 4 ? kern<4> : mode == 5 ? kern<5> : kern<6>;
            k<<<148, warps * 32>>>(o, 100, 1.0001f, 0.9999f);
            cudaEventRecord(e0);
            k<<<148, warps * 32>>>(o, n, 1.0001f, 0.9999f);
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            float ms;
            cudaEventElapsedTime(&ms, e0, e1);
            const double instr_per_thread = (mode <= 1 ? 16.0 : 8.0) * n;  // DFMA/DADD: 8 chains
            const double warp_instr_sm = instr_per_thread * warps;
            const double cycles = ms * 1e-3 * clk_khz * 1e3;  // at the nominal max clock
            const double ops_per_instr = (mode <= 1 || mode >= 5) ? 32 : 64;
            printf("%-24s warps/SM %2d: %.2f warp-instr/clk/SM, %.1f fp32 ops/clk/SM (nominal clock)\n", names[mode], warps,
                   warp_instr_sm / cycles, warp_instr_sm * ops_per_instr / cycles);
        }
    return 0;
}
