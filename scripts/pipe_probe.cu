// pipe_probe.cu -- throughput of the instructions in the gridder's inner loop, alone and in pairs, to
// find which pipes they share: MUFU.SIN/COS (sincos), F2FP.F16.F32.PACK_AB (f32 -> f16x2), FHFMA
// (f16*f16+f32), FFMA2, HMMA.16816.  Each kernel runs independent chains per thread (ILP 8), 32 warps/SM.
// Prints warp-instructions per clock per SM for each instruction class in the mix.
#include <cstdio>
#include <cstdint>
#include <cuda_fp16.h>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t f2fp(float a, float b) {
    uint32_t r;
    asm volatile("cvt.rn.f16x2.f32 %0, %1, %2;" : "=r"(r) : "f"(a), "f"(b));
    return r;
}
__device__ __forceinline__ float fhfma(uint32_t h2, float c) {
    float d;
    asm volatile("{\n.reg .f16 a, b, m;\nmov.b32 {a, b}, %1;\nmov.b16 m, 0xBC00;\nfma.rn.f32.f16 %0, a, m, %2;\n}"
                 : "=f"(d) : "r"(h2), "f"(c));
    return d;
}
__device__ __forceinline__ float msin(float x) {
    float r;
    asm volatile("sin.approx.f32 %0, %1;" : "=f"(r) : "f"(x));
    return r;
}
__device__ __forceinline__ void hmma(float (&d)[4], uint32_t a0, uint32_t a1, uint32_t a2, uint32_t a3, uint32_t b0, uint32_t b1) {
    asm volatile("mma.sync.aligned.m16n8k16.row.col.f32.f16.f16.f32 {%0,%1,%2,%3},{%4,%5,%6,%7},{%8,%9},{%0,%1,%2,%3};"
                 : "+f"(d[0]), "+f"(d[1]), "+f"(d[2]), "+f"(d[3]) : "r"(a0), "r"(a1), "r"(a2), "r"(a3), "r"(b0), "r"(b1));
}

// MIX bits: 1 = sin (MUFU, 8 per iteration), 2 = f2fp (8), 4 = fhfma (8), 8 = hmma (2)
template <int MIX>
__global__ void mix(float *out, int iters) {
    float x[8];
    uint32_t h[8];
    float acc[2][4] = {};
    for (int i = 0; i < 8; ++i) { x[i] = threadIdx.x * 1e-3f + i; h[i] = 0x3c003c00u + i; }
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int i = 0; i < 8; ++i) {
            if (MIX & 1) x[i] = msin(x[i]);
            if (MIX & 2) h[i] = f2fp(x[i], __uint_as_float(h[i]));
            if (MIX & 4) x[i] = fhfma(h[i], x[i]);
        }
        if (MIX & 8) {
            hmma(acc[0], h[0], h[1], h[2], h[3], h[4], h[5]);
            hmma(acc[1], h[4], h[5], h[6], h[7], h[0], h[1]);
        }
    }
    float s = 0;
    for (int i = 0; i < 8; ++i) s += x[i] + __uint_as_float(h[i]);
    s += acc[0][0] + acc[1][1];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

template <int MIX>
void run(const char *name, float *out) {
    const int iters = 4096, blocks = 148 * 4, threads = 256;  // 32 warps / SM
    mix<MIX><<<blocks, threads>>>(out, 16);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0); cudaEventCreate(&e1);
    cudaEventRecord(e0);
    mix<MIX><<<blocks, threads>>>(out, iters);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    const double warp_iters = double(blocks) * (threads / 32) * iters;
    const double clk = ms * 1e-3 * 1.965e9 * 148;  // SM-clocks
    printf("%-28s per SM per clk:", name);
    if (MIX & 1) printf("  MUFU %.3f", 8 * warp_iters / clk);
    if (MIX & 2) printf("  F2FP %.3f", 8 * warp_iters / clk);
    if (MIX & 4) printf("  FHFMA %.3f", 8 * warp_iters / clk);
    if (MIX & 8) printf("  HMMA %.3f", 2 * warp_iters / clk);
    printf("  (warp-instr)  %s\n", cudaGetErrorString(cudaGetLastError()));
}

int main() {
    float *out; cudaMalloc(&out, 148 * 4 * 256 * 4);
    run<1>("MUFU.SIN", out);
    run<2>("F2FP", out);
    run<4>("FHFMA", out);
    run<8>("HMMA", out);
    run<1 | 2>("MUFU + F2FP", out);
    run<1 | 4>("MUFU + FHFMA", out);
    run<2 | 4>("F2FP + FHFMA", out);
    run<1 | 8>("MUFU + HMMA", out);
    run<2 | 8>("F2FP + HMMA", out);
    run<1 | 2 | 4 | 8>("all", out);
    return 0;
}
