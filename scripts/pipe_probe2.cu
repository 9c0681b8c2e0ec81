// pipe_probe2.cu -- do FFMA2 / FMUL2, PRMT and HMMA.16816 overlap on sm_100?  Independent chains (ILP 8 per
// class), 32 warps/SM; prints warp-instructions per clock per SM of each class, alone and mixed.
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>
typedef unsigned long long f2p;
__device__ __forceinline__ f2p fma2(f2p a, f2p b, f2p c) { f2p r; asm volatile("fma.rn.f32x2 %0,%1,%2,%3;" : "=l"(r) : "l"(a), "l"(b), "l"(c)); return r; }
__device__ __forceinline__ uint32_t prmt(uint32_t a, uint32_t b) { uint32_t r; asm volatile("prmt.b32 %0, %1, %2, 0x6521;" : "=r"(r) : "r"(a), "r"(b)); return r; }
__device__ __forceinline__ float ffma(float a, float b, float c) { float r; asm volatile("fma.rn.f32 %0,%1,%2,%3;" : "=f"(r) : "f"(a), "f"(b), "f"(c)); return r; }
__device__ __forceinline__ void hmma(float (&d)[4], uint32_t a0, uint32_t a1, uint32_t a2, uint32_t a3, uint32_t b0, uint32_t b1) {
    asm volatile("mma.sync.aligned.m16n8k16.row.col.f32.f16.f16.f32 {%0,%1,%2,%3},{%4,%5,%6,%7},{%8,%9},{%0,%1,%2,%3};"
                 : "+f"(d[0]), "+f"(d[1]), "+f"(d[2]), "+f"(d[3]) : "r"(a0), "r"(a1), "r"(a2), "r"(a3), "r"(b0), "r"(b1));
}
// MIX bits: 1 = FFMA2 (8 / iter), 2 = PRMT (8), 4 = HMMA (2 independent), 8 = scalar FFMA (8)
template <int MIX, int NF, int NP, int NH>
__global__ void mix(float *out, int iters) {
    f2p x[8]; uint32_t p[8]; float f[8];
    float acc[4][4] = {};
    for (int i = 0; i < 8; ++i) { x[i] = 0x3f8000003f800000ull + threadIdx.x + i; p[i] = 0x3c003c00u + i * 7 + threadIdx.x; f[i] = i * 0.1f; }
    const f2p m = 0x3f7fffff3f7fffffull, c = 0x3c0000003c000000ull;
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int i = 0; i < 8; ++i) {
            if ((MIX & 1) && i < NF) x[i] = fma2(x[i], m, c);
            if ((MIX & 2) && i < NP) p[i] = prmt(p[i], p[(i + 1) & 7]);
            if (MIX & 8) f[i] = ffma(f[i], 0.999f, 0.001f);
        }
        if (MIX & 4) {
#pragma unroll
            for (int h = 0; h < NH; ++h) hmma(acc[h], p[0], p[1], p[2], p[3], p[4], p[5]);
        }
    }
    float s = 0;
    for (int i = 0; i < 8; ++i) s += __uint_as_float(uint32_t(x[i])) + __uint_as_float(p[i]) + f[i];
    for (int h = 0; h < 4; ++h) s += acc[h][0];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
template <int MIX, int NF = 8, int NP = 8, int NH = 2>
void run(const char *name, float *out) {
    const int iters = 4096, blocks = 148 * 4, threads = 256;
    mix<MIX, NF, NP, NH><<<blocks, threads>>>(out, 16);
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    cudaEventRecord(e0); mix<MIX, NF, NP, NH><<<blocks, threads>>>(out, iters); cudaEventRecord(e1); cudaEventSynchronize(e1);
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    const double wi = double(blocks) * (threads / 32) * iters, clk = ms * 1e-3 * 1.965e9 * 148;
    printf("%-34s", name);
    if (MIX & 1) printf("  FFMA2 %.3f", NF * wi / clk);
    if (MIX & 2) printf("  PRMT %.3f", NP * wi / clk);
    if (MIX & 4) printf("  HMMA %.3f", NH * wi / clk);
    if (MIX & 8) printf("  FFMA %.3f", 8 * wi / clk);
    printf("   (warp-instr / clk / SM)  %.3f ms\n", ms);
}
int main() {
    float *out; cudaMalloc(&out, 148 * 4 * 256 * 4);
    run<1>("FFMA2", out);
    run<8>("FFMA", out);
    run<2>("PRMT", out);
    run<4>("HMMA x2", out);
    run<4, 8, 8, 4>("HMMA x4", out);
    run<1 | 2>("FFMA2 + PRMT", out);
    run<1 | 4>("FFMA2 8 + HMMA 2", out);
    run<1 | 4, 4, 8, 2>("FFMA2 4 + HMMA 2", out);
    run<2 | 4>("PRMT 8 + HMMA 2", out);
    run<1 | 2 | 4>("FFMA2 8 + PRMT 8 + HMMA 2", out);
    run<1 | 2 | 4, 8, 4, 1>("FFMA2 8 + PRMT 4 + HMMA 1", out);
    run<8 | 4>("FFMA 8 + HMMA 2", out);
    return 0;
}
