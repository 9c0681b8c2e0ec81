// rho_forms_probe.cu -- design probe (not part of the product): which FMA encodings reach the FP32 pipe
// peak on sm_100 when mixed with sincos at the paper's rho = 17?  Forms:
//   0 scalar FFMA, 3 registers (acc = c * v + acc)        -- the paper's kernels
//   1 packed FFMA2, 3 distinct 64-bit registers           -- rho_kernel_x2 of the library
//   2 scalar FFMA, multiplier an immediate                 -- 2 register reads
//   3 packed FFMA2, multiplier a uniform (kernel-parameter) pair
//   4 packed FFMA2, multiplier = the addend's partner (a, a, c): 2 distinct 64-bit registers
// Prints TOps/s (2 per FMA + 2 per sincos) for rho = 17 and rho = 64.
#include <cstdio>
#include <cuda_runtime.h>
typedef unsigned long long u64;
__device__ __forceinline__ u64 ffma2(u64 a, u64 b, u64 c) { u64 r; asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(r) : "l"(a), "l"(b), "l"(c)); return r; }
__device__ __forceinline__ u64 pk(float x, float y) { u64 r; asm("mov.b64 %0, {%1, %2};" : "=l"(r) : "f"(x), "f"(y)); return r; }
__device__ __forceinline__ float2 up(u64 v) { float2 r; asm("mov.b64 {%0, %1}, %2;" : "=f"(r.x), "=f"(r.y) : "l"(v)); return r; }

template <int FORM, int RHO>
__global__ void __launch_bounds__(256) k(float *out, int iters, u64 ucoef) {
    constexpr int U = 4;   // unit pairs
    const int tid = blockIdx.x * blockDim.x + threadIdx.x;
    u64 sn[U], cs[U], acc[U][8];
    float c1 = 0.25f + 0.01f * (tid & 7);
    u64 coef = pk(c1, c1 + 0.01f);
    for (int k = 0; k < U; ++k) { sn[k] = pk(0.1f * k + 1e-6f * (tid & 1023), 0.2f); cs[k] = pk(0.37f, 0.41f + 0.01f * k); for (int j = 0; j < 8; ++j) acc[k][j] = 0; }
    const u64 x = pk(0.731f + 1e-7f * (tid & 255), 0.689f);
#pragma unroll 1
    for (int i = 0; i < iters; ++i) {
#pragma unroll
        for (int k = 0; k < U; ++k) {
            const float2 ph = up(ffma2(x, cs[k], sn[k]));
            float s0, c0, s1, c1_;
            __sincosf(ph.x, &s0, &c0);
            __sincosf(ph.y, &s1, &c1_);
            sn[k] = pk(s0, s1); cs[k] = pk(c0, c1_);
#pragma unroll
            for (int j = 0; j < RHO - 1; ++j) {
                const u64 v = (j & 1) ? sn[k] : cs[k];
                u64 &a = acc[k][j & 7];
                if (FORM == 1) a = ffma2(coef, v, a);
                else if (FORM == 3) a = ffma2(ucoef, v, a);
                else if (FORM == 4) a = ffma2(v, v, a);
                else {
                    float2 va = up(v), aa = up(a);
                    if (FORM == 0) { aa.x = fmaf(c1, va.x, aa.x); aa.y = fmaf(c1, va.y, aa.y); }
                    else { aa.x = fmaf(0.2734375f, va.x, aa.x); aa.y = fmaf(0.2734375f, va.y, aa.y); }
                    a = pk(aa.x, aa.y);
                }
            }
        }
    }
    float s = 0;
    for (int k = 0; k < U; ++k) { float2 a = up(sn[k]), b = up(cs[k]); s += a.x + a.y + b.x + b.y; for (int j = 0; j < 8; ++j) { float2 c = up(acc[k][j]); s += c.x + c.y; } }
    out[tid] = s;
}

template <int FORM, int RHO>
void run(float *d, int sms) {
    int per = 0; cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, k<FORM, RHO>, 256, 0);
    const int blocks = sms * per * 4, iters = 8192;
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    k<FORM, RHO><<<blocks, 256>>>(d, iters / 8, 0x3e8a00003e800000ull);
    float best = 1e30f;
    for (int r = 0; r < 3; ++r) {
        cudaEventRecord(a); k<FORM, RHO><<<blocks, 256>>>(d, iters, 0x3e8a00003e800000ull); cudaEventRecord(b);
        cudaEventSynchronize(b); float ms; cudaEventElapsedTime(&ms, a, b); if (ms < best) best = ms;
    }
    const double sincos = double(blocks) * 256 * 8 * iters;
    printf("form %d rho %2d: %6.1f TOps/s  (%d blocks/SM)\n", FORM, RHO, sincos * (2.0 * RHO + 2) / (best * 1e-3) / 1e12, per);
}

int main() {
    float *d; cudaMalloc(&d, 148 * 64 * 256 * 4 * 4);
    int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    run<0, 17>(d, sms); run<1, 17>(d, sms); run<2, 17>(d, sms); run<3, 17>(d, sms); run<4, 17>(d, sms);
    run<0, 64>(d, sms); run<1, 64>(d, sms); run<2, 64>(d, sms); run<3, 64>(d, sms); run<4, 64>(d, sms);
    return 0;
}
