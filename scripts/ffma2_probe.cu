// ffma2_probe.cu -- design probe: FFMA vs packed FFMA2 (f32x2) throughput, and the rho=17 pair mix with
// the 16 MAC FMAs as 8 FFMA2 (not part of the product).
#include <cstdio>
#include <cuda_runtime.h>
typedef unsigned long long u64;
__device__ __forceinline__ u64 ffma2(u64 a, u64 b, u64 c) { u64 r; asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(r) : "l"(a), "l"(b), "l"(c)); return r; }
__device__ __forceinline__ u64 pk(float x, float y) { return (u64(__float_as_uint(y)) << 32) | __float_as_uint(x); }

__global__ void ffma1(float *out, int iters) {
    float acc[16]; float a = threadIdx.x * 1e-3f, b = 1.0001f;
    for (int j = 0; j < 16; ++j) acc[j] = j;
    for (int i = 0; i < iters; ++i)
#pragma unroll
        for (int j = 0; j < 16; ++j) acc[j] = fmaf(acc[j], b, a);
    float s = 0; for (int j = 0; j < 16; ++j) s += acc[j]; out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
__global__ void ffma2k(float *out, int iters) {
    u64 acc[16]; u64 a = pk(threadIdx.x * 1e-3f, 1e-4f), b = pk(1.0001f, 0.9999f);
    for (int j = 0; j < 16; ++j) acc[j] = pk(j, j + 1);
    for (int i = 0; i < iters; ++i)
#pragma unroll
        for (int j = 0; j < 16; ++j) acc[j] = ffma2(acc[j], b, a);
    float s = 0; for (int j = 0; j < 16; ++j) s += __uint_as_float(unsigned(acc[j])) + __uint_as_float(unsigned(acc[j] >> 32));
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
// pair mix: per unit: phase FFMA, sincos, 8 FFMA2 (= 16 FMA) into 4 packed accumulators x 2
__global__ void pairmix2(float *out, int iters) {
    const int U = 4;
    float sn[U], cs[U]; u64 acc[U][4]; u64 v01 = pk(0.3f, 0.2f), v23 = pk(-0.1f, 0.4f), v45 = pk(0.5f, -0.6f), v67 = pk(0.7f, 0.8f);
    for (int k = 0; k < U; ++k) { sn[k] = 0.1f * k + threadIdx.x * 1e-6f; cs[k] = 0.37f; for (int j = 0; j < 4; ++j) acc[k][j] = 0; }
    const float x = 0.731f;
    for (int i = 0; i < iters; ++i) {
#pragma unroll
        for (int k = 0; k < U; ++k) {
            float ph = fmaf(x, cs[k], sn[k]);
            __sincosf(ph, &sn[k], &cs[k]);
            u64 c2 = pk(cs[k], cs[k]), s2 = pk(sn[k], sn[k]);
            acc[k][0] = ffma2(v01, c2, acc[k][0]); acc[k][1] = ffma2(v23, c2, acc[k][1]);
            acc[k][2] = ffma2(v45, c2, acc[k][2]); acc[k][3] = ffma2(v67, c2, acc[k][3]);
            acc[k][0] = ffma2(v23, s2, acc[k][0]); acc[k][1] = ffma2(v01, s2, acc[k][1]);
            acc[k][2] = ffma2(v67, s2, acc[k][2]); acc[k][3] = ffma2(v45, s2, acc[k][3]);
        }
    }
    float s = 0;
    for (int k = 0; k < U; ++k) { s += sn[k] + cs[k]; for (int j = 0; j < 4; ++j) s += __uint_as_float(unsigned(acc[k][j])) + __uint_as_float(unsigned(acc[k][j] >> 32)); }
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
template <typename F> void time_it(const char *name, F launch, double work, const char *unit) {
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    launch(); cudaDeviceSynchronize(); cudaEventRecord(e0); launch(); cudaEventRecord(e1); cudaEventSynchronize(e1);
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    printf("%-34s %8.3f ms %10.3f %s  (%.2f per SM per clk @1965)\n", name, ms, work / (ms * 1e-3) / 1e12, unit, work / (ms * 1e-3) / 148 / 1.965e9);
}
int main() {
    float *out; cudaMalloc(&out, 148 * 64 * 1024 * 4);
    const int it = 8192, B = 148 * 8, T = 256;
    time_it("FFMA (16 chains)", [&] { ffma1<<<B, T>>>(out, it); }, double(B) * T * it * 16, "T FMA/s");
    time_it("FFMA2 (16 chains, 2 FMA each)", [&] { ffma2k<<<B, T>>>(out, it); }, double(B) * T * it * 32, "T FMA/s");
    time_it("pair mix: FFMA+sincos+8 FFMA2", [&] { pairmix2<<<B, T>>>(out, it / 4); }, double(B) * T * (it / 4) * 4, "T pairs/s");
    printf("status %s\n", cudaGetErrorString(cudaGetLastError()));
}
