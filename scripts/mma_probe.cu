// mma_probe.cu -- throughput of warp-level mma.sync shapes on the local GPU (design probe for the
// tensor-core gridder/degridder; not part of the product).  nvcc -gencode arch=compute_100a,code=sm_100a
#include <cstdio>
#include <cuda_fp16.h>
#include <cuda_runtime.h>

template <int CHAINS>
__global__ void hmma_f16(float *out, int iters) {
    unsigned a[4], b[2];
    float c[CHAINS][4];
    for (int i = 0; i < 4; ++i) a[i] = 0x3c003c00u ^ (threadIdx.x * 7 + i);
    for (int i = 0; i < 2; ++i) b[i] = 0x3c003c00u ^ (threadIdx.x * 3 + i);
    for (int k = 0; k < CHAINS; ++k)
        for (int i = 0; i < 4; ++i) c[k][i] = 0.f;
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int k = 0; k < CHAINS; ++k)
            asm volatile("mma.sync.aligned.m16n8k16.row.col.f32.f16.f16.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, {%0,%1,%2,%3};"
                         : "+f"(c[k][0]), "+f"(c[k][1]), "+f"(c[k][2]), "+f"(c[k][3])
                         : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b[0]), "r"(b[1]));
    }
    float s = 0;
    for (int k = 0; k < CHAINS; ++k) s += c[k][0] + c[k][1] + c[k][2] + c[k][3];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

template <int CHAINS>
__global__ void hmma_tf32(float *out, int iters) {
    unsigned a[4], b[2];
    float c[CHAINS][4];
    for (int i = 0; i < 4; ++i) a[i] = __float_as_uint(1.0f + threadIdx.x * 1e-3f + i);
    for (int i = 0; i < 2; ++i) b[i] = __float_as_uint(0.5f + threadIdx.x * 1e-3f + i);
    for (int k = 0; k < CHAINS; ++k)
        for (int i = 0; i < 4; ++i) c[k][i] = 0.f;
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int k = 0; k < CHAINS; ++k)
            asm volatile("mma.sync.aligned.m16n8k8.row.col.f32.tf32.tf32.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, {%0,%1,%2,%3};"
                         : "+f"(c[k][0]), "+f"(c[k][1]), "+f"(c[k][2]), "+f"(c[k][3])
                         : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b[0]), "r"(b[1]));
    }
    float s = 0;
    for (int k = 0; k < CHAINS; ++k) s += c[k][0] + c[k][1] + c[k][2] + c[k][3];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

// sincos-only throughput (MUFU bound): 8 independent chains per thread
__global__ void sincos_only(float *out, int iters) {
    float x[8], acc = 0.f;
    for (int k = 0; k < 8; ++k) x[k] = threadIdx.x * 1e-3f + k;
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int k = 0; k < 8; ++k) {
            float s, c;
            __sincosf(x[k], &s, &c);
            x[k] = fmaf(c, 0.5f, s);
        }
    }
    for (int k = 0; k < 8; ++k) acc += x[k];
    out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
}

template <typename F>
void time_it(const char *name, F launch, double work_per_launch, const char *unit) {
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    launch();
    cudaDeviceSynchronize();
    cudaEventRecord(e0);
    launch();
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    int clk;
    cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
    printf("%-28s %8.3f ms  %10.2f %s  (%.1f per SM per clk at %.0f MHz)\n", name, ms,
           work_per_launch / (ms * 1e-3) / 1e12, unit, work_per_launch / (ms * 1e-3) / 148 / (clk * 1e3),
           clk / 1e3);
}

int main() {
    float *out;
    cudaMalloc(&out, 148 * 64 * 1024 * sizeof(float));
    const int iters = 4096;
    for (int warps : {4, 8, 16}) {
        const int threads = 32 * warps, blocks = 148 * 2;
        char nm[64];
        snprintf(nm, 64, "hmma f16 m16n8k16 w%d x4", warps);
        time_it(nm, [&] { hmma_f16<4><<<blocks, threads>>>(out, iters); },
                double(blocks) * warps * iters * 4 * 16 * 8 * 16, "T MAC/s");
        snprintf(nm, 64, "hmma tf32 m16n8k8 w%d x4", warps);
        time_it(nm, [&] { hmma_tf32<4><<<blocks, threads>>>(out, iters); },
                double(blocks) * warps * iters * 4 * 16 * 8 * 8, "T MAC/s");
    }
    time_it("sincos (8 chains)", [&] { sincos_only<<<148 * 8, 256>>>(out, iters); },
            double(148 * 8) * 256 * iters * 8, "T sincos/s");
    cudaError_t e = cudaGetLastError();
    printf("status %s\n", cudaGetErrorString(e));
    return 0;
}
