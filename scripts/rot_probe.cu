// rot_probe.cu -- design probe: gridder inner loop per timestep, direct phasors vs accumulator rotation.
//
// Channels of one timestep are J groups of 8 (j = 0..J-1, slot s = 0..7, channel 8j + s).  With uniform
// channel spacing the phase is linear in the channel, so Phi(8j + s) = Phi(s) * E^j with
// E = exp(i 8 dnu/c Q_t) per pixel and timestep.  Hence, per pixel,
//     S_t = sum_j sum_s Phi(8j+s) V(8j+s) = sum_j E^j (sum_s Phi(s) V(8j+s)) = sum_j E^j D_j
// where every D_j is an mma of the SAME A fragment (the slot-s phasors) with group j's B fragment.
// DIRECT: J k-blocks x {4 phasors, 4 splits, 3 mma} per tile (the current kernel).
// ROT:    1 k-block of phasors, J x 3 mma into fresh D_j, E by sincos, E^j by recurrence, acc += E^j D_j.
// Memory-free except the B fragments read from shared memory as in the kernel.
#include <cstdint>
#include <cstdio>
#include <cuda_fp16.h>
#include <cuda_runtime.h>
typedef unsigned long long u64;
__device__ __forceinline__ u64 pk(float a, float b) { u64 r; asm("mov.b64 %0, {%1,%2};" : "=l"(r) : "f"(a), "f"(b)); return r; }
__device__ __forceinline__ float2 up(u64 v) { float2 r; asm("mov.b64 {%0,%1}, %2;" : "=f"(r.x), "=f"(r.y) : "l"(v)); return r; }
__device__ __forceinline__ u64 dup(float a) { return pk(a, a); }
__device__ __forceinline__ u64 fma2(u64 a, u64 b, u64 c) { u64 r; asm("fma.rn.f32x2 %0,%1,%2,%3;" : "=l"(r) : "l"(a), "l"(b), "l"(c)); return r; }
__device__ __forceinline__ u64 mul2(u64 a, u64 b) { u64 r; asm("mul.rn.f32x2 %0,%1,%2;" : "=l"(r) : "l"(a), "l"(b)); return r; }
__device__ __forceinline__ uint32_t h2b(__half2 h) { return *reinterpret_cast<uint32_t *>(&h); }
__device__ __forceinline__ void split_mx(float x, float y, uint32_t &hi, uint32_t &lo) {
    hi = h2b(__floats2half2_rn(x, y));
    float lx, ly;
    asm("{\n.reg .f16 a, b, m;\nmov.b32 {a, b}, %2;\nmov.b16 m, 0xBC00;\n"
        "fma.rn.f32.f16 %0, a, m, %3;\nfma.rn.f32.f16 %1, b, m, %4;\n}"
        : "=f"(lx), "=f"(ly) : "r"(hi), "f"(x), "f"(y));
    lo = h2b(__floats2half2_rn(lx, ly));
}
__device__ __forceinline__ void mma(float (&d)[4], const uint32_t (&a)[4], uint32_t b0, uint32_t b1) {
    asm("mma.sync.aligned.m16n8k16.row.col.f32.f16.f16.f32 {%0,%1,%2,%3},{%4,%5,%6,%7},{%8,%9},{%0,%1,%2,%3};"
        : "+f"(d[0]), "+f"(d[1]), "+f"(d[2]), "+f"(d[3]) : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b0), "r"(b1));
}
__device__ __forceinline__ void mma0(float (&d)[4], const uint32_t (&a)[4], uint32_t b0, uint32_t b1) {
    const float z = 0.0f;
    asm("mma.sync.aligned.m16n8k16.row.col.f32.f16.f16.f32 {%0,%1,%2,%3},{%4,%5,%6,%7},{%8,%9},{%10,%10,%10,%10};"
        : "=f"(d[0]), "=f"(d[1]), "=f"(d[2]), "=f"(d[3]) : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b0), "r"(b1), "f"(z));
}

template <int MT, int J, bool ROT, int W, int MINB>
__global__ void __launch_bounds__(W * 32, MINB) loop(float *out, int iters) {
    __shared__ uint4 frag_s[J][32];
    __shared__ float4 coef_s[2];
    __shared__ float4 dfk_s[J][4];
    const int lane = threadIdx.x & 31, q = lane & 3;
    for (int i = threadIdx.x; i < J * 32; i += blockDim.x)
        frag_s[i / 32][i % 32] = make_uint4(0x3c003c00u ^ i, 0x3c003c01u, 0x3c013c00u, i);
    if (threadIdx.x < J * 4) dfk_s[threadIdx.x / 4][threadIdx.x % 4] = make_float4(1e-3f * threadIdx.x, 2e-3f, 3e-3f, 4e-3f * threadIdx.x);
    if (threadIdx.x == 0) { coef_s[0] = make_float4(0.1f, 0.2f, 0.3f, 0); coef_s[1] = make_float4(1e-3f, 2e-3f, 3e-3f, 0); }
    __syncthreads();
    u64 pl[MT], pm[MT], pn[MT];
    float acc[MT][4];
    for (int i = 0; i < MT; ++i) {
        pl[i] = pk(0.01f * i + lane * 1e-4f, 0.02f); pm[i] = pk(0.03f, 0.01f * lane); pn[i] = pk(1e-4f, 2e-4f);
        for (int j = 0; j < 4; ++j) acc[i][j] = 0;
    }
    const u64 dq = pk(1e-3f * q, 2e-3f), dq4 = pk(3e-3f, 4e-3f * q);
    const u64 est = dup(8.0f * 1.3e-4f);
    for (int it = 0; it < iters; ++it) {
        const float4 cB = coef_s[0], cQ = coef_s[1];
        u64 Bv[MT], Qv[MT];
#pragma unroll
        for (int i = 0; i < MT; ++i) {
            Bv[i] = fma2(dup(cB.x + it * 1e-6f), pl[i], fma2(dup(cB.y), pm[i], mul2(dup(cB.z), pn[i])));
            Qv[i] = fma2(dup(cQ.x), pl[i], fma2(dup(cQ.y), pm[i], mul2(dup(cQ.z + it * 1e-9f), pn[i])));
        }
        if (!ROT) {
#pragma unroll 1
            for (int kb = 0; kb < J; ++kb) {
                const uint4 bf = frag_s[kb][lane];
                const float4 df = dfk_s[kb][q];
                const u64 dq = pk(df.x, df.y), dq4 = pk(df.z, df.w);
                uint32_t ah[MT][4], al[MT][4];
#pragma unroll
                for (int i = 0; i < MT; ++i) {
                    const float2 p0 = up(fma2(dq, Qv[i], Bv[i])), p1 = up(fma2(dq4, Qv[i], Bv[i]));
                    float sn[4], cs[4];
                    __sincosf(p0.x, &sn[0], &cs[0]); __sincosf(p0.y, &sn[1], &cs[1]);
                    __sincosf(p1.x, &sn[2], &cs[2]); __sincosf(p1.y, &sn[3], &cs[3]);
#pragma unroll
                    for (int j = 0; j < 4; ++j) split_mx(cs[j], sn[j], ah[i][j], al[i][j]);
                }
#pragma unroll
                for (int i = 0; i < MT; ++i) mma(acc[i], ah[i], bf.x, bf.y);
#pragma unroll
                for (int i = 0; i < MT; ++i) mma(acc[i], ah[i], bf.z, bf.w);
#pragma unroll
                for (int i = 0; i < MT; ++i) mma(acc[i], al[i], bf.x, bf.y);
            }
        } else {
#pragma unroll
            for (int i = 0; i < MT; ++i) {
                uint32_t ah[4], al[4];
                const float2 p0 = up(fma2(dq, Qv[i], Bv[i])), p1 = up(fma2(dq4, Qv[i], Bv[i]));
                float sn[4], cs[4];
                __sincosf(p0.x, &sn[0], &cs[0]); __sincosf(p0.y, &sn[1], &cs[1]);
                __sincosf(p1.x, &sn[2], &cs[2]); __sincosf(p1.y, &sn[3], &cs[3]);
#pragma unroll
                for (int j = 0; j < 4; ++j) split_mx(cs[j], sn[j], ah[j], al[j]);
                // E = exp(i 8 dnu Q) of rows g, g+8
                const float2 e = up(mul2(est, Qv[i]));
                float es0, ec0, es1, ec1;
                __sincosf(e.x, &es0, &ec0);
                __sincosf(e.y, &es1, &ec1);
                float pr0 = 1.0f, pi0 = 0.0f, pr1 = 1.0f, pi1 = 0.0f;  // E^j
#pragma unroll
                for (int j = 0; j < J; ++j) {
                    const uint4 bf = frag_s[j][lane];
                    float d[4];
                    mma0(d, ah, bf.x, bf.y);
                    mma(d, ah, bf.z, bf.w);
                    mma(d, al, bf.x, bf.y);
                    if (j == 0) {
#pragma unroll
                        for (int k = 0; k < 4; ++k) acc[i][k] += d[k];
                    } else {
                        if (j == 1) { pr0 = ec0; pi0 = es0; pr1 = ec1; pi1 = es1; }
                        else {
                            const float a0 = pr0 * ec0 - pi0 * es0, b0 = pr0 * es0 + pi0 * ec0;
                            const float a1 = pr1 * ec1 - pi1 * es1, b1 = pr1 * es1 + pi1 * ec1;
                            pr0 = a0; pi0 = b0; pr1 = a1; pi1 = b1;
                        }
                        acc[i][0] = fmaf(pr0, d[0], fmaf(-pi0, d[1], acc[i][0]));
                        acc[i][1] = fmaf(pr0, d[1], fmaf(pi0, d[0], acc[i][1]));
                        acc[i][2] = fmaf(pr1, d[2], fmaf(-pi1, d[3], acc[i][2]));
                        acc[i][3] = fmaf(pr1, d[3], fmaf(pi1, d[2], acc[i][3]));
                    }
                }
            }
        }
    }
    float s = 0;
    for (int i = 0; i < MT; ++i) for (int j = 0; j < 4; ++j) s += acc[i][j];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

template <int MT, int J, bool ROT, int warps, int bps>
void run(float *out) {
    const int iters = 1024;
    const int blocks = 148 * bps, threads = 32 * warps;
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0); cudaEventCreate(&e1);
    loop<MT, J, ROT, warps, bps><<<blocks, threads>>>(out, 16);
    cudaDeviceSynchronize();
    cudaEventRecord(e0);
    loop<MT, J, ROT, warps, bps><<<blocks, threads>>>(out, iters);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    const double pairs = double(blocks) * threads * iters * MT * 4 * J;
    printf("%-6s MT %d J %d warps/SM %3d: %6.2f pairs/clk/SM (at 1965 MHz)\n", ROT ? "ROT" : "DIRECT", MT, J,
           warps * bps, pairs / (ms * 1e-3) / 148 / 1.965e9);
}

int main() {
    float *out;
    cudaMalloc(&out, 148 * 64 * 1024 * 4);
    run<3, 2, false, 12, 2>(out);
    run<3, 2, true, 12, 2>(out);
    run<3, 2, true, 12, 1>(out);
    run<3, 2, true, 8, 3>(out);
    run<2, 2, true, 18, 1>(out);
    run<3, 4, false, 12, 2>(out);
    run<3, 4, true, 12, 2>(out);
    run<4, 4, false, 16, 2>(out);
    run<4, 4, true, 16, 2>(out);
    run<4, 4, true, 16, 1>(out);
    run<4, 2, true, 16, 2>(out);
    run<2, 4, true, 16, 2>(out);
    printf("%s\n", cudaGetErrorString(cudaGetLastError()));
}
