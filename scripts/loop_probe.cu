// loop_probe.cu -- attribute the cost of the tensor-core gridder inner loop (design probe).
// Per k-block per thread: MT tiles x {4 phases (FFMA2 x2), 4 sincos, 4 splits, 3 mma}.  Variants
// drop parts to see which one binds.  Grid = 148 x BPS blocks of W warps, no memory traffic.
#include <cstdio>
#include <cstdint>
#include <cuda_fp16.h>
#include <cuda_runtime.h>
typedef unsigned long long u64;
__device__ __forceinline__ u64 pk(float a, float b) { u64 r; asm("mov.b64 %0, {%1,%2};" : "=l"(r) : "f"(a), "f"(b)); return r; }
__device__ __forceinline__ float2 up(u64 v) { float2 r; asm("mov.b64 {%0,%1}, %2;" : "=f"(r.x), "=f"(r.y) : "l"(v)); return r; }
__device__ __forceinline__ u64 fma2(u64 a, u64 b, u64 c) { u64 r; asm("fma.rn.f32x2 %0,%1,%2,%3;" : "=l"(r) : "l"(a), "l"(b), "l"(c)); return r; }
__device__ __forceinline__ u64 sub2(u64 a, u64 b) { u64 r; asm("sub.rn.f32x2 %0,%1,%2;" : "=l"(r) : "l"(a), "l"(b)); return r; }
__device__ __forceinline__ uint32_t h2b(__half2 h) { return *reinterpret_cast<uint32_t *>(&h); }
__device__ __forceinline__ void split(float x, float y, uint32_t &hi, uint32_t &lo) {
    float hx = __uint_as_float(__float_as_uint(x) & 0xffffe000u), hy = __uint_as_float(__float_as_uint(y) & 0xffffe000u);
    float2 d = up(sub2(pk(x, y), pk(hx, hy)));
    hi = h2b(__floats2half2_rn(hx, hy)); lo = h2b(__floats2half2_rn(d.x, d.y));
}
// bf16 split without conversions: hi = upper halves (PRMT), lo = x - hi (FADD2), truncated by PRMT
// hi = rn_f16(x, y); lo = rn_f16(x - hi, y - hi) with the mixed-precision FHFMA (f16 * f16 + f32)
__device__ __forceinline__ void split_mx(float x, float y, uint32_t &hi, uint32_t &lo) {
    const __half2 h = __floats2half2_rn(x, y);
    hi = h2b(h);
    float lx, ly;
    asm("{\n.reg .f16 a, b, m;\nmov.b32 {a, b}, %2;\nmov.b16 m, 0xBC00;\n"
        "fma.rn.f32.f16 %0, a, m, %3;\nfma.rn.f32.f16 %1, b, m, %4;\n}"
        : "=f"(lx), "=f"(ly) : "r"(hi), "f"(x), "f"(y));
    lo = h2b(__floats2half2_rn(lx, ly));
}
__device__ __forceinline__ void split_bf(float x, float y, uint32_t &hi, uint32_t &lo) {
    hi = __byte_perm(__float_as_uint(x), __float_as_uint(y), 0x7632);
    float hx = __uint_as_float(__float_as_uint(x) & 0xffff0000u), hy = __uint_as_float(__float_as_uint(y) & 0xffff0000u);
    float2 d = up(sub2(pk(x, y), pk(hx, hy)));
    lo = __byte_perm(__float_as_uint(d.x), __float_as_uint(d.y), 0x7632);
}
__device__ __forceinline__ void mma_bf(float (&d)[4], const uint32_t (&a)[4], uint32_t b0, uint32_t b1) {
    asm("mma.sync.aligned.m16n8k16.row.col.f32.bf16.bf16.f32 {%0,%1,%2,%3},{%4,%5,%6,%7},{%8,%9},{%0,%1,%2,%3};"
        : "+f"(d[0]), "+f"(d[1]), "+f"(d[2]), "+f"(d[3]) : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b0), "r"(b1));
}
__device__ __forceinline__ void mma(float (&d)[4], const uint32_t (&a)[4], uint32_t b0, uint32_t b1) {
    asm("mma.sync.aligned.m16n8k16.row.col.f32.f16.f16.f32 {%0,%1,%2,%3},{%4,%5,%6,%7},{%8,%9},{%0,%1,%2,%3};"
        : "+f"(d[0]), "+f"(d[1]), "+f"(d[2]), "+f"(d[3]) : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b0), "r"(b1));
}

__device__ __forceinline__ u64 add2(u64 a, u64 b) { u64 r; asm("add.rn.f32x2 %0,%1,%2;" : "=l"(r) : "l"(a), "l"(b)); return r; }
__device__ __forceinline__ u64 mul2(u64 a, u64 b) { u64 r; asm("mul.rn.f32x2 %0,%1,%2;" : "=l"(r) : "l"(a), "l"(b)); return r; }
// sincos on the FMA pipe, two arguments packed: exact reduction to r in [-1/2, 1/2] turns, minimax
// sin(pi r) = r P(r^2), cos(pi r) = Q(r^2), double angle.  |err| <= 7.3e-7.
__device__ __forceinline__ void poly_sincos2(u64 x, u64 &sn, u64 &cs) {
    const u64 M = pk(12582912.0f, 12582912.0f);
    u64 r = mul2(x, pk(0.15915494309189535f, 0.15915494309189535f));
    const u64 k = sub2(add2(r, M), M);
    r = sub2(r, k);
    const u64 t = mul2(r, r);
    u64 ps = fma2(pk(0.07755820453166962f, 0.07755820453166962f), t, pk(-0.5982410311698914f, -0.5982410311698914f));
    ps = fma2(ps, t, pk(2.550069570541382f, 2.550069570541382f));
    ps = fma2(ps, t, pk(-5.167709827423096f, -5.167709827423096f));
    ps = fma2(ps, t, pk(3.1415927410125732f, 3.1415927410125732f));
    ps = mul2(ps, r);
    u64 pc = fma2(pk(0.21968808770179749f, 0.21968808770179749f), t, pk(-1.3318758010864258f, -1.3318758010864258f));
    pc = fma2(pc, t, pk(4.058411121368408f, 4.058411121368408f));
    pc = fma2(pc, t, pk(-4.934792995452881f, -4.934792995452881f));
    pc = fma2(pc, t, pk(0.9999999403953552f, 0.9999999403953552f));
    const u64 u = add2(ps, ps);
    sn = mul2(u, pc);
    const float2 uu = up(u);
    cs = fma2(pk(-uu.x, -uu.y), ps, pk(1.0f, 1.0f));
}
// MODE bits: 1 = sincos, 2 = split, 4 = mma
template <int MT, int MODE>
__global__ void loop(float *out, int iters) {
    const int lane = threadIdx.x & 31;
    u64 B[MT], Q[MT];
    float acc[MT][4];
    for (int i = 0; i < MT; ++i) { B[i] = pk(0.1f * i + lane * 1e-3f, 0.2f); Q[i] = pk(0.3f, 0.4f + i * 1e-2f); for (int j = 0; j < 4; ++j) acc[i][j] = 0; }
    uint32_t b0 = 0x3c003c00u ^ lane, b1 = 0x3c003c01u, b2 = 0x3c013c00u, b3 = lane;
    u64 dq = pk(1e-3f, 2e-3f), dq4 = pk(3e-3f, 4e-3f);
    for (int it = 0; it < iters; ++it) {
        dq = fma2(dq, pk(1.0000001f, 1.0000001f), pk(1e-7f, 1e-7f));
        dq4 = fma2(dq4, pk(1.0000001f, 1.0000001f), pk(2e-7f, 2e-7f));
        uint32_t ah[MT][4], al[MT][4];
#pragma unroll
        for (int i = 0; i < MT; ++i) {
            float2 p0 = up(fma2(dq, Q[i], B[i])), p1 = up(fma2(dq4, Q[i], B[i]));
            float ph[4] = {p0.x, p0.y, p1.x, p1.y}, sn[4], cs[4];
#pragma unroll
            for (int j = 0; j < 4; ++j) {
                if ((MODE & 32) && j >= 2) continue;
                if (MODE & 1) __sincosf(ph[j], &sn[j], &cs[j]); else { sn[j] = ph[j] * 0.5f; cs[j] = ph[j] + 0.25f; }
            }
            if (MODE & 32) {   // slots 2, 3 on the FMA pipe (50% of the phasors)
                u64 s2, c2;
                poly_sincos2(pk(p1.x, p1.y), s2, c2);
                const float2 a = up(s2), b = up(c2);
                sn[2] = a.x; sn[3] = a.y; cs[2] = b.x; cs[3] = b.y;
            }
#pragma unroll
            for (int j = 0; j < 4; ++j) {
                if (MODE & 64) split_mx(cs[j], sn[j], ah[i][j], al[i][j]);
                else if (MODE & 8) split_bf(cs[j], sn[j], ah[i][j], al[i][j]);
                else if (MODE & 2) split(cs[j], sn[j], ah[i][j], al[i][j]);
                else { ah[i][j] = __float_as_uint(cs[j]); al[i][j] = __float_as_uint(sn[j]); }
            }
        }
        if (MODE & 16) {   // tcgen05-style: stage the split A operands in shared memory (2 x STS.128 / tile)
            __shared__ uint4 stage[2][48][32];
            const int slot = it & 1;
#pragma unroll
            for (int i = 0; i < MT; ++i) {
                stage[slot][((threadIdx.x >> 5) * MT + i) % 24][lane] = make_uint4(ah[i][0], ah[i][1], ah[i][2], ah[i][3]);
                stage[slot][((threadIdx.x >> 5) * MT + i) % 24 + 24][lane] = make_uint4(al[i][0], al[i][1], al[i][2], al[i][3]);
            }
            if ((it & 7) == 7) __syncwarp();
            acc[0][0] += 1e-30f * __uint_as_float(stage[slot ^ 1][0][lane].x);
        } else if ((MODE & 4) && (MODE & 8)) {
#pragma unroll
            for (int i = 0; i < MT; ++i) mma_bf(acc[i], ah[i], b0, b1);
#pragma unroll
            for (int i = 0; i < MT; ++i) mma_bf(acc[i], ah[i], b2, b3);
#pragma unroll
            for (int i = 0; i < MT; ++i) mma_bf(acc[i], al[i], b0, b1);
        } else if (MODE & 4) {
#pragma unroll
            for (int i = 0; i < MT; ++i) mma(acc[i], ah[i], b0, b1);
#pragma unroll
            for (int i = 0; i < MT; ++i) mma(acc[i], ah[i], b2, b3);
#pragma unroll
            for (int i = 0; i < MT; ++i) mma(acc[i], al[i], b0, b1);
        } else {
#pragma unroll
            for (int i = 0; i < MT; ++i)
#pragma unroll
                for (int j = 0; j < 4; ++j) acc[i][j] += __uint_as_float(ah[i][j] ^ al[i][j]);
        }
    }
    float s = 0; for (int i = 0; i < MT; ++i) for (int j = 0; j < 4; ++j) s += acc[i][j];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
template <int MT, int MODE>
void run(const char *name, int warps, int bps, float *out) {
    const int iters = 2048;
    const int blocks = 148 * bps, threads = 32 * warps;
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    loop<MT, MODE><<<blocks, threads>>>(out, 16); cudaDeviceSynchronize();
    cudaEventRecord(e0); loop<MT, MODE><<<blocks, threads>>>(out, iters); cudaEventRecord(e1); cudaEventSynchronize(e1);
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    double pairs = double(blocks) * threads * iters * MT * 4;
    int clk; cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
    printf("%-34s warps/SM %3d: %6.2f pairs/clk/SM\n", name, warps * bps, pairs / (ms * 1e-3) / 148 / 1.965e9);
}

// software-pipelined variant: sincos of iteration it+1 are issued before the split + mma of iteration it
template <int MT>
__global__ void loop_pipe(float *out, int iters) {
    const int lane = threadIdx.x & 31;
    u64 B[MT], Q[MT];
    float acc[MT][4];
    for (int i = 0; i < MT; ++i) { B[i] = pk(0.1f * i + lane * 1e-3f, 0.2f); Q[i] = pk(0.3f, 0.4f + i * 1e-2f); for (int j = 0; j < 4; ++j) acc[i][j] = 0; }
    uint32_t b0 = 0x3c003c00u ^ lane, b1 = 0x3c003c01u, b2 = 0x3c013c00u, b3 = lane;
    u64 dq = pk(1e-3f, 2e-3f), dq4 = pk(3e-3f, 4e-3f);
    float sn[MT][4], cs[MT][4];
    auto phasors = [&](float (&sn_)[MT][4], float (&cs_)[MT][4]) {
        dq = fma2(dq, pk(1.0000001f, 1.0000001f), pk(1e-7f, 1e-7f));
        dq4 = fma2(dq4, pk(1.0000001f, 1.0000001f), pk(2e-7f, 2e-7f));
#pragma unroll
        for (int i = 0; i < MT; ++i) {
            float2 p0 = up(fma2(dq, Q[i], B[i])), p1 = up(fma2(dq4, Q[i], B[i]));
            __sincosf(p0.x, &sn_[i][0], &cs_[i][0]); __sincosf(p0.y, &sn_[i][1], &cs_[i][1]);
            __sincosf(p1.x, &sn_[i][2], &cs_[i][2]); __sincosf(p1.y, &sn_[i][3], &cs_[i][3]);
        }
    };
    phasors(sn, cs);
    for (int it = 0; it < iters; ++it) {
        uint32_t ah[MT][4], al[MT][4];
#pragma unroll
        for (int i = 0; i < MT; ++i)
#pragma unroll
            for (int j = 0; j < 4; ++j) split(cs[i][j], sn[i][j], ah[i][j], al[i][j]);
        phasors(sn, cs);   // next iteration's MUFU work, independent of the mma below
#pragma unroll
        for (int i = 0; i < MT; ++i) mma(acc[i], ah[i], b0, b1);
#pragma unroll
        for (int i = 0; i < MT; ++i) mma(acc[i], ah[i], b2, b3);
#pragma unroll
        for (int i = 0; i < MT; ++i) mma(acc[i], al[i], b0, b1);
    }
    float s = 0; for (int i = 0; i < MT; ++i) for (int j = 0; j < 4; ++j) s += acc[i][j];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
template <int MT>
void run_pipe(const char *name, int warps, int bps, float *out) {
    const int iters = 2048;
    const int blocks = 148 * bps, threads = 32 * warps;
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    loop_pipe<MT><<<blocks, threads>>>(out, 16); cudaDeviceSynchronize();
    cudaEventRecord(e0); loop_pipe<MT><<<blocks, threads>>>(out, iters); cudaEventRecord(e1); cudaEventSynchronize(e1);
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    double pairs = double(blocks) * threads * iters * MT * 4;
    printf("%-34s warps/SM %3d: %6.2f pairs/clk/SM\n", name, warps * bps, pairs / (ms * 1e-3) / 148 / 1.965e9);
}
int main() {
    float *out; cudaMalloc(&out, 148 * 64 * 1024 * 4);
    for (int bps : {2, 3}) {
        run<3, 7>("f16 full (sincos+split+mma)", 12, bps, out);
        run<3, 7 | 64>("full, FHFMA split", 12, bps, out);
        run<3, 6 | 64>("FHFMA split + mma only", 12, bps, out);
        run<3, 6>("LOP3 split + mma only", 12, bps, out);
    }
    printf("%s\n", cudaGetErrorString(cudaGetLastError()));
}
