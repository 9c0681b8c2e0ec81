// split_probe.cu -- design probe: the N~ = 32 degridder k-block loop (R = 16 rows per lane, two rotation
// chains, 8 m-tiles, 3 mma per tile) with three forms of the phasor operand split:
//   VAR 0  the kernel's split: hi = cvt.rn.f16x2(c, s), lo = cvt(c - hi, s - hi) via two FHFMA  (4 / phasor)
//   VAR 1  fixed-point split by byte permutation: W = sigma Z + M (one FFMA2 per packed pair) puts an
//          18-bit offset fixed-point Z in the low bits of an fp32 in [2^23, 2^24) whose upper bytes are
//          the f16 exponent patterns; hi = PRMT(bytes 1, 2), lo = PRMT(bytes 0, 3)            (3 / phasor)
//   VAR 2  as 1, with the rotation run on W itself (W' = W E + M (1 - E)): no FFMA2 for the split (2 / phasor)
//   loop8  R = 8 rows per lane with the VAR 1 split, one or two rotation chains
//   loopi  the integer form: 16-bit fixed-point phasor as two u8 limbs (one PRMT per phasor), three
//          mma.m16n8k32 u8 x s8 per tile into s32 accumulators (the kernels' degridder_rot16i)
// VARF bit 4 drops the mma (the ALU side alone), bits 8/16 keep 2 / 1 of the 3 products, bit 32 the rotation.
// Same shared-memory operands as the kernel (B fragments, slot l/m/n), no global traffic.
// Prints pairs per clock per SM at the nominal 1965 MHz (profiles/r02zd_split_probe.txt).
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cuda_fp16.h>
#include <cuda_runtime.h>
typedef unsigned long long f2p;
__device__ __forceinline__ f2p pk(float a, float b) { f2p r; asm("mov.b64 %0, {%1,%2};" : "=l"(r) : "f"(a), "f"(b)); return r; }
__device__ __forceinline__ float2 unpk(f2p v) { float2 r; asm("mov.b64 {%0,%1}, %2;" : "=f"(r.x), "=f"(r.y) : "l"(v)); return r; }
__device__ __forceinline__ f2p dup(float a) { return pk(a, a); }
__device__ __forceinline__ f2p fma2(f2p a, f2p b, f2p c) { f2p r; asm("fma.rn.f32x2 %0,%1,%2,%3;" : "=l"(r) : "l"(a), "l"(b), "l"(c)); return r; }
__device__ __forceinline__ f2p mul2(f2p a, f2p b) { f2p r; asm("mul.rn.f32x2 %0,%1,%2;" : "=l"(r) : "l"(a), "l"(b)); return r; }
__device__ __forceinline__ uint32_t h2b(__half2 h) { return *reinterpret_cast<uint32_t *>(&h); }
__device__ __forceinline__ void split2(float x, float y, uint32_t &hi, uint32_t &lo) {
    hi = h2b(__floats2half2_rn(x, y));
    float dx, dy;
    asm("{\n.reg .f16 a, b, m;\nmov.b32 {a, b}, %2;\nmov.b16 m, 0xBC00;\n"
        "fma.rn.f32.f16 %0, a, m, %3;\nfma.rn.f32.f16 %1, b, m, %4;\n}"
        : "=f"(dx), "=f"(dy) : "r"(hi), "f"(x), "f"(y));
    lo = h2b(__floats2half2_rn(dx, dy));
}
__device__ __forceinline__ uint32_t prmt(float a, float b, uint32_t sel) {
    uint32_t r;
    asm("prmt.b32 %0, %1, %2, %3;" : "=r"(r) : "r"(__float_as_uint(a)), "r"(__float_as_uint(b)), "r"(sel));
    return r;
}
__device__ __forceinline__ void mma16816(float (&d)[4], const uint32_t (&a)[4], uint32_t b0, uint32_t b1) {
    asm("mma.sync.aligned.m16n8k16.row.col.f32.f16.f16.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, {%0,%1,%2,%3};"
        : "+f"(d[0]), "+f"(d[1]), "+f"(d[2]), "+f"(d[3]) : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b0), "r"(b1));
}
__device__ __forceinline__ void mma3(float (&d)[4], const uint32_t (&ah)[4], const uint32_t (&al)[4], const uint4 &b) {
    mma16816(d, ah, b.x, b.y);
    mma16816(d, ah, b.z, b.w);
    mma16816(d, al, b.x, b.y);
}

constexpr int NKB = 128;     // N~ = 32: 1024 pixels / 8
constexpr float kSig = 131000.0f;
constexpr float kM = 15335424.0f;   // 2^23 + 0x680000 + 2^17

template <int VARF, int W, int MINB, int UNR>
__global__ void __launch_bounds__(W * 32, MINB) loop(float *out, int units) {
    constexpr int VAR = VARF & 3;
    constexpr bool NOMMA = VARF & 4;
    constexpr int NMMA = (VARF >> 3) & 3;   // 0: 3 mma per tile, 1: 2, 2: 1
    constexpr bool NOROT = VARF & 32;
    extern __shared__ __align__(16) unsigned char smem[];
    uint4 *frag_s = reinterpret_cast<uint4 *>(smem);
    float4 *lmn_s = reinterpret_cast<float4 *>(smem + NKB * 32 * 16);
    for (int i = threadIdx.x; i < NKB * 32; i += blockDim.x)
        frag_s[i] = make_uint4(0x3c003c00u ^ (i & 0x3ff), 0x3c003c01u, 0x14011401u, 0x14001400u ^ (i & 0xff));
    for (int i = threadIdx.x; i < NKB * 8; i += blockDim.x)
        lmn_s[i] = make_float4(1e-3f * (i & 31), 2e-3f * (i >> 5), 3e-4f * (i & 7), 1e-4f);
    __syncthreads();
    const int lane = threadIdx.x & 31, q = lane & 3;
    float total = 0.0f;
    for (int u = 0; u < units; ++u) {
        const float fu = 0.3f + 1e-3f * u + 1e-4f * lane, fv = 0.2f, fw = 0.05f;
        const f2p cu = dup(fu), cv = dup(fv), cw = dup(fw);
        const f2p eu = dup(0.011f), ev = dup(0.007f), ew = dup(0.001f);
        float acc[8][4];
#pragma unroll
        for (int i = 0; i < 8; ++i)
#pragma unroll
            for (int j = 0; j < 4; ++j) acc[i][j] = 0.0f;
#pragma unroll UNR
        for (int kb = 0; kb < NKB; ++kb) {
            const uint4 bf = frag_s[kb * 32 + lane];
            const float4 lm = lmn_s[(kb * 4 + q) * 2], nn = lmn_s[(kb * 4 + q) * 2 + 1];
            const f2p l2 = pk(lm.x, lm.y), m2 = pk(lm.z, lm.w), n2 = pk(nn.x, nn.y);
            const float2 p = unpk(fma2(cu, l2, fma2(cv, m2, mul2(cw, n2))));
            const float2 e = unpk(fma2(eu, l2, fma2(ev, m2, mul2(ew, n2))));
            float s0, c0q, s1, c1q, es0, ec0, es1, ec1;
            __sincosf(p.x, &s0, &c0q);
            __sincosf(p.y, &s1, &c1q);
            __sincosf(e.x, &es0, &ec0);
            __sincosf(e.y, &es1, &ec1);
            f2p C = pk(c0q, c1q), S = pk(s0, s1);
            const f2p EC = pk(ec0, ec1), ES = pk(es0, es1), NES = pk(-es0, -es1);
            const f2p ph8 = fma2(dup(8.0f), pk(e.x, e.y), pk(p.x, p.y));
            const float2 p8 = unpk(ph8);
            float s8a, c8a, s8b, c8b;
            __sincosf(p8.x, &s8a, &c8a);
            __sincosf(p8.y, &s8b, &c8b);
            f2p C2 = pk(c8a, c8b), S2 = pk(s8a, s8b);
            f2p Kc, Ks;
            const f2p SIG = dup(kSig), MM = dup(kM);
            if (VAR == 2) {
                const f2p MN = dup(-kM);
                Kc = fma2(MN, EC, fma2(MM, ES, MM));
                Ks = fma2(MN, EC, fma2(MN, ES, MM));
                C = fma2(C, SIG, MM); S = fma2(S, SIG, MM);
                C2 = fma2(C2, SIG, MM); S2 = fma2(S2, SIG, MM);
            }
#pragma unroll
            for (int i = 0; i < 4; ++i) {
                uint32_t ah[4], al[4], bh[4], bl[4];
#pragma unroll
                for (int h2 = 0; h2 < 2; ++h2) {
                    if ((i > 0 || h2 > 0) && !NOROT) {
                        if (VAR == 2) {
                            const f2p Cn = fma2(C, EC, fma2(S, NES, Kc));
                            S = fma2(C, ES, fma2(S, EC, Ks));
                            C = Cn;
                            const f2p Cm = fma2(C2, EC, fma2(S2, NES, Kc));
                            S2 = fma2(C2, ES, fma2(S2, EC, Ks));
                            C2 = Cm;
                        } else {
                            const f2p Cn = fma2(C, EC, mul2(S, NES));
                            S = fma2(C, ES, mul2(S, EC));
                            C = Cn;
                            const f2p Cm = fma2(C2, EC, mul2(S2, NES));
                            S2 = fma2(C2, ES, mul2(S2, EC));
                            C2 = Cm;
                        }
                    }
                    if (VAR == 0) {
                        const float2 cc = unpk(C), ss = unpk(S), cc2 = unpk(C2), ss2 = unpk(S2);
                        split2(cc.x, ss.x, ah[h2], al[h2]);
                        split2(cc.y, ss.y, ah[2 + h2], al[2 + h2]);
                        split2(cc2.x, ss2.x, bh[h2], bl[h2]);
                        split2(cc2.y, ss2.y, bh[2 + h2], bl[2 + h2]);
                    } else {
                        float2 cc, ss, cc2, ss2;
                        if (VAR == 1) {
                            cc = unpk(fma2(C, SIG, MM)); ss = unpk(fma2(S, SIG, MM));
                            cc2 = unpk(fma2(C2, SIG, MM)); ss2 = unpk(fma2(S2, SIG, MM));
                        } else {
                            cc = unpk(C); ss = unpk(S); cc2 = unpk(C2); ss2 = unpk(S2);
                        }
                        ah[h2] = prmt(cc.x, ss.x, 0x6521); al[h2] = prmt(cc.x, ss.x, 0x7430);
                        ah[2 + h2] = prmt(cc.y, ss.y, 0x6521); al[2 + h2] = prmt(cc.y, ss.y, 0x7430);
                        bh[h2] = prmt(cc2.x, ss2.x, 0x6521); bl[h2] = prmt(cc2.x, ss2.x, 0x7430);
                        bh[2 + h2] = prmt(cc2.y, ss2.y, 0x6521); bl[2 + h2] = prmt(cc2.y, ss2.y, 0x7430);
                    }
                }
                if (NOMMA) {
#pragma unroll
                    for (int j = 0; j < 4; ++j) {
                        acc[i][j] += __uint_as_float(ah[j] ^ al[j]);
                        acc[i + 4][j] += __uint_as_float(bh[j] ^ bl[j]);
                    }
                } else if (NMMA == 0) {
                    mma3(acc[i], ah, al, bf);
                    mma3(acc[i + 4], bh, bl, bf);
                } else if (NMMA == 1) {
                    mma16816(acc[i], ah, bf.x, bf.y); mma16816(acc[i + 4], bh, bf.x, bf.y);
                    mma16816(acc[i], al, bf.z, bf.w); mma16816(acc[i + 4], bl, bf.z, bf.w);
                } else {
                    uint32_t x[4], y[4];
                    for (int j = 0; j < 4; ++j) { x[j] = ah[j] ^ al[j]; y[j] = bh[j] ^ bl[j]; }
                    mma16816(acc[i], x, bf.x, bf.y); mma16816(acc[i + 4], y, bf.z, bf.w);
                }
            }
        }
#pragma unroll
        for (int i = 0; i < 8; ++i) total += acc[i][0] + acc[i][1] + acc[i][2] + acc[i][3];
    }
    out[blockIdx.x * blockDim.x + threadIdx.x] = total;
}

template <int VAR, int W, int MINB, int UNR>
void run(const char *name, float *out, int ctas_per_sm) {
    auto k = loop<VAR, W, MINB, UNR>;
    const size_t smem = NKB * 32 * 16 + NKB * 8 * 16;
    cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
    cudaFuncAttributes fa;
    cudaFuncGetAttributes(&fa, k);
    const int blocks = 148 * ctas_per_sm, units = 40;
    k<<<blocks, W * 32, smem>>>(out, 2);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0); cudaEventCreate(&e1);
    float best = 1e30f;
    for (int rep = 0; rep < 3; ++rep) {
        cudaEventRecord(e0);
        k<<<blocks, W * 32, smem>>>(out, units);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms; cudaEventElapsedTime(&ms, e0, e1);
        best = ms < best ? ms : best;
    }
    const double pairs = double(blocks) * W * units * 128.0 * 1024.0;
    printf("%-44s regs %3d  %.3f ms  %.2f pairs/clk/SM  %s\n", name, fa.numRegs, best,
           pairs / (best * 1e-3) / 148 / 1.965e9, cudaGetErrorString(cudaGetLastError()));
}


// R = 8 rows per lane (4 m-tiles), FX split, CH rotation chains (1: rows 1..7 from row 0; 2: rows 4..7 from row 4)
template <int W, int MINB, int UNR, int CH>
__global__ void __launch_bounds__(W * 32, MINB) loop8(float *out, int units) {
    extern __shared__ __align__(16) unsigned char smem[];
    uint4 *frag_s = reinterpret_cast<uint4 *>(smem);
    float4 *lmn_s = reinterpret_cast<float4 *>(smem + NKB * 32 * 16);
    for (int i = threadIdx.x; i < NKB * 32; i += blockDim.x)
        frag_s[i] = make_uint4(0x3c003c00u ^ (i & 0x3ff), 0x3c003c01u, 0x14011401u, 0x14001400u ^ (i & 0xff));
    for (int i = threadIdx.x; i < NKB * 8; i += blockDim.x)
        lmn_s[i] = make_float4(1e-3f * (i & 31), 2e-3f * (i >> 5), 3e-4f * (i & 7), 1e-4f);
    __syncthreads();
    const int lane = threadIdx.x & 31, q = lane & 3;
    float total = 0.0f;
    for (int u = 0; u < 2 * units; ++u) {
        const float fu = 0.3f + 1e-3f * u + 1e-4f * lane, fv = 0.2f, fw = 0.05f;
        const f2p cu = dup(fu), cv = dup(fv), cw = dup(fw);
        const f2p eu = dup(0.011f), ev = dup(0.007f), ew = dup(0.001f);
        float acc[4][4];
#pragma unroll
        for (int i = 0; i < 4; ++i)
#pragma unroll
            for (int j = 0; j < 4; ++j) acc[i][j] = 0.0f;
#pragma unroll UNR
        for (int kb = 0; kb < NKB; ++kb) {
            const uint4 bf = frag_s[kb * 32 + lane];
            const float4 lm = lmn_s[(kb * 4 + q) * 2], nn = lmn_s[(kb * 4 + q) * 2 + 1];
            const f2p l2 = pk(lm.x, lm.y), m2 = pk(lm.z, lm.w), n2 = pk(nn.x, nn.y);
            const float2 p = unpk(fma2(cu, l2, fma2(cv, m2, mul2(cw, n2))));
            const float2 e = unpk(fma2(eu, l2, fma2(ev, m2, mul2(ew, n2))));
            float s0, c0q, s1, c1q, es0, ec0, es1, ec1;
            __sincosf(p.x, &s0, &c0q);
            __sincosf(p.y, &s1, &c1q);
            __sincosf(e.x, &es0, &ec0);
            __sincosf(e.y, &es1, &ec1);
            f2p C = pk(c0q, c1q), S = pk(s0, s1);
            const f2p EC = pk(ec0, ec1), ES = pk(es0, es1), NES = pk(-es0, -es1);
            f2p C2 = C, S2 = S;
            if (CH == 2) {
                const float2 p4 = unpk(fma2(dup(4.0f), pk(e.x, e.y), pk(p.x, p.y)));
                float s4a, c4a, s4b, c4b;
                __sincosf(p4.x, &s4a, &c4a);
                __sincosf(p4.y, &s4b, &c4b);
                C2 = pk(c4a, c4b); S2 = pk(s4a, s4b);
            }
            const f2p SIG = dup(kSig), MM = dup(kM);
#pragma unroll
            for (int i = 0; i < (CH == 2 ? 2 : 4); ++i) {
                uint32_t ah[4], al[4], bh[4], bl[4];
#pragma unroll
                for (int h2 = 0; h2 < 2; ++h2) {
                    if (i > 0 || h2 > 0) {
                        const f2p Cn = fma2(C, EC, mul2(S, NES));
                        S = fma2(C, ES, mul2(S, EC));
                        C = Cn;
                        if (CH == 2) {
                            const f2p Cm = fma2(C2, EC, mul2(S2, NES));
                            S2 = fma2(C2, ES, mul2(S2, EC));
                            C2 = Cm;
                        }
                    }
                    float2 cc = unpk(fma2(C, SIG, MM)), ss = unpk(fma2(S, SIG, MM));
                    ah[h2] = prmt(cc.x, ss.x, 0x6521); al[h2] = prmt(cc.x, ss.x, 0x7430);
                    ah[2 + h2] = prmt(cc.y, ss.y, 0x6521); al[2 + h2] = prmt(cc.y, ss.y, 0x7430);
                    if (CH == 2) {
                        float2 cc2 = unpk(fma2(C2, SIG, MM)), ss2 = unpk(fma2(S2, SIG, MM));
                        bh[h2] = prmt(cc2.x, ss2.x, 0x6521); bl[h2] = prmt(cc2.x, ss2.x, 0x7430);
                        bh[2 + h2] = prmt(cc2.y, ss2.y, 0x6521); bl[2 + h2] = prmt(cc2.y, ss2.y, 0x7430);
                    }
                }
                mma3(acc[i], ah, al, bf);
                if (CH == 2) mma3(acc[i + 2], bh, bl, bf);
            }
        }
#pragma unroll
        for (int i = 0; i < 4; ++i) total += acc[i][0] + acc[i][1] + acc[i][2] + acc[i][3];
    }
    out[blockIdx.x * blockDim.x + threadIdx.x] = total;
}

template <int W, int MINB, int UNR, int CH>
void run8(const char *name, float *out, int ctas_per_sm) {
    auto k = loop8<W, MINB, UNR, CH>;
    const size_t smem = NKB * 32 * 16 + NKB * 8 * 16;
    cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
    cudaFuncAttributes fa;
    cudaFuncGetAttributes(&fa, k);
    const int blocks = 148 * ctas_per_sm, units = 40;
    k<<<blocks, W * 32, smem>>>(out, 2);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0); cudaEventCreate(&e1);
    float best = 1e30f;
    for (int rep = 0; rep < 3; ++rep) {
        cudaEventRecord(e0);
        k<<<blocks, W * 32, smem>>>(out, units);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms; cudaEventElapsedTime(&ms, e0, e1);
        best = ms < best ? ms : best;
    }
    const double pairs = double(blocks) * W * units * 128.0 * 1024.0;
    printf("%-44s regs %3d  %.3f ms  %.2f pairs/clk/SM  %s\n", name, fa.numRegs, best,
           pairs / (best * 1e-3) / 148 / 1.965e9, cudaGetErrorString(cudaGetLastError()));
}


// IMMA form: A = 16-bit offset fixed-point phasor as two u8 limbs (one PRMT per phasor: bytes 0, 1 of the
// (cos, sin) words), B = 24-bit subgrid as three s8 limbs, three m16n8k32 u8 x s8 mma per tile (weights
// 2^24, 2^16, 2^8) into three s32 accumulators.  R rows per lane, one rotation chain.
__device__ __forceinline__ void imma(int (&d)[4], const uint32_t (&a)[4], uint32_t b0, uint32_t b1) {
    asm("mma.sync.aligned.m16n8k32.row.col.s32.u8.s8.s32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, {%0,%1,%2,%3};"
        : "+r"(d[0]), "+r"(d[1]), "+r"(d[2]), "+r"(d[3]) : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b0), "r"(b1));
}
template <int W, int MINB, int UNR, int R, int CH = 1>
__global__ void __launch_bounds__(W * 32, MINB) loopi(float *out, int units) {
    constexpr int NTL = R / 2;
    extern __shared__ __align__(16) unsigned char smem[];
    uint4 *frag_s = reinterpret_cast<uint4 *>(smem);      // [NKB][32] {w24, w16}
    uint2 *frag2_s = reinterpret_cast<uint2 *>(smem + NKB * 32 * 16);   // [NKB][32] {w8}
    float4 *lmn_s = reinterpret_cast<float4 *>(smem + NKB * 32 * 24);
    for (int i = threadIdx.x; i < NKB * 32; i += blockDim.x) {
        frag_s[i] = make_uint4(0x01020304u ^ (i & 0x3ff), 0x05060708u, 0x7f017f01u, 0x11223344u ^ (i & 0xff));
        frag2_s[i] = make_uint2(0x01020304u ^ i, 0x05060708u);
    }
    for (int i = threadIdx.x; i < NKB * 8; i += blockDim.x)
        lmn_s[i] = make_float4(1e-3f * (i & 31), 2e-3f * (i >> 5), 3e-4f * (i & 7), 1e-4f);
    __syncthreads();
    const int lane = threadIdx.x & 31, q = lane & 3;
    float total = 0.0f;
    for (int u = 0; u < units * 16 / R; ++u) {
        const float fu = 0.3f + 1e-3f * u + 1e-4f * lane, fv = 0.2f, fw = 0.05f;
        const f2p cu = dup(fu), cv = dup(fv), cw = dup(fw);
        const f2p eu = dup(0.011f), ev = dup(0.007f), ew = dup(0.001f);
        int acc[NTL][3][4];
#pragma unroll
        for (int i = 0; i < NTL; ++i)
#pragma unroll
            for (int w = 0; w < 3; ++w)
#pragma unroll
                for (int j = 0; j < 4; ++j) acc[i][w][j] = 0;
#pragma unroll UNR
        for (int kb = 0; kb < NKB; ++kb) {
            const uint4 b01 = frag_s[kb * 32 + lane];
            const uint2 b2 = frag2_s[kb * 32 + lane];
            const float4 lm = lmn_s[(kb * 4 + q) * 2], nn = lmn_s[(kb * 4 + q) * 2 + 1];
            const f2p l2 = pk(lm.x, lm.y), m2 = pk(lm.z, lm.w), n2 = pk(nn.x, nn.y);
            const float2 p = unpk(fma2(cu, l2, fma2(cv, m2, mul2(cw, n2))));
            const float2 e = unpk(fma2(eu, l2, fma2(ev, m2, mul2(ew, n2))));
            float s0, c0q, s1, c1q, es0, ec0, es1, ec1;
            __sincosf(p.x, &s0, &c0q);
            __sincosf(p.y, &s1, &c1q);
            __sincosf(e.x, &es0, &ec0);
            __sincosf(e.y, &es1, &ec1);
            f2p C = pk(c0q, c1q), S = pk(s0, s1);
            const f2p EC = pk(ec0, ec1), ES = pk(es0, es1), NES = pk(-es0, -es1);
            const f2p SIG = dup(32767.0f), MM = dup(8421376.0f);   // 2^23 + 2^15
            f2p C2 = C, S2 = S;
            if (CH == 2) {
                const float2 ph = unpk(fma2(dup(float(R / 2)), pk(e.x, e.y), pk(p.x, p.y)));
                float sa, ca, sb, cb;
                __sincosf(ph.x, &sa, &ca);
                __sincosf(ph.y, &sb, &cb);
                C2 = pk(ca, cb); S2 = pk(sa, sb);
            }
#pragma unroll
            for (int i = 0; i < NTL / CH; ++i) {
                uint32_t a[4], b[4];
#pragma unroll
                for (int h2 = 0; h2 < 2; ++h2) {
                    if (i > 0 || h2 > 0) {
                        const f2p Cn = fma2(C, EC, mul2(S, NES));
                        S = fma2(C, ES, mul2(S, EC));
                        C = Cn;
                        if (CH == 2) {
                            const f2p Cm = fma2(C2, EC, mul2(S2, NES));
                            S2 = fma2(C2, ES, mul2(S2, EC));
                            C2 = Cm;
                        }
                    }
                    const float2 cc = unpk(fma2(C, SIG, MM)), ss = unpk(fma2(S, SIG, MM));
                    a[h2] = prmt(cc.x, ss.x, 0x5410);
                    a[2 + h2] = prmt(cc.y, ss.y, 0x5410);
                    if (CH == 2) {
                        const float2 cc2 = unpk(fma2(C2, SIG, MM)), ss2 = unpk(fma2(S2, SIG, MM));
                        b[h2] = prmt(cc2.x, ss2.x, 0x5410);
                        b[2 + h2] = prmt(cc2.y, ss2.y, 0x5410);
                    }
                }
                imma(acc[i][0], a, b01.x, b01.y);
                imma(acc[i][1], a, b01.z, b01.w);
                imma(acc[i][2], a, b2.x, b2.y);
                if (CH == 2) {
                    imma(acc[i + NTL / 2][0], b, b01.x, b01.y);
                    imma(acc[i + NTL / 2][1], b, b01.z, b01.w);
                    imma(acc[i + NTL / 2][2], b, b2.x, b2.y);
                }
            }
        }
#pragma unroll
        for (int i = 0; i < NTL; ++i)
#pragma unroll
            for (int j = 0; j < 4; ++j)
                total += 16777216.0f * float(acc[i][0][j]) + 65536.0f * float(acc[i][1][j]) + 256.0f * float(acc[i][2][j]);
    }
    out[blockIdx.x * blockDim.x + threadIdx.x] = total;
}

template <int W, int MINB, int UNR, int R, int CH = 1>
void runi(const char *name, float *out, int ctas_per_sm) {
    auto k = loopi<W, MINB, UNR, R, CH>;
    const size_t smem = NKB * 32 * 24 + NKB * 8 * 16;
    cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
    cudaFuncAttributes fa;
    cudaFuncGetAttributes(&fa, k);
    const int blocks = 148 * ctas_per_sm, units = 40;
    k<<<blocks, W * 32, smem>>>(out, 2);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0); cudaEventCreate(&e1);
    float best = 1e30f;
    for (int rep = 0; rep < 3; ++rep) {
        cudaEventRecord(e0);
        k<<<blocks, W * 32, smem>>>(out, units);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms; cudaEventElapsedTime(&ms, e0, e1);
        best = ms < best ? ms : best;
    }
    const double pairs = double(blocks) * W * units * 128.0 * 1024.0;
    printf("%-44s regs %3d  %.3f ms  %.2f pairs/clk/SM  %s\n", name, fa.numRegs, best,
           pairs / (best * 1e-3) / 148 / 1.965e9, cudaGetErrorString(cudaGetLastError()));
}

// Host check of the byte-permutation split: hi + lo == 3086 + (sigma Z rounded) / 128 exactly.
__global__ void check(const float *z, float *err, int n) {
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= n) return;
    const float zc = z[2 * i], zs = z[2 * i + 1];
    const float wc = fmaf(zc, kSig, kM), ws = fmaf(zs, kSig, kM);
    const uint32_t hi = prmt(wc, ws, 0x6521), lo = prmt(wc, ws, 0x7430);
    const __half2 h = *reinterpret_cast<const __half2 *>(&hi), l = *reinterpret_cast<const __half2 *>(&lo);
    const float vc = __low2float(h) + __low2float(l), vs = __high2float(h) + __high2float(l);
    // vc = 3086 + round(sigma zc) / 128  ->  z' = (vc - 3086) * 128 / sigma
    err[2 * i] = (vc - 3086.0f) * 128.0f / kSig - zc;
    err[2 * i + 1] = (vs - 3086.0f) * 128.0f / kSig - zs;
}

int main(int argc, char **argv) {
    const int only = argc > 1 ? atoi(argv[1]) : -1;
    float *out;
    cudaMalloc(&out, 148 * 4 * 1024 * 4);
    {
        const int n = 1 << 20;
        float *hz = new float[2 * n], *he = new float[2 * n], *dz, *de;
        unsigned s = 12345;
        for (int i = 0; i < 2 * n; ++i) { s = s * 1664525u + 1013904223u; hz[i] = (int(s >> 8) - (1 << 23)) / float(1 << 23); }
        hz[0] = 1.0f; hz[1] = -1.0f;
        cudaMalloc(&dz, 8 * n); cudaMalloc(&de, 8 * n);
        cudaMemcpy(dz, hz, 8 * n, cudaMemcpyHostToDevice);
        check<<<n / 256, 256>>>(dz, de, n);
        cudaMemcpy(he, de, 8 * n, cudaMemcpyDeviceToHost);
        double mx = 0, ss = 0;
        for (int i = 0; i < 2 * n; ++i) { mx = fmax(mx, fabs(he[i])); ss += double(he[i]) * he[i]; }
        printf("PRMT split: max |err| %.3e (bound 0.5/sigma = %.3e), rms %.3e\n", mx, 0.5 / kSig, sqrt(ss / (2 * n)));
    }
    run<1, 8, 2, 2>("VAR1 R16 s2 W8 minB2 U2 (f16 fixed-point)", out, 2);
    run8<8, 2, 1, 1>("R8 1 chain W8 minB2 U1 (f16 fixed-point)", out, 2);
    runi<8, 2, 2, 8>("IMMA R8 W8 minB2 U2 (16 warps)", out, 2);
    runi<8, 2, 1, 8>("IMMA R8 W8 minB2 U1 (16 warps)", out, 2);
    runi<8, 1, 2, 8>("IMMA R8 W8 minB1 U2 (1 CTA: 8 warps)", out, 1);
    runi<4, 2, 1, 16>("IMMA R16 W4 minB2 U1 (8 warps)", out, 2);
    runi<4, 2, 2, 16>("IMMA R16 W4 minB2 U2 (8 warps)", out, 2);
    runi<4, 2, 1, 16, 2>("IMMA R16 s2 W4 minB2 U1 (8 warps)", out, 2);
    runi<6, 2, 1, 16>("IMMA R16 W6 minB2 U1 (12 warps)", out, 2);
    runi<6, 2, 1, 16, 2>("IMMA R16 s2 W6 minB2 U1 (12 warps)", out, 2);
    runi<8, 1, 1, 16>("IMMA R16 W8 minB1 U1 (8 warps)", out, 1);
    runi<4, 2, 1, 8>("IMMA R8 W4 minB2 U1 (8 warps)", out, 2);
    return 0;
}
