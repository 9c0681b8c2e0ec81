// idg_kernels_tc.cu -- tensor-core sm_100a gridder and degridder (Veenboer et al., IPDPS 2017).
//
// The pixel x visibility phasor contraction of Alg. 1 / Alg. 2 is a dense complex matrix product:
//     gridder    S[pixel][pol]  = sum_v  Phi[pixel][v]     V[v][pol]      (Phi = exp(+i phi))
//     degridder  V[v][pol]      = sum_p  Phi*[v][p]        S[p][pol]
// written as a real product with K = 2 x (visibilities or pixels) and N = 8 = 4 pols x (re, im):
//     A[m][2k] = cos phi, A[m][2k+1] = sin phi;  B[2k][2pol], B[2k+1][2pol], ... encode the complex MAC
// so one warp-level mma.m16n8k16 covers 16 pixels (or visibilities) x 8 visibilities (or pixels) =
// 128 (pixel, visibility) pairs.  The 16 multiply-adds per pair of the paper move to the tensor
// cores; the ALUs keep the phase (1 FMA), the sincos (FMUL + MUFU.SIN + MUFU.COS) and the
// operand split.  Precision: every operand is split into f16 hi + lo (x = hi + lo to ~22 bits) and the
// product is formed as hi*hi + hi*lo + lo*hi with fp32 accumulation (three mma per tile).  f16 range:
// visibilities / subgrid pixels are scaled by a power of two per batch / per item (exact).
//
// Operand layouts (PTX mma.m16n8k16, g = lane/4, q = lane%4):
//   A regs: {A[g][2q..2q+1]}, {A[g+8][2q..]}, {A[g][2q+8..]}, {A[g+8][2q+8..]}  -> thread computes the
//           phasors of (row g, k-slot q), (row g+8, q), (row g, q+4), (row g+8, q+4)
//   B regs: {B[2q..2q+1][g]}, {B[2q+8..2q+9][g]}  -> prepared once per k-block in shared memory
//   D regs: D[g][2q..2q+1], D[g+8][2q..2q+1]      -> (row g, pol q, re/im), (row g+8, pol q, re/im)
#include <cuda_fp16.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstdint>
#include <mutex>
#include <vector>

#include "idg_device.cuh"
#include "idg_internal.h"

namespace idg {
namespace {

using dev::ItemSetup;

__device__ __forceinline__ uint32_t h2_bits(__half2 h) { return *reinterpret_cast<uint32_t *>(&h); }

// Packed f32x2 helpers (sm_100: FFMA2 / FMUL2 / FADD2 execute two fp32 lanes per issue slot).
using f2p = uint64_t;
__device__ __forceinline__ f2p pk(float lo, float hi) {
    f2p r;
    asm("mov.b64 %0, {%1, %2};" : "=l"(r) : "f"(lo), "f"(hi));
    return r;
}
__device__ __forceinline__ f2p dup(float v) { return pk(v, v); }
__device__ __forceinline__ float2 unpk(f2p v) {
    float2 r;
    asm("mov.b64 {%0, %1}, %2;" : "=f"(r.x), "=f"(r.y) : "l"(v));
    return r;
}
__device__ __forceinline__ f2p fma2(f2p a, f2p b, f2p c) {
    f2p r;
    asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(r) : "l"(a), "l"(b), "l"(c));
    return r;
}
__device__ __forceinline__ f2p mul2(f2p a, f2p b) {
    f2p r;
    asm("mul.rn.f32x2 %0, %1, %2;" : "=l"(r) : "l"(a), "l"(b));
    return r;
}
__device__ __forceinline__ f2p sub2(f2p a, f2p b) {
    f2p r;
    asm("sub.rn.f32x2 %0, %1, %2;" : "=l"(r) : "l"(a), "l"(b));
    return r;
}

// (x, y) -> f16x2 hi = rn(x, y) and lo = rn(x - hi, y - hi): x = hi + lo to ~22 significant bits.
// x - hi is one mixed-precision FHFMA per value (fma.rn.f32.f16: hi * -1 + x, f16 operands, f32 result;
// exact, since hi is x rounded), so a split is F2FP + 2 FHFMA + F2FP.  Used for the phasors (per pair, on
// the critical path) and for the B operands (once per batch / item).  For |x| < 2^-14 (f16 subnormal)
// the residual error is below 2^-25.
__device__ __forceinline__ void split2(float x, float y, uint32_t &hi, uint32_t &lo) {
    hi = h2_bits(__floats2half2_rn(x, y));
    float dx, dy;
    asm("{\n.reg .f16 a, b, m;\nmov.b32 {a, b}, %2;\nmov.b16 m, 0xBC00;\n"
        "fma.rn.f32.f16 %0, a, m, %3;\nfma.rn.f32.f16 %1, b, m, %4;\n}"
        : "=f"(dx), "=f"(dy) : "r"(hi), "f"(x), "f"(y));
    lo = h2_bits(__floats2half2_rn(dx, dy));
}
__device__ __forceinline__ void split_phasor(float x, float y, uint32_t &hi, uint32_t &lo) { split2(x, y, hi, lo); }

// Fixed-point phasor split by byte permutation (the degridders' A operand; scripts/split_probe.cu).
// W = fl(sigma z + M) with M = 2^23 + 0x680000 + 2^17 is an fp32 in [2^23, 2^24) (ulp 1), so its bits are
// 0x4B | 0x68 + (X >> 16) | X >> 8 | X (bytes 3..0) with X = 2^17 + rn(sigma z) in [0, 2^18) for |z| <= 1.
// Read as f16: bytes (1, 2) = 2048 + 2 (X >> 8) (binade [2048, 4096), ulp 2) and bytes (0, 3) =
// 14 + (X & 255) / 128 (binade [8, 16), ulp 1/128), so hi + lo = 2062 + X / 128 = kFxOffset + kFxGain z_q
// exactly, z_q = rn(sigma z) / sigma (|z - z_q| <= 2^-18).  One FFMA2 per packed pair + two PRMT per
// phasor replace F2FP + 2 FHFMA + F2FP.  The products hi*(B_hi + B_lo) + lo*B_hi then carry
// kFxOffset * sum_k B_k + kFxLo * sum_k B_lo,k per output column (the same for every visibility), removed
// in the epilogue (degridder_setup_tc computes the column sums); lo*B_lo beyond its constant part is
// <= 2 |B_lo| per term (2^-20 of a term) and dropped.
constexpr float kFxSigma = 130944.0f;     // 2^17 - 128: gain sigma / 128 = 1023
constexpr float kFxMagic = 15335424.0f;   // 2^23 + 0x680000 + 2^17
constexpr float kFxOffset = 3086.0f;      // 2062 + 2^17 / 128
constexpr float kFxLo = 14.0f;            // constant part of lo
constexpr float kFxGain = 1023.0f;
__device__ __forceinline__ uint32_t prmt(float a, float b, uint32_t sel) {
    uint32_t r;
    asm("prmt.b32 %0, %1, %2, %3;" : "=r"(r) : "r"(__float_as_uint(a)), "r"(__float_as_uint(b)), "r"(sel));
    return r;
}
// C = (cos, cos), S = (sin, sin) of the phasors at k-slots q and q+4 (packed): their A registers.
__device__ __forceinline__ void split_fx(f2p C, f2p S, uint32_t &hq, uint32_t &lq, uint32_t &hq4, uint32_t &lq4) {
    const float2 w = unpk(fma2(C, dup(kFxSigma), dup(kFxMagic)));
    const float2 v = unpk(fma2(S, dup(kFxSigma), dup(kFxMagic)));
    hq = prmt(w.x, v.x, 0x6521);
    lq = prmt(w.x, v.x, 0x7430);
    hq4 = prmt(w.y, v.y, 0x6521);
    lq4 = prmt(w.y, v.y, 0x7430);
}

// Integer tensor-core form of the degridder contraction (FX = 2; scripts/split_probe.cu "IMMA").  A phasor
// component z becomes the 16-bit offset fixed-point X = 2^15 + rn(sigma z) held in the low half of
// W = fl(sigma z + 2^23 + 2^15) (fp32 in [2^23, 2^24): ulp 1), i.e. two u8 limbs a_l = X & 255, a_h = X >> 8;
// one PRMT gathers (c_l, c_h, s_l, s_h) of a phasor into the A register of mma.m16n8k32 (u8), one FFMA2
// per packed pair forms W.  The corrected subgrid value x (24-bit signed fixed point, per-item power-of-two
// scale) is three signed-digit s8 limbs x = 2^16 x_h + 2^8 x_m + x_l, and A x = 2^24 a_h x_h +
// 2^16 (a_l x_h + a_h x_m) + 2^8 (a_l x_m + a_h x_l) + a_l x_l: one s32-accumulated mma per weight class
// (B bytes (0, x_h), (x_h, x_m), (x_m, x_l) against (a_l, a_h)), a_l x_l (<= 2^-24 of a term) dropped.
// Integer products and sums are exact; the offset 2^15 sum_k x_k per output column is removed in the
// epilogue.  One PRMT per phasor (the f16 forms need two: the hi and the lo register).
constexpr float kI8Sigma = 32767.0f;
constexpr float kI8Magic = 8421376.0f;    // 2^23 + 2^15
__device__ __forceinline__ void split_i8(f2p C, f2p S, uint32_t &aq, uint32_t &aq4) {
    const float2 w = unpk(fma2(C, dup(kI8Sigma), dup(kI8Magic)));
    const float2 v = unpk(fma2(S, dup(kI8Sigma), dup(kI8Magic)));
    aq = prmt(w.x, v.x, 0x5410);
    aq4 = prmt(w.y, v.y, 0x5410);
}
__device__ __forceinline__ void imma16832(int (&d)[4], const uint32_t (&a)[4], uint32_t b0, uint32_t b1) {
    asm("mma.sync.aligned.m16n8k32.row.col.s32.u8.s8.s32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, {%0,%1,%2,%3};"
        : "+r"(d[0]), "+r"(d[1]), "+r"(d[2]), "+r"(d[3]) : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b0), "r"(b1));
}
// The three weight classes of one tile; bf = {(x_h, x_m) limbs of slots q, q+4, (x_m, x_l) limbs of slots
// q, q+4}, the (0, x_h) class derived from the first by a byte permutation.
__device__ __forceinline__ void imma3(int (&d)[3][4], const uint32_t (&a)[4], const uint4 &bf, uint32_t h0, uint32_t h1) {
    imma16832(d[0], a, h0, h1);
    imma16832(d[1], a, bf.x, bf.y);
    imma16832(d[2], a, bf.z, bf.w);
}
__device__ __forceinline__ uint32_t i8_high_limbs(uint32_t w16) {
    uint32_t r;
    asm("prmt.b32 %0, %1, 0, 0x2404;" : "=r"(r) : "r"(w16));
    return r;
}
// (2^24 d0 + 2^16 d1 + 2^8 d2 - off) inv, exact in fp64 up to the final product
__device__ __forceinline__ float i8_out(const int (&d)[3][4], int j, double off, double inv) {
    const double t = fma(double(d[0][j]), 16777216.0, fma(double(d[1][j]), 65536.0, double(d[2][j]) * 256.0));
    return float((t - off) * inv);
}


__device__ __forceinline__ void mma16816(float (&d)[4], uint32_t a0, uint32_t a1, uint32_t a2, uint32_t a3,
                                         uint32_t b0, uint32_t b1) {
    asm("mma.sync.aligned.m16n8k16.row.col.f32.f16.f16.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, "
        "{%0,%1,%2,%3};"
        : "+f"(d[0]), "+f"(d[1]), "+f"(d[2]), "+f"(d[3])
        : "r"(a0), "r"(a1), "r"(a2), "r"(a3), "r"(b0), "r"(b1));
}

// D = A B (fresh accumulator: C = 0).
__device__ __forceinline__ void mma16816_zero(float (&d)[4], uint32_t a0, uint32_t a1, uint32_t a2, uint32_t a3,
                                              uint32_t b0, uint32_t b1) {
    const float z = 0.0f;
    asm("mma.sync.aligned.m16n8k16.row.col.f32.f16.f16.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, "
        "{%10,%10,%10,%10};"
        : "=f"(d[0]), "=f"(d[1]), "=f"(d[2]), "=f"(d[3])
        : "r"(a0), "r"(a1), "r"(a2), "r"(a3), "r"(b0), "r"(b1), "f"(z));
}

// The three split products of one tile: D += Ahi Bhi + Ahi Blo + Alo Bhi.
__device__ __forceinline__ void mma3(float (&d)[4], const uint32_t (&ah)[4], const uint32_t (&al)[4],
                                     const uint4 &b) {
    mma16816(d, ah[0], ah[1], ah[2], ah[3], b.x, b.y);
    mma16816(d, ah[0], ah[1], ah[2], ah[3], b.z, b.w);
    mma16816(d, al[0], al[1], al[2], al[3], b.x, b.y);
}

// Power-of-two scale s with max * s in [2^13, 2^14) (f16 max is 65504); 1 for max == 0.
__device__ __forceinline__ float pow2_scale(float mx) {
    if (!(mx > 0.0f)) return 1.0f;
    int e = int((__float_as_uint(mx) >> 23) & 0xff) - 127;
    int sexp = min(max(13 - e, -120), 120);
    return __uint_as_float(uint32_t(127 + sexp) << 23);
}

template <int WARPS>
__device__ __forceinline__ float block_max(float v, float *red_s) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v = fmaxf(v, __shfl_xor_sync(0xffffffffu, v, o));
    __syncthreads();
    if ((threadIdx.x & 31) == 0) red_s[threadIdx.x >> 5] = v;
    __syncthreads();
    float m = red_s[0];
#pragma unroll
    for (int w = 1; w < WARPS; ++w) m = fmaxf(m, red_s[w]);
    return m;
}

__device__ __forceinline__ float4 abs_max4(float4 v, float m) {
    return make_float4(fmaxf(m, fmaxf(fmaxf(fabsf(v.x), fabsf(v.y)), fmaxf(fabsf(v.z), fabsf(v.w)))), 0, 0, 0);
}

// ------------------------------------------------------------------------------------------------
// Subgrid DFT on the tensor cores (a4 / a7).  The centred 2-D DFT (R-5) is two passes of a complex
// matrix product with the DFT matrix F[x][k] = exp(sign 2 pi i (k - N~/2)(x - N~/2) / N~):
//     out[r][k] = sum_x in[r][x] F[x][k],   rows r = (pol, a): 4 N~ rows; K = N = N~ complex.
// As a real product (K rows 2x, 2x+1 = re, im of in[.][x]; N columns 2k, 2k+1 = re, im of out[.][k]) it
// is (N~/4) x (N~/4) tiles of mma.m16n8k16 with N~/8 k-steps, split-f16 (hi*hi + hi*lo + lo*hi, fp32
// accumulation) like the contraction; the input is scaled by a power of two into f16 range.  Per
// output and pass this replaces N~ complex MACs on the CUDA cores (2 LDS + 4 FFMA each).
// ------------------------------------------------------------------------------------------------
// B fragments of F: entry (k-step ks, n-tile nt, lane (g, q)) = {hi, hi, lo, lo} of
// (B[2x][n], B[2x+1][n]) for x = 8 ks + q and x + 4, n = 8 nt + g, with B[2x][2k] = Re F,
// B[2x+1][2k] = -Im F, B[2x][2k+1] = Im F, B[2x+1][2k+1] = Re F.  N~^2 entries per subgrid size and
// direction, computed on the host in fp64 once per device (ensure_dft_tables) and read through the
// read-only cache (9 KB for N~ = 24: L1-resident for every CTA).
constexpr int kDftTabEntries = 16 * 16 + 24 * 24 + 32 * 32;
__device__ uint4 g_dft_tab[2][kDftTabEntries];   // [0]: sign -1 (gridding), [1]: sign +1 (degridding)
__host__ __device__ constexpr int dft_tab_offset(int ns) { return ns == 16 ? 0 : ns == 24 ? 256 : 832; }
template <int NS>
__device__ __forceinline__ const uint4 *dft_tab(int sign) {
    return g_dft_tab[sign < 0 ? 0 : 1] + dft_tab_offset(NS);
}

// Copy the table of one direction into shared memory (cp.async, 16 B per thread-op; completes at the
// caller's cp.async.wait_all + barrier).
template <int NS>
__device__ __forceinline__ void dft_tab_to_smem(uint4 *dst, int sign) {
    const uint4 *src = dft_tab<NS>(sign);
    for (int e = threadIdx.x; e < NS * NS; e += blockDim.x) {
        const unsigned d = static_cast<unsigned>(__cvta_generic_to_shared(dst + e));
        asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(d), "l"(src + e) : "memory");
    }
}
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_all;" ::: "memory"); }

// One pass: in[r][x] = src[pol * N~^2 + a * RS + x * KS] for r = pol N~ + a, multiplied by `scale`
// (power of two: f16 range); emit(pol, a, k, out[r][k] * outmul) for every output.  Warps take 16x8
// output tiles round robin.
// NP < 4: the first NP polarisations of src only (rows r = pol N~ + a, pol < NP).
template <int NS, int WARPS, int NP = 4, typename Emit>
__device__ __forceinline__ void dft_pass_tc(const float2 *src, int RS, int KS, const uint4 *tab, float scale,
                                            float outmul, Emit emit) {
    constexpr int NPIX = NS * NS;
    constexpr int MTL = NP * NS / 16, NTL = NS / 4, KST = NS / 8;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, g = lane >> 2, q = lane & 3;
    for (int tile = warp; tile < MTL * NTL; tile += WARPS) {
        const int mt = tile / NTL, nt = tile - mt * NTL;
        const int r0 = mt * 16 + g, r1 = r0 + 8;
        const int p0 = r0 / NS, a0 = r0 - p0 * NS, p1 = r1 / NS, a1 = r1 - p1 * NS;
        const float2 *s0 = src + p0 * NPIX + a0 * RS, *s1 = src + p1 * NPIX + a1 * RS;
        float d[4] = {0.0f, 0.0f, 0.0f, 0.0f};
#pragma unroll
        for (int ks = 0; ks < KST; ++ks) {
            const int x = ks * 8 + q;
            const float2 v00 = s0[x * KS], v10 = s1[x * KS], v01 = s0[(x + 4) * KS], v11 = s1[(x + 4) * KS];
            uint32_t ah[4], al[4];
            split2(v00.x * scale, v00.y * scale, ah[0], al[0]);   // A[g][2q..2q+1]
            split2(v10.x * scale, v10.y * scale, ah[1], al[1]);   // A[g+8][2q..2q+1]
            split2(v01.x * scale, v01.y * scale, ah[2], al[2]);   // A[g][2q+8..2q+9]
            split2(v11.x * scale, v11.y * scale, ah[3], al[3]);   // A[g+8][2q+8..2q+9]
            const uint4 b = tab[(ks * NTL + nt) * 32 + lane];
            mma16816(d, ah[0], ah[1], ah[2], ah[3], b.x, b.y);
            mma16816(d, ah[0], ah[1], ah[2], ah[3], b.z, b.w);
            mma16816(d, al[0], al[1], al[2], al[3], b.x, b.y);
        }
        const int k = nt * 4 + q;
        emit(p0, a0, k, make_float2(d[0] * outmul, d[1] * outmul));
        emit(p1, a1, k, make_float2(d[2] * outmul, d[3] * outmul));
    }
}

// a3 + a4 + a5 with the tensor-core DFT.  On entry (after a barrier) sub_s[pol][pix] holds the raw
// image-domain sums of the item; tmp_s holds 4 N~^2 complex, tab N~^2 uint4 (the DFT table).
template <int NS, int WARPS>
__device__ __forceinline__ void gridder_epilogue_tc(const KernelArgs &a, const ItemSetup &s, float2 *sub_s,
                                                    float2 *tmp_s, uint4 *tab, float *red_s) {
    constexpr int NPIX = NS * NS;
    const idg_metadata &md = s.md;
    dft_tab_to_smem<NS>(tab, -1);
    float mx = 0.0f;
    for (int pix = threadIdx.x; pix < NPIX; pix += WARPS * 32)
        mx = fmaxf(mx, dev::gridder_aterm_pixel<NS>(a, s, sub_s, pix));     // a3
    cp_async_wait_all();
    const float sc = pow2_scale(block_max<WARPS>(mx, red_s));  // (its barriers publish sub_s and tab)
    // a4 rows: T[pol][y][kx] -> tmp_s[pol][kx][y], kept scaled by sc / 32 (|T| <= N~ max|S|)
    dft_pass_tc<NS, WARPS>(sub_s, NS, 1, tab, sc, 1.0f / 32.0f, [&](int pol, int y, int kx, float2 v) {
        tmp_s[pol * NPIX + kx * NS + y] = v;
    });
    __syncthreads();
    // a4 columns + a5: G[pol][ky][kx] = sum_y T[pol][y][kx] F[y][ky], added to the grid
    if (a.subgrids) {   // host adder: the transformed subgrid goes to its slot of the subgrid buffer
        float2 *sp = a.subgrids + int64_t(blockIdx.x) * 4 * NPIX;
        dft_pass_tc<NS, WARPS>(tmp_s, NS, 1, tab, 1.0f, 32.0f / sc, [&](int pol, int kx, int ky, float2 v) {
            sp[(pol * NS + ky) * NS + kx] = v;
        });
        return;
    }
    if (a.bands) {   // banded grid: each element goes to its owner's band (peer memory)
        dft_pass_tc<NS, WARPS>(tmp_s, NS, 1, tab, 1.0f, 32.0f / sc, [&](int pol, int kx, int ky, float2 v) {
            dev::grid_add(a, md.z, pol, md.y + ky, md.x + kx, v);
        });
        __threadfence_system();
        return;
    }
    const int64_t gs = a.grid_size;
    float2 *gp = a.grid + (int64_t(md.z) * 4 * gs + md.y) * gs + md.x;
    dft_pass_tc<NS, WARPS>(tmp_s, NS, 1, tab, 1.0f, 32.0f / sc, [&](int pol, int kx, int ky, float2 v) {
        dev::red_add(gp + (int64_t(pol) * gs + ky) * gs + kx, v);
    });
}

// a6 + a7 with the tensor-core DFT: splitter (grid -> sub_s), centred inverse DFT (columns, then rows);
// on return (after a barrier) sub_s[pol][y][x] holds the image-domain subgrid before a8; tab is N~^2
// uint4 of scratch for the DFT table (dead on return).  `overlap()`
// runs while the splitter's loads are in flight (its shared-memory writes are published by the
// barriers that follow).
template <int NS, int WARPS, typename Overlap>
__device__ __forceinline__ void degridder_prologue_tc(const KernelArgs &a, const ItemSetup &s, float2 *sub_s,
                                                      float2 *tmp_s, uint4 *tab, float *red_s, Overlap overlap) {
    constexpr int NPIX = NS * NS;
    constexpr int NT = WARPS * 32;
    constexpr int PER = (4 * NPIX + NT - 1) / NT;
    const idg_metadata &md = s.md;
    // a6 reads the item's window of the grid, or (host splitter) its slot of the subgrid buffer
    const int64_t gs = a.subgrids ? NS : a.grid_size;
    const float2 *gp = a.subgrids ? a.subgrids + int64_t(blockIdx.x) * 4 * NPIX
                                  : a.grid + (int64_t(md.z) * 4 * gs + md.y) * gs + md.x;
    float2 v[PER];
#pragma unroll
    for (int i = 0; i < PER; ++i) {   // a6: all loads in flight before any use
        const int o = threadIdx.x + i * NT;
        if (o < 4 * NPIX) {
            const int pol = o / NPIX, rem = o - pol * NPIX, ky = rem / NS, kx = rem - ky * NS;
            v[i] = a.bands && !a.subgrids ? *dev::grid_elem(a, md.z, pol, md.y + ky, md.x + kx)   // owner's band
                                          : gp[(int64_t(pol) * gs + ky) * gs + kx];
        }
    }
    dft_tab_to_smem<NS>(tab, +1);
    overlap();
    float mx = 0.0f;
#pragma unroll
    for (int i = 0; i < PER; ++i) {
        const int o = threadIdx.x + i * NT;
        if (o < 4 * NPIX) {
            sub_s[o] = v[i];
            mx = fmaxf(mx, fmaxf(fabsf(v[i].x), fabsf(v[i].y)));
        }
    }
    cp_async_wait_all();
    const float sc = pow2_scale(block_max<WARPS>(mx, red_s));  // (its barriers publish sub_s and tab)
    // a7 columns: rows (pol, kx), K = ky -> tmp_s[pol][y][kx], kept scaled by sc / 32
    dft_pass_tc<NS, WARPS>(sub_s, 1, NS, tab, sc, 1.0f / 32.0f, [&](int pol, int kx, int y, float2 w) {
        tmp_s[pol * NPIX + y * NS + kx] = w;
    });
    __syncthreads();
    // a7 rows: rows (pol, y), K = kx -> sub_s[pol][y][x]
    dft_pass_tc<NS, WARPS>(tmp_s, NS, 1, tab, 1.0f, 32.0f / sc, [&](int pol, int y, int x, float2 w) {
        sub_s[pol * NPIX + y * NS + x] = w;
    });
    __syncthreads();
}

// ------------------------------------------------------------------------------------------------
// Tensor-core gridder.  One CTA per work item; WARPS warps x MT m-tiles x 16 pixels = N~^2.
// k-block = 8 visibilities = 8 consecutive channels of one timestep (requires C~ % 8 == 0).
// ------------------------------------------------------------------------------------------------
constexpr int kTcBatchKB = 64;  // default k-blocks per shared-memory batch (512 visibilities)

inline size_t gridder_tc_smem_bytes(int NS, int max_channels, int kbb_ = kTcBatchKB) {
    const size_t kbb = kbb_;
    const size_t main = kbb * 8 * 32 /*raw*/ + kbb * 32 * 16 /*frag*/ + kbb * 4 * 16 /*df*/ +
                        (kbb + 1) * 32 /*coef*/ + size_t(max_channels) * 4;
    const size_t epi = size_t(2) * 4 * NS * NS * sizeof(float2) + size_t(NS) * NS * 16;  // sub_s, tmp_s, DFT table
    return std::max(main, epi) + 16;
}

// The direct kernel: one sincos per (pixel, visibility) pair, any channel spacing (the fallback of the
// rotation gridder for non-uniform channel tables and items of varying channel counts).
template <int NS, int WARPS, int MT, int MINB, int KBB_ = kTcBatchKB>
__global__ void __launch_bounds__(WARPS * 32, MINB) gridder_tc_kernel(const KernelArgs a) {
    constexpr int NT = WARPS * 32;
    constexpr int NPIX = NS * NS;
    static_assert(WARPS * MT * 16 == NPIX, "warps x m-tiles x 16 must cover the subgrid");
    constexpr int h = NS / 2;
    constexpr int KBB = KBB_;
    constexpr int VB = KBB * 8;
    extern __shared__ __align__(16) unsigned char smem[];
    float4 *raw_s = reinterpret_cast<float4 *>(smem);                // [VB][2]
    uint4 *frag_s = reinterpret_cast<uint4 *>(raw_s + 2 * VB);       // [KBB][32]
    float4 *dfk_s = reinterpret_cast<float4 *>(frag_s + KBB * 32);   // [KBB][4] (df_q, df_q, df_q4, df_q4)
    float4 *coef_s = reinterpret_cast<float4 *>(dfk_s + KBB * 4);    // [KBB+1][2]
    float *df_s = reinterpret_cast<float *>(coef_s + 2 * (KBB + 1)); // [nc]
    __shared__ float red_s[WARPS];

    const int item = a.order[blockIdx.x];
    const ItemSetup s = dev::item_setup(a, item, NS);
    const idg_metadata &md = s.md;
    const int nc = s.nc;
    const int kpt = nc >> 3;                     // k-blocks per timestep
    const int nkb = md.nr_timesteps * kpt;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, g = lane >> 2, q = lane & 3;

    for (int c = threadIdx.x; c < nc; c += NT)
        df_s[c] = float((a.frequencies[md.channel_begin + c] / kSpeedOfLight) - s.f_ref);

    // (l, m, n) of the thread's two rows (pixels g and g+8 of each m-tile), packed as f32x2 pairs
    f2p pl[MT], pm[MT], pn[MT];
    float acc[MT][4];
#pragma unroll
    for (int i = 0; i < MT; ++i) {
        float l2[2], m2[2], n2[2];
#pragma unroll
        for (int r = 0; r < 2; ++r) {
            const int pix = (warp * MT + i) * 16 + g + 8 * r;
            const int x = pix % NS, y = pix / NS;
            l2[r] = float(x - h) * a.cell_l;
            m2[r] = float(y - h) * a.cell_l;
            n2[r] = dev::w_term_n(l2[r], m2[r]);
        }
        pl[i] = pk(l2[0], l2[1]);
        pm[i] = pk(m2[0], m2[1]);
        pn[i] = pk(n2[0], n2[1]);
#pragma unroll
        for (int j = 0; j < 4; ++j) acc[i][j] = 0.0f;
    }
    float cur_scale = 0.0f;

    const int64_t row = int64_t(a.nr_channels) * 4;  // float2 per timestep
    const float2 *vis0 = a.vis + (int64_t(md.baseline) * a.nr_timesteps + md.time_offset) * row +
                         int64_t(md.channel_begin) * 4;

    for (int kb0 = 0; kb0 < nkb; kb0 += KBB) {
        const int kb1 = min(kb0 + KBB, nkb);
        const int nvb = (kb1 - kb0) * 8;
        const int t_first = kb0 / kpt, t_last = (kb1 - 1) / kpt;
        __syncthreads();  // previous batch fully consumed
        // (1) raw visibilities of k-blocks [kb0, kb1)
        for (int i = threadIdx.x; i < 2 * nvb; i += NT) {
            const int j = i >> 1;
            const int kb = kb0 + (j >> 3);
            const int t = kb / kpt;
            const int c = (kb - t * kpt) * 8 + (j & 7);
            raw_s[i] = dev::ld_stream(reinterpret_cast<const float4 *>(vis0 + int64_t(t) * row + c * 4) + (i & 1));
        }
        // (2) per-timestep phase coefficients (fp64 -> fp32)
        for (int t = t_first + int(threadIdx.x); t <= t_last; t += NT) {
            float4 cB, cQ;
            dev::timestep_coefficients(a, s, md.time_offset + t, cB, cQ);
            coef_s[2 * (t - t_first)] = cB;
            coef_s[2 * (t - t_first) + 1] = cQ;
        }
        // (3) channel offsets of the two k-slots q, q+4 of every k-block
        for (int i = threadIdx.x; i < (kb1 - kb0) * 4; i += NT) {
            const int kb = kb0 + (i >> 2);
            const int c = (kb % kpt) * 8 + (i & 3);
            dfk_s[i] = make_float4(df_s[c], df_s[c], df_s[c + 4], df_s[c + 4]);
        }
        __syncthreads();
        // (4) f16 range: power-of-two scale from the batch maximum; never increase the running scale
        float mx = 0.0f;
        for (int i = threadIdx.x; i < 2 * nvb; i += NT) mx = abs_max4(raw_s[i], mx).x;
        // (an all-zero batch, e.g. flagged data, leaves the scale alone: it carries no range information)
        const float bmax = block_max<WARPS>(mx, red_s);
        const float bscale = bmax > 0.0f ? pow2_scale(bmax) : 0.0f;
        if (bscale == 0.0f) {
        } else if (cur_scale == 0.0f) {
            cur_scale = bscale;
        } else if (bscale < cur_scale) {
            const float f = bscale / cur_scale;  // exact power of two
#pragma unroll
            for (int i = 0; i < MT; ++i)
#pragma unroll
                for (int j = 0; j < 4; ++j) acc[i][j] *= f;
            cur_scale = bscale;
        }
        // (5) B fragments: entry (k-block, lane): column g = 2 pol + im, k-slots q and q+4
        for (int i = threadIdx.x; i < (kb1 - kb0) * 32; i += NT) {
            const int kbl = i >> 5, ln = i & 31, gg = ln >> 2, qq = ln & 3;
            const int pol = gg >> 1, im = gg & 1;
            uint32_t hi[2], lo[2];
#pragma unroll
            for (int r = 0; r < 2; ++r) {
                const float4 v4 = raw_s[2 * (kbl * 8 + qq + 4 * r) + (pol >> 1)];
                const float vr = ((pol & 1) ? v4.z : v4.x) * cur_scale;
                const float vi = ((pol & 1) ? v4.w : v4.y) * cur_scale;
                // column 2pol:   rows (cos, sin) -> ( Vre, -Vim );  column 2pol+1: ( Vim, Vre )
                split2(im ? vi : vr, im ? vr : -vi, hi[r], lo[r]);
            }
            frag_s[i] = make_uint4(hi[0], hi[1], lo[0], lo[1]);
        }
        __syncthreads();
        // (6) the contraction: per k-block, MT tiles x (4 phasors + 3 mma) per thread.  Each batch
        //     accumulates into a fresh fragment that is then added in fp32: the tensor-core
        //     accumulation error grows with the batch (512 visibilities), not with the whole item.
        float part[MT][4];
#pragma unroll
        for (int i = 0; i < MT; ++i)
#pragma unroll
            for (int j = 0; j < 4; ++j) part[i][j] = 0.0f;
        for (int t = t_first; t <= t_last; ++t) {
            // B_t, Q_t of both rows of every tile (packed pairs), once per timestep
            const float4 cB = coef_s[2 * (t - t_first)], cQ = coef_s[2 * (t - t_first) + 1];
            f2p Bv[MT], Qv[MT];
#pragma unroll
            for (int i = 0; i < MT; ++i) {
                Bv[i] = fma2(dup(cB.x), pl[i], fma2(dup(cB.y), pm[i], mul2(dup(cB.z), pn[i])));
                Qv[i] = fma2(dup(cQ.x), pl[i], fma2(dup(cQ.y), pm[i], mul2(dup(cQ.z), pn[i])));
            }
            const int k_begin = max(kb0, t * kpt), k_end = min(kb1, (t + 1) * kpt);
#pragma unroll 1
            for (int kb = k_begin; kb < k_end; ++kb) {
                const uint4 bf = frag_s[(kb - kb0) * 32 + lane];
                const float4 df = dfk_s[(kb - kb0) * 4 + q];
                const f2p dq = pk(df.x, df.y), dq4 = pk(df.z, df.w);
                uint32_t ah[MT][4], al[MT][4];
#pragma unroll
                for (int i = 0; i < MT; ++i) {
                    const float2 ph0 = unpk(fma2(dq, Qv[i], Bv[i]));   // (row g, row g+8) at slot q
                    float sn[4], cs[4];
                    __sincosf(ph0.x, &sn[0], &cs[0]);
                    __sincosf(ph0.y, &sn[1], &cs[1]);
                    const float2 ph1 = unpk(fma2(dq4, Qv[i], Bv[i]));  // (row g, row g+8) at slot q+4
                    __sincosf(ph1.x, &sn[2], &cs[2]);
                    __sincosf(ph1.y, &sn[3], &cs[3]);
#pragma unroll
                    for (int j = 0; j < 4; ++j) split_phasor(cs[j], sn[j], ah[i][j], al[i][j]);
                }
                // pass-major issue: consecutive mma are independent (different tiles)
#pragma unroll
                for (int i = 0; i < MT; ++i) mma16816(part[i], ah[i][0], ah[i][1], ah[i][2], ah[i][3], bf.x, bf.y);
#pragma unroll
                for (int i = 0; i < MT; ++i) mma16816(part[i], ah[i][0], ah[i][1], ah[i][2], ah[i][3], bf.z, bf.w);
#pragma unroll
                for (int i = 0; i < MT; ++i) mma16816(part[i], al[i][0], al[i][1], al[i][2], al[i][3], bf.x, bf.y);
            }
        }
#pragma unroll
        for (int i = 0; i < MT; ++i)
#pragma unroll
            for (int j = 0; j < 4; ++j) acc[i][j] += part[i][j];
    }

    // ---- epilogue: D fragments -> sub_s[pol][pixel], then a3 + a4 + a5 ---------------------------
    __syncthreads();
    float2 *sub_s = reinterpret_cast<float2 *>(smem);
    float2 *tmp_s = sub_s + 4 * NPIX;
    const float inv = cur_scale > 0.0f ? 1.0f / cur_scale : 1.0f;
#pragma unroll
    for (int i = 0; i < MT; ++i) {
        const int p0 = (warp * MT + i) * 16 + g;
        sub_s[q * NPIX + p0] = make_float2(acc[i][0] * inv, acc[i][1] * inv);
        sub_s[q * NPIX + p0 + 8] = make_float2(acc[i][2] * inv, acc[i][3] * inv);
    }
    __syncthreads();
    gridder_epilogue_tc<NS, WARPS>(a, s, sub_s, tmp_s, reinterpret_cast<uint4 *>(tmp_s + 4 * NPIX), red_s);
}

inline size_t gridder_rot_smem_bytes(int NS, int kbb_ = kTcBatchKB) {
    const size_t kbb = kbb_;
    const size_t main = kbb * 8 * 32 /*raw*/ + kbb * 32 * 16 /*frag*/ + (kbb + 1) * 32 /*coef*/;
    const size_t epi = size_t(2) * 4 * NS * NS * sizeof(float2) + size_t(NS) * NS * 16;  // sub_s, tmp_s, DFT table
    return std::max(main, epi) + 16;
}

// ------------------------------------------------------------------------------------------------
// gridder_rot2: the rotation gridder with every item holding exactly KPT channel groups (8 KPT
// channels, uniform spacing) and the group step E_t derived from the slot phasors instead of its own
// sincos.  Slots q and q+4 of group 0 are channels 4 apart, so
//     Phi(t, q+4) conj(Phi(t, q)) = exp(i 4 dnu/c Q_t) = E4,   E_t = exp(i 8 dnu/c Q_t) = E4^2
// (two complex products on the FMA pipe, packed over the thread's two pixel rows): the MUFU work per
// (pixel, timestep) is that of the 8 group-0 phasors only (LOFAR: 0.5 sincos per pair, SKA: 0.25).
// The slot phases are formed from per-lane, per-timestep coefficients c_s = B_t + df_s Q_t (3 FFMA2 per
// slot and tile), group 0 accumulates in place, the groups' mma chains are interleaved, and there are
// no runtime channel-group branches.  Exact in exact arithmetic; E carries the rounding of two
// sincos and two complex products (~1e-6 relative), E^j that of j - 1 more products.
// ------------------------------------------------------------------------------------------------
__device__ __forceinline__ f2p add2(f2p a, f2p b) {
    f2p r;
    asm("add.rn.f32x2 %0, %1, %2;" : "=l"(r) : "l"(a), "l"(b));
    return r;
}

// PKR = 1: the rotation of the groups j > 0 on packed f32x2 pairs.  E^j advances for both pixel rows in one
// pair of FFMA2 / FMUL2 (4 instead of 8 scalar instructions), and E^j D_j is accumulated as
// acc += Re(E^j) D_j, acc2 += Im(E^j) D_j on the (re, im) pairs the mma writes (two FFMA2 with a
// broadcast operand instead of four FFMA per pixel row); i acc2 joins acc once per item (complex
// multiplication by i is linear).  The same products, half the instructions of the rotation -- but the
// extra accumulators spill at 64-80 registers: measured LOFAR 32.4 -> 36.6 ms, SKA-T1024 145 -> 157-192 ms
// (sweep r02f), so PKR = 0 stays the default.
// HOR = 1: the rotated groups are summed in Horner form, sum_j E^j D_j = D_0 + E (D_1 + E (D_2 + E D_3)),
// passes in descending group order: one complex multiply-add by E per group (4 FFMA per pixel row) instead
// of advancing E^j (4 FMUL / FFMA) and multiplying by it (4 FFMA).  Same value in exact arithmetic; the
// rounding of J - 1 complex products either way.  Measured (SKA, J = 4): 1162 -> 1125 ms per launch (r02j),
// SKA-T1024 145.2 -> 139.7 ms (nsm) -> 135.6 ms (lmnsm: fewer spills, r02l); for J = 2 both forms are the
// same 4 FFMA per row (predict: equal).
template <int NS, int WARPS, int MT, int MINB, int KPT, int GP, int KBB_ = kTcBatchKB, int TU = 1, int NSM = 0,
          int PKR = 0, int HOR = 0>
__global__ void __launch_bounds__(WARPS * 32, MINB) gridder_rot2_kernel(const KernelArgs a) {
    constexpr int NT = WARPS * 32;
    constexpr int NPIX = NS * NS;
    static_assert(WARPS * MT * 16 == NPIX, "warps x m-tiles x 16 must cover the subgrid");
    static_assert(KPT >= 1 && KPT <= 4 && KBB_ % KPT == 0 && KPT % GP == 0, "channel groups per timestep / pass");
    constexpr int h = NS / 2;
    constexpr int KBB = KBB_;
    constexpr int VB = KBB * 8;
    constexpr int NC = 8 * KPT;                  // channels of every item
    constexpr int TPB = KBB / KPT;               // timesteps per batch
    extern __shared__ __align__(16) unsigned char smem[];
    float4 *raw_s = reinterpret_cast<float4 *>(smem);                // [VB][2]
    uint4 *frag_s = reinterpret_cast<uint4 *>(raw_s + 2 * VB);       // [KBB][32]
    float4 *coef_s = reinterpret_cast<float4 *>(frag_s + KBB * 32);  // [TPB][2]
    f2p *n_s = reinterpret_cast<f2p *>(coef_s + 2 * (KBB + 1));     // NSM: [NPIX / 16][8] n of rows (g, g+8)
    __shared__ float red_s[WARPS];

    const int item = a.order[blockIdx.x];
    const ItemSetup s = dev::item_setup(a, item, NS);
    const idg_metadata &md = s.md;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, g = lane >> 2, q = lane & 3;

    // channel offsets from the reference frequency of slots q and q+4 of group 0
    const float dq = float(a.frequencies[md.channel_begin + q] / kSpeedOfLight - s.f_ref);
    const float dq4 = float(a.frequencies[md.channel_begin + q + 4] / kSpeedOfLight - s.f_ref);

    f2p pl[MT], pm[MT], pn[MT];
    float acc[MT][4];
#pragma unroll
    for (int i = 0; i < MT; ++i) {
        float l2[2], m2[2], n2[2];
#pragma unroll
        for (int r = 0; r < 2; ++r) {
            const int pix = (warp * MT + i) * 16 + g + 8 * r;
            const int x = pix % NS, y = pix / NS;
            l2[r] = float(x - h) * a.cell_l;
            m2[r] = float(y - h) * a.cell_l;
            n2[r] = dev::w_term_n(l2[r], m2[r]);
        }
        pl[i] = pk(l2[0], l2[1]);
        pm[i] = pk(m2[0], m2[1]);
        pn[i] = pk(n2[0], n2[1]);
        // NSM: the w-term n lives in shared memory (8 fewer live registers per tile pair at N~ = 32)
        if (NSM && q == 0) n_s[(warp * MT + i) * 8 + g] = pn[i];
        if (NSM == 2 && q == 0) {   // NSM = 2: l and m as well, after the n pairs: [NPIX / 16][8] {l pair, m pair}
            f2p *lm = n_s + NPIX / 2 + ((warp * MT + i) * 8 + g) * 2;
            lm[0] = pl[i];
            lm[1] = pm[i];
        }
#pragma unroll
        for (int j = 0; j < 4; ++j) acc[i][j] = 0.0f;
    }
    // PKR: the Im(E^j) parts of the rotated groups, per tile and pixel row as (re, im) pairs
    f2p acc2[PKR ? MT : 1][2];
#pragma unroll
    for (int i = 0; i < (PKR ? MT : 1); ++i) acc2[i][0] = acc2[i][1] = 0ull;
    float cur_scale = 0.0f;

    const int64_t row = int64_t(a.nr_channels) * 4;  // float2 per timestep
    const float2 *vis0 = a.vis + (int64_t(md.baseline) * a.nr_timesteps + md.time_offset) * row +
                         int64_t(md.channel_begin) * 4;

    for (int t0 = 0; t0 < md.nr_timesteps; t0 += TPB) {
        const int t1 = min(t0 + TPB, md.nr_timesteps);
        const int nkb = (t1 - t0) * KPT;
        const int nvb = nkb * 8;
        __syncthreads();  // previous batch fully consumed
        // (1) raw visibilities of timesteps [t0, t1): index j = (t - t0) NC + c
        for (int i = threadIdx.x; i < 2 * nvb; i += NT) {
            const int j = i >> 1;
            const int t = j / NC, c = j - t * NC;
            raw_s[i] = dev::ld_stream(reinterpret_cast<const float4 *>(vis0 + int64_t(t0 + t) * row + c * 4) + (i & 1));
        }
        // (2) per-timestep phase coefficients (fp64 -> fp32)
        for (int t = t0 + int(threadIdx.x); t < t1; t += NT) {
            float4 cB, cQ;
            dev::timestep_coefficients(a, s, md.time_offset + t, cB, cQ);
            coef_s[2 * (t - t0)] = cB;
            coef_s[2 * (t - t0) + 1] = cQ;
        }
        __syncthreads();
        // (3) f16 range: power-of-two scale from the batch maximum; never increase the running scale
        float mx = 0.0f;
        for (int i = threadIdx.x; i < 2 * nvb; i += NT) mx = abs_max4(raw_s[i], mx).x;
        // (an all-zero batch, e.g. flagged data, leaves the scale alone: it carries no range information)
        const float bmax = block_max<WARPS>(mx, red_s);
        const float bscale = bmax > 0.0f ? pow2_scale(bmax) : 0.0f;
        if (bscale == 0.0f) {
        } else if (cur_scale == 0.0f) {
            cur_scale = bscale;
        } else if (bscale < cur_scale) {
            const float f = bscale / cur_scale;  // exact power of two
#pragma unroll
            for (int i = 0; i < MT; ++i) {
#pragma unroll
                for (int j = 0; j < 4; ++j) acc[i][j] *= f;
                if constexpr (PKR) {
                    acc2[i][0] = mul2(acc2[i][0], dup(f));
                    acc2[i][1] = mul2(acc2[i][1], dup(f));
                }
            }
            cur_scale = bscale;
        }
        // (4) B fragments of every (timestep, group): column g = 2 pol + im, k-slots q and q+4
        for (int i = threadIdx.x; i < nkb * 32; i += NT) {
            const int kbl = i >> 5, ln = i & 31, gg = ln >> 2, qq = ln & 3;
            const int pol = gg >> 1, im = gg & 1;
            uint32_t hi[2], lo[2];
#pragma unroll
            for (int r = 0; r < 2; ++r) {
                const float4 v4 = raw_s[2 * (kbl * 8 + qq + 4 * r) + (pol >> 1)];
                const float vr = ((pol & 1) ? v4.z : v4.x) * cur_scale;
                const float vi = ((pol & 1) ? v4.w : v4.y) * cur_scale;
                split2(im ? vi : vr, im ? vr : -vi, hi[r], lo[r]);
            }
            frag_s[i] = make_uint4(hi[0], hi[1], lo[0], lo[1]);
        }
        __syncthreads();
        // (5) per timestep: group-0 phasors of every tile, E_t from them, one fresh D_j per group j > 0
#pragma unroll TU
        for (int t = t0; t < t1; ++t) {
            const float4 cB = coef_s[2 * (t - t0)], cQ = coef_s[2 * (t - t0) + 1];
            // slot coefficients c_s = B_t + df_s Q_t (u, v, w components)
            const float c0u = fmaf(dq, cQ.x, cB.x), c0v = fmaf(dq, cQ.y, cB.y), c0w = fmaf(dq, cQ.z, cB.z);
            const float c4u = fmaf(dq4, cQ.x, cB.x), c4v = fmaf(dq4, cQ.y, cB.y), c4w = fmaf(dq4, cQ.z, cB.z);
            const uint4 *fr = frag_s + (t - t0) * KPT * 32 + lane;
#pragma unroll
            for (int i = 0; i < MT; ++i) {
                uint4 bf0[GP];   // B fragments of the first pass, loaded ahead of the sincos
                constexpr int FIRST = HOR ? KPT - GP : 0;
#pragma unroll
                for (int j = 0; j < GP; ++j) bf0[j] = fr[(FIRST + j) * 32];
                f2p nv = pn[i], lv = pl[i], mv = pm[i];
                if constexpr (NSM) {
                    // re-read every timestep (volatile: not hoisted into registers, which is the point)
                    const uint32_t addr = uint32_t(__cvta_generic_to_shared(n_s + (warp * MT + i) * 8 + g));
                    asm volatile("ld.shared.b64 %0, [%1];" : "=l"(nv) : "r"(addr));
                    if constexpr (NSM == 2) {
                        const uint32_t a2 = uint32_t(__cvta_generic_to_shared(n_s + NPIX / 2 + ((warp * MT + i) * 8 + g) * 2));
                        asm volatile("ld.shared.v2.b64 {%0, %1}, [%2];" : "=l"(lv), "=l"(mv) : "r"(a2));
                    }
                }
                const float2 ph0 = unpk(fma2(dup(c0u), lv, fma2(dup(c0v), mv, mul2(dup(c0w), nv))));
                const float2 ph1 = unpk(fma2(dup(c4u), lv, fma2(dup(c4v), mv, mul2(dup(c4w), nv))));
                float sn[4], cs[4];
                __sincosf(ph0.x, &sn[0], &cs[0]);   // row g,   slot q
                __sincosf(ph0.y, &sn[1], &cs[1]);   // row g+8, slot q
                __sincosf(ph1.x, &sn[2], &cs[2]);   // row g,   slot q+4
                __sincosf(ph1.y, &sn[3], &cs[3]);   // row g+8, slot q+4
                uint32_t ah[4], al[4];
#pragma unroll
                for (int j = 0; j < 4; ++j) split_phasor(cs[j], sn[j], ah[j], al[j]);
                if constexpr (KPT == 1) {
                    mma3(acc[i], ah, al, bf0[0]);
                } else if constexpr (HOR) {
                    float2 er = make_float2(1.0f, 1.0f), ei = make_float2(0.0f, 0.0f);   // E_t of rows (g, g+8)
                    float h[4];   // Horner sum of the groups j >= 1: rows g (h0, h1) and g+8 (h2, h3)
#pragma unroll
                    for (int p0 = KPT - GP; p0 >= 0; p0 -= GP) {
                        uint4 bf[GP];
                        float d[GP][4];
#pragma unroll
                        for (int j = 0; j < GP; ++j) bf[j] = p0 == KPT - GP ? bf0[j] : fr[(p0 + j) * 32];
#pragma unroll
                        for (int k = 0; k < 3; ++k) {
                            const uint32_t *A = k < 2 ? ah : al;
#pragma unroll
                            for (int j = 0; j < GP; ++j) {
                                const uint32_t b0 = k == 1 ? bf[j].z : bf[j].x, b1 = k == 1 ? bf[j].w : bf[j].y;
                                if (p0 + j == 0)
                                    mma16816(acc[i], A[0], A[1], A[2], A[3], b0, b1);
                                else if (k == 0)
                                    mma16816_zero(d[j], A[0], A[1], A[2], A[3], b0, b1);
                                else
                                    mma16816(d[j], A[0], A[1], A[2], A[3], b0, b1);
                            }
                        }
                        if (p0 == KPT - GP) {
                            // E4 = Phi(q+4) conj(Phi(q)), E = E4^2, packed over rows (g, g+8)
                            const f2p C0 = pk(cs[0], cs[1]), S0 = pk(sn[0], sn[1]);
                            const f2p C4 = pk(cs[2], cs[3]), S4 = pk(sn[2], sn[3]);
                            const f2p r4 = fma2(C4, C0, mul2(S4, S0));
                            const f2p i4 = sub2(mul2(S4, C0), mul2(C4, S0));
                            er = unpk(sub2(mul2(r4, r4), mul2(i4, i4)));
                            ei = unpk(mul2(add2(r4, r4), i4));
                        }
#pragma unroll
                        for (int j = GP - 1; j >= 0; --j) {
                            if (p0 + j == 0) continue;
                            if (p0 + j == KPT - 1) {
#pragma unroll
                                for (int k = 0; k < 4; ++k) h[k] = d[j][k];
                            } else {   // h = D_j + E h
                                const float h0 = fmaf(er.x, h[0], fmaf(-ei.x, h[1], d[j][0]));
                                const float h1 = fmaf(er.x, h[1], fmaf(ei.x, h[0], d[j][1]));
                                const float h2 = fmaf(er.y, h[2], fmaf(-ei.y, h[3], d[j][2]));
                                const float h3 = fmaf(er.y, h[3], fmaf(ei.y, h[2], d[j][3]));
                                h[0] = h0; h[1] = h1; h[2] = h2; h[3] = h3;
                            }
                        }
                    }
                    // acc += E h (group 0 was accumulated in place by its mma)
                    acc[i][0] = fmaf(er.x, h[0], fmaf(-ei.x, h[1], acc[i][0]));
                    acc[i][1] = fmaf(er.x, h[1], fmaf(ei.x, h[0], acc[i][1]));
                    acc[i][2] = fmaf(er.y, h[2], fmaf(-ei.y, h[3], acc[i][2]));
                    acc[i][3] = fmaf(er.y, h[3], fmaf(ei.y, h[2], acc[i][3]));
                } else {
                    float2 er, ei;   // E_t of rows (g, g+8)
                    float pr0 = 1.0f, pi0 = 0.0f, pr1 = 1.0f, pi1 = 0.0f;   // E^j of rows g, g+8
                    f2p ER = 0, EI = 0, PR = 0, PI = 0;                    // PKR: the same packed over the rows
                    // groups in passes of GP: interleaved mma chains, group 0 into the accumulator,
                    // groups j > 0 fresh and rotated by E^j
#pragma unroll
                    for (int p0 = 0; p0 < KPT; p0 += GP) {
                        uint4 bf[GP];
                        float d[GP][4];
#pragma unroll
                        for (int j = 0; j < GP; ++j) bf[j] = p0 == 0 ? bf0[j] : fr[(p0 + j) * 32];
#pragma unroll
                        for (int k = 0; k < 3; ++k) {
                            const uint32_t *A = k < 2 ? ah : al;
#pragma unroll
                            for (int j = 0; j < GP; ++j) {
                                const uint32_t b0 = k == 1 ? bf[j].z : bf[j].x, b1 = k == 1 ? bf[j].w : bf[j].y;
                                if (p0 + j == 0)
                                    mma16816(acc[i], A[0], A[1], A[2], A[3], b0, b1);
                                else if (k == 0)
                                    mma16816_zero(d[j], A[0], A[1], A[2], A[3], b0, b1);
                                else
                                    mma16816(d[j], A[0], A[1], A[2], A[3], b0, b1);
                            }
                        }
                        if (p0 == 0) {
                            // E4 = Phi(q+4) conj(Phi(q)), E = E4^2, packed over rows (g, g+8)
                            const f2p C0 = pk(cs[0], cs[1]), S0 = pk(sn[0], sn[1]);
                            const f2p C4 = pk(cs[2], cs[3]), S4 = pk(sn[2], sn[3]);
                            const f2p r4 = fma2(C4, C0, mul2(S4, S0));
                            const f2p i4 = sub2(mul2(S4, C0), mul2(C4, S0));
                            ER = sub2(mul2(r4, r4), mul2(i4, i4));
                            EI = mul2(add2(r4, r4), i4);
                            er = unpk(ER);
                            ei = unpk(EI);
                        }
#pragma unroll
                        for (int j = 0; j < GP; ++j) {
                            if (p0 + j == 0) continue;
                            if constexpr (PKR) {
                                if (p0 + j == 1) {
                                    PR = ER;
                                    PI = EI;
                                } else {   // E^j = E^(j-1) E for both rows
                                    const f2p nr = fma2(PR, ER, mul2(PI, sub2(0ull, EI)));
                                    PI = fma2(PR, EI, mul2(PI, ER));
                                    PR = nr;
                                }
                                const float2 pr = unpk(PR), pi = unpk(PI);
                                f2p a0 = pk(acc[i][0], acc[i][1]), a1 = pk(acc[i][2], acc[i][3]);
                                const f2p d0 = pk(d[j][0], d[j][1]), d1 = pk(d[j][2], d[j][3]);
                                a0 = fma2(dup(pr.x), d0, a0);               // row g:   Re(E^j) D
                                a1 = fma2(dup(pr.y), d1, a1);               // row g+8
                                acc2[i][0] = fma2(dup(pi.x), d0, acc2[i][0]);  // Im(E^j) D
                                acc2[i][1] = fma2(dup(pi.y), d1, acc2[i][1]);
                                const float2 u0 = unpk(a0), u1 = unpk(a1);
                                acc[i][0] = u0.x; acc[i][1] = u0.y; acc[i][2] = u1.x; acc[i][3] = u1.y;
                                continue;
                            }
                            if (p0 + j == 1) {
                                pr0 = er.x; pi0 = ei.x; pr1 = er.y; pi1 = ei.y;
                            } else {
                                const float a0 = fmaf(pr0, er.x, -pi0 * ei.x), b0 = fmaf(pr0, ei.x, pi0 * er.x);
                                const float a1 = fmaf(pr1, er.y, -pi1 * ei.y), b1 = fmaf(pr1, ei.y, pi1 * er.y);
                                pr0 = a0; pi0 = b0; pr1 = a1; pi1 = b1;
                            }
                            acc[i][0] = fmaf(pr0, d[j][0], fmaf(-pi0, d[j][1], acc[i][0]));
                            acc[i][1] = fmaf(pr0, d[j][1], fmaf(pi0, d[j][0], acc[i][1]));
                            acc[i][2] = fmaf(pr1, d[j][2], fmaf(-pi1, d[j][3], acc[i][2]));
                            acc[i][3] = fmaf(pr1, d[j][3], fmaf(pi1, d[j][2], acc[i][3]));
                        }
                    }
                }
            }
        }
    }

    // ---- epilogue: D fragments -> sub_s[pol][pixel], then a3 + a4 + a5 ---------------------------
    __syncthreads();
    float2 *sub_s = reinterpret_cast<float2 *>(smem);
    float2 *tmp_s = sub_s + 4 * NPIX;
    const float inv = cur_scale > 0.0f ? 1.0f / cur_scale : 1.0f;
#pragma unroll
    for (int i = 0; i < MT; ++i) {
        if constexpr (PKR) {   // acc + i acc2
            const float2 b0 = unpk(acc2[i][0]), b1 = unpk(acc2[i][1]);
            acc[i][0] -= b0.y; acc[i][1] += b0.x; acc[i][2] -= b1.y; acc[i][3] += b1.x;
        }
        const int p0 = (warp * MT + i) * 16 + g;
        sub_s[q * NPIX + p0] = make_float2(acc[i][0] * inv, acc[i][1] * inv);
        sub_s[q * NPIX + p0 + 8] = make_float2(acc[i][2] * inv, acc[i][3] * inv);
    }
    __syncthreads();
    gridder_epilogue_tc<NS, WARPS>(a, s, sub_s, tmp_s, reinterpret_cast<uint4 *>(tmp_s + 4 * NPIX), red_s);
}

// ------------------------------------------------------------------------------------------------
// Tensor-core degridder.  One CTA per work item.  Prologue (a6-a8) leaves the corrected subgrid as
// B fragments (k-block = 8 pixels) + per-pixel {l, m, n}; m-tile = 16 consecutive visibilities of
// the item (flattened (t, c) order); each warp takes MT tiles at a time over all k-blocks.
// ------------------------------------------------------------------------------------------------
inline size_t degridder_tc_smem_bytes(int NS, int max_timesteps, int max_channels) {
    const size_t npix = size_t(NS) * NS;
    return npix * 64 /*sub+tmp | frag*/ + npix * 4 * 8 / 2 /*lmn slot pairs: 32 B per 2 pixels*/ +
           size_t(max_timesteps) * 32 /*B_t, Q_t of the item's timesteps*/ + size_t(max_channels) * 4 /*df*/ + 16;
}

// Shared-memory layout of the tensor-core degridders (bytes: degridder_tc_smem_bytes).
template <int NS>
struct DegridSmem {
    static constexpr int NPIX = NS * NS, NKB = NPIX / 8;
    float2 *sub_s, *tmp_s;   // [4][NS][NS] each (prologue)
    uint4 *frag_s;           // [NKB][32] B fragments (after the prologue; aliases sub_s / tmp_s)
    float4 *lmn_s;           // [NKB][4][2] slot pairs {l_q, l_q4, m_q, m_q4}, {n_q, n_q4, 0, 0}
    float4 *bq_s;            // [T~][2]: B_t, Q_t of the item
    float *df_s;             // [C~]: nu/c - f_ref
    __device__ DegridSmem(unsigned char *smem, int max_timesteps) {
        sub_s = reinterpret_cast<float2 *>(smem);
        tmp_s = sub_s + 4 * NPIX;
        frag_s = reinterpret_cast<uint4 *>(smem);
        lmn_s = reinterpret_cast<float4 *>(smem + size_t(NPIX) * 64);
        bq_s = lmn_s + NKB * 8;
        df_s = reinterpret_cast<float *>(bq_s + 2 * max_timesteps);
    }
};

// Degridder prologue shared by the tensor-core degridders: per-timestep phase coefficients, a6 + a7
// (tensor-core DFT), a8 per pixel, and the corrected subgrid as split B fragments (k-block = 8 pixels)
// + per-pixel {l, m, n}.  Ends with a barrier; returns 1 / (the power-of-two f16 range scale).
// off_s (optional, [8 (WARPS + 1)], the tail is scratch): per B column n, kFxOffset * sum_k (B_hi + B_lo)[k][n] - kFxLo * sum_k B_lo[k][n]
// over the item's K rows -- the constant the fixed-point A operand adds to every output of column n.
// BM = 1: the B fragments as the s8 limbs of the integer form (FX = 2) instead: per (k-block, lane)
// {(x_h, x_m) of slot q, of q+4, (x_m, x_l) of slot q, of q+4}; off_s (16-byte aligned, 16 (WARPS + 1) + 8
// floats) gets 2^15 sum_k x[k][n] as doubles at double index n (the per-warp scratch follows them);
// returns 1 / (scale sigma).
template <int NS, int WARPS, int BM = 0>
__device__ __forceinline__ float degridder_setup_tc(const KernelArgs &a, const ItemSetup &s, const DegridSmem<NS> &sm,
                                                    float *red_s, float *off_s = nullptr) {
    constexpr int NT = WARPS * 32;
    constexpr int NPIX = NS * NS;
    constexpr int PPT = (NPIX + NT - 1) / NT;
    constexpr int h = NS / 2;
    const idg_metadata &md = s.md;
    const int nc = s.nc;
    // per-timestep phase coefficients B_t = 2 pi (uvw_t f_ref - uvw0), Q_t = 2 pi uvw_t (fp64 -> fp32,
    // once per item) and channel offsets df_c = nu_c/c - f_ref: a visibility's coefficients are then
    // B_t + df_c Q_t (fp32 FMAs, as in the gridder), with no fp64 work in front of each tile
    for (int t = threadIdx.x; t < md.nr_timesteps; t += NT) {
        float4 cB, cQ;
        dev::timestep_coefficients(a, s, md.time_offset + t, cB, cQ);
        sm.bq_s[2 * t] = cB;
        sm.bq_s[2 * t + 1] = cQ;
    }
    for (int c = threadIdx.x; c < nc; c += NT)
        sm.df_s[c] = float(a.frequencies[md.channel_begin + c] / kSpeedOfLight - s.f_ref);
    // a6 + a7 (tensor-core DFT; its table aliases lmn_s, written only after it)
    degridder_prologue_tc<NS, WARPS>(a, s, sm.sub_s, sm.tmp_s, reinterpret_cast<uint4 *>(sm.lmn_s), red_s, [] {});
    float2 rr[PPT][4];
    float mx = 0.0f;
#pragma unroll
    for (int i = 0; i < PPT; ++i) {
        const int pix = threadIdx.x + i * NT;
        if (pix < NPIX) {
            const float2 sv[4] = {sm.sub_s[pix], sm.sub_s[NPIX + pix], sm.sub_s[2 * NPIX + pix], sm.sub_s[3 * NPIX + pix]};
            dev::degridder_aterm_pixel<NS>(a, s, sv, pix, rr[i]);   // a8
#pragma unroll
            for (int p = 0; p < 4; ++p) mx = fmaxf(mx, fmaxf(fabsf(rr[i][p].x), fabsf(rr[i][p].y)));
            const int y = pix / NS, x = pix - y * NS;
            const float l = float(x - h) * a.cell_l, m = float(y - h) * a.cell_l;
            // slot pair (q, q+4) of k-block kb: {l_q, l_q4, m_q, m_q4}, {n_q, n_q4, 0, 0}
            const int kb = pix >> 3, slot = pix & 7, half = slot >> 2;
            float *rec = reinterpret_cast<float *>(sm.lmn_s + (kb * 4 + (slot & 3)) * 2);
            rec[half] = l;
            rec[2 + half] = m;
            rec[4 + half] = dev::w_term_n(l, m);
            rec[6 + half] = 0.0f;
        }
    }
    if constexpr (BM == 1) {
        // integer limbs: x = rn(value * scale) with max |x| in [2^21, 2^22) (power of two: exact scaling)
        const float bmx = block_max<WARPS>(mx, red_s);
        float scale = 1.0f;
        if (bmx > 0.0f) {
            const int e = int((__float_as_uint(bmx) >> 23) & 0xff) - 127;
            scale = __uint_as_float(uint32_t(127 + min(max(21 - e, -120), 120)) << 23);
        }
        uint32_t *frag_w = reinterpret_cast<uint32_t *>(sm.frag_s);
        double colx[8];
#pragma unroll
        for (int gg = 0; gg < 8; ++gg) colx[gg] = 0.0;
        auto limbs = [](int x, int &h, int &m, int &l) {   // signed digits, x = 2^16 h + 2^8 m + l
            l = ((x + 128) & 255) - 128;
            const int y = (x - l) >> 8;
            m = ((y + 128) & 255) - 128;
            h = (y - m) >> 8;
        };
#pragma unroll
        for (int i = 0; i < PPT; ++i) {
            const int pix = threadIdx.x + i * NT;
            if (pix < NPIX) {
                const int kb = pix >> 3, slot = pix & 7, qq = slot & 3, half = slot >> 2;
#pragma unroll
                for (int gg = 0; gg < 8; ++gg) {
                    const int pol = gg >> 1;
                    const int xr = __float2int_rn(rr[i][pol].x * scale), xi = __float2int_rn(rr[i][pol].y * scale);
                    // column 2pol: (cos, sin) rows -> (Sre, Sim); column 2pol+1 -> (Sim, -Sre)
                    const int xc = (gg & 1) ? xi : xr, xs = (gg & 1) ? -xr : xi;
                    int ch, cm, cl, sh, sm_, sl;
                    limbs(xc, ch, cm, cl);
                    limbs(xs, sh, sm_, sl);
                    const int e = (kb * 32 + gg * 4 + qq) * 4;
                    frag_w[e + half] = (uint32_t(ch) & 255u) | (uint32_t(cm) & 255u) << 8 | (uint32_t(sh) & 255u) << 16 |
                                       (uint32_t(sm_) & 255u) << 24;
                    frag_w[e + 2 + half] = (uint32_t(cm) & 255u) | (uint32_t(cl) & 255u) << 8 | (uint32_t(sm_) & 255u) << 16 |
                                           (uint32_t(sl) & 255u) << 24;
                    colx[gg] += double(xc) + double(xs);
                }
            }
        }
        double *offd = reinterpret_cast<double *>(off_s);   // [8] results, then [WARPS][8] scratch
        double *red_d = offd + 8;
#pragma unroll
        for (int gg = 0; gg < 8; ++gg) {
            double v = colx[gg];
#pragma unroll
            for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
            if ((threadIdx.x & 31) == 0) red_d[8 * (threadIdx.x >> 5) + gg] = v;
        }
        __syncthreads();
        if (threadIdx.x < 8) {
            double v = 0.0;
            for (int w = 0; w < WARPS; ++w) v += red_d[8 * w + threadIdx.x];
            offd[threadIdx.x] = 32768.0 * v;
        }
        __syncthreads();
        return float(1.0 / (double(scale) * double(kI8Sigma)));
    }
    const float scale = pow2_scale(block_max<WARPS>(mx, red_s));  // barriers: sub_s reads are done
    uint32_t *frag_w = reinterpret_cast<uint32_t *>(sm.frag_s);
    float colb[8], coll[8];   // this thread's part of the column sums of B_hi + B_lo and of B_lo (off_s)
#pragma unroll
    for (int gg = 0; gg < 8; ++gg) colb[gg] = coll[gg] = 0.0f;
#pragma unroll
    for (int i = 0; i < PPT; ++i) {
        const int pix = threadIdx.x + i * NT;
        if (pix < NPIX) {
            const int kb = pix >> 3, slot = pix & 7, qq = slot & 3, half = slot >> 2;
#pragma unroll
            for (int gg = 0; gg < 8; ++gg) {
                const int pol = gg >> 1;
                const float sr = rr[i][pol].x * scale, si = rr[i][pol].y * scale;
                uint32_t hi, lo;
                // V += S exp(-i phi): column 2pol rows (cos, sin) -> (Sre, Sim); column 2pol+1 -> (Sim, -Sre)
                split2((gg & 1) ? si : sr, (gg & 1) ? -sr : si, hi, lo);
                const int e = (kb * 32 + gg * 4 + qq) * 4;
                frag_w[e + half] = hi;
                frag_w[e + 2 + half] = lo;
                if (off_s) {
                    const float2 fh = __half22float2(*reinterpret_cast<const __half2 *>(&hi));
                    const float2 fl = __half22float2(*reinterpret_cast<const __half2 *>(&lo));
                    coll[gg] += fl.x + fl.y;
                    colb[gg] += (fh.x + fh.y) + (fl.x + fl.y);
                }
            }
        }
    }
    if (off_s) {
        // deterministic block sums of the column partials: warp shuffles, then per-warp rows off_s[8 + 8 w]
        // summed in warp order
#pragma unroll
        for (int gg = 0; gg < 8; ++gg) {
            float v = kFxOffset * colb[gg] - kFxLo * coll[gg];
#pragma unroll
            for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
            if ((threadIdx.x & 31) == 0) off_s[8 + 8 * (threadIdx.x >> 5) + gg] = v;
        }
        __syncthreads();
        if (threadIdx.x < 8) {
            float v = 0.0f;
            for (int w = 0; w < WARPS; ++w) v += off_s[8 + 8 * w + threadIdx.x];
            off_s[threadIdx.x] = v;
        }
    }
    __syncthreads();
    return __frcp_rn(scale);
}

// FX: the A operand, 1: fixed-point f16 split (split_fx), 2: the integer form (split_i8 + imma3).
template <int NS, int WARPS, int MT, int MINB, int FX = 1>
__global__ void __launch_bounds__(WARPS * 32, MINB) degridder_tc_kernel(const KernelArgs a) {
    constexpr int NPIX = NS * NS;
    constexpr int NKB = NPIX / 8;
    static_assert(NPIX % 8 == 0, "pixels per k-block");
    static_assert(FX == 1 || FX == 2, "A operand form");
    extern __shared__ __align__(16) unsigned char smem[];
    const DegridSmem<NS> sm(smem, a.max_timesteps_in_item);
    const uint4 *frag_s = sm.frag_s;
    const float4 *lmn_s = sm.lmn_s, *bq_s = sm.bq_s;
    const float *df_s = sm.df_s;
    __shared__ float red_s[WARPS];
    __shared__ __align__(16) float off_s[FX == 2 ? 16 * (WARPS + 1) : 8 * (WARPS + 1)];

    const int item = a.order[blockIdx.x];
    const ItemSetup s = dev::item_setup(a, item, NS);
    const idg_metadata &md = s.md;
    const int nc = s.nc;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, g = lane >> 2, q = lane & 3;
    // fixed-point A operand: output = (acc - column offset) * inv
    const float inv0 = degridder_setup_tc<NS, WARPS, FX == 2 ? 1 : 0>(a, s, sm, red_s, off_s);
    const float inv = FX == 1 ? inv0 * (1.0f / kFxGain) : inv0;
    const float off0 = FX == 1 ? off_s[2 * q] : 0.0f, off1 = FX == 1 ? off_s[2 * q + 1] : 0.0f;
    const double *offd = reinterpret_cast<const double *>(off_s);   // FX = 2
    const double ioff0 = FX == 2 ? offd[2 * q] : 0.0, ioff1 = FX == 2 ? offd[2 * q + 1] : 0.0;

    const int nvis = md.nr_timesteps * nc;
    const int ntiles = (nvis + 15) >> 4;
    // t = v / nc without an integer division: (v + 1/2) / nc is at least 1/(2 nc) away from an integer,
    // and the fp32 quotient's error (v / nc) 2^-23 is smaller for v < 2^22 (else: integer division)
    const float rnc = __frcp_rn(float(nc));
    const bool fdiv = nvis < (1 << 22);
    auto tstep = [&](int v) { return fdiv ? __float2int_rz((float(v) + 0.5f) * rnc) : v / nc; };
    const int64_t row = int64_t(a.nr_channels) * 4;
    float2 *vis0 = a.vis + (int64_t(md.baseline) * a.nr_timesteps + md.time_offset) * row +
                   int64_t(md.channel_begin) * 4;
    for (int tile0 = warp * MT; tile0 < ntiles; tile0 += WARPS * MT) {
        f2p cu[MT][2], cv[MT][2], cw[MT][2];  // (coefficient, coefficient) pairs of rows g and g+8
        float acc[FX == 2 ? 1 : MT][4];
        int iacc[FX == 2 ? MT : 1][3][4];
#pragma unroll
        for (int i = 0; i < MT; ++i) {
#pragma unroll
            for (int r = 0; r < 2; ++r) {
                const int v = (tile0 + i) * 16 + g + 8 * r;
                float fu = 0.0f, fv = 0.0f, fw = 0.0f;
                if (v < nvis) {
                    const int t = tstep(v), c = v - t * nc;
                    const float4 cB = bq_s[2 * t], cQ = bq_s[2 * t + 1];
                    const float df = df_s[c];
                    fu = fmaf(df, cQ.x, cB.x);
                    fv = fmaf(df, cQ.y, cB.y);
                    fw = fmaf(df, cQ.z, cB.z);
                }
                cu[i][r] = dup(fu);
                cv[i][r] = dup(fv);
                cw[i][r] = dup(fw);
            }
#pragma unroll
            for (int j = 0; j < 4; ++j) {
                if constexpr (FX == 2) {
                    iacc[i][0][j] = iacc[i][1][j] = iacc[i][2][j] = 0;
                } else {
                    acc[i][j] = 0.0f;
                }
            }
        }
#pragma unroll 1
        for (int kb = 0; kb < NKB; ++kb) {
            const uint4 bf = frag_s[kb * 32 + lane];
            const float4 lm = lmn_s[(kb * 4 + q) * 2], nn = lmn_s[(kb * 4 + q) * 2 + 1];
            const f2p l2 = pk(lm.x, lm.y), m2 = pk(lm.z, lm.w), n2 = pk(nn.x, nn.y);
            uint32_t ah[MT][4], al[MT][4];
#pragma unroll
            for (int i = 0; i < MT; ++i) {
                // phases of (row, slot q) and (row, slot q+4) in one FFMA2 chain per row
                const float2 p0 = unpk(fma2(cu[i][0], l2, fma2(cv[i][0], m2, mul2(cw[i][0], n2))));
                const float2 p1 = unpk(fma2(cu[i][1], l2, fma2(cv[i][1], m2, mul2(cw[i][1], n2))));
                float sn[4], cs[4];
                __sincosf(p0.x, &sn[0], &cs[0]);  // row g,   slot q
                __sincosf(p0.y, &sn[2], &cs[2]);  // row g,   slot q+4
                __sincosf(p1.x, &sn[1], &cs[1]);  // row g+8, slot q
                __sincosf(p1.y, &sn[3], &cs[3]);  // row g+8, slot q+4
                if constexpr (FX == 2) {
                    split_i8(pk(cs[0], cs[1]), pk(sn[0], sn[1]), ah[i][0], ah[i][1]);
                    split_i8(pk(cs[2], cs[3]), pk(sn[2], sn[3]), ah[i][2], ah[i][3]);
                } else {
                    split_fx(pk(cs[0], cs[1]), pk(sn[0], sn[1]), ah[i][0], al[i][0], ah[i][1], al[i][1]);
                    split_fx(pk(cs[2], cs[3]), pk(sn[2], sn[3]), ah[i][2], al[i][2], ah[i][3], al[i][3]);
                }
            }
            if constexpr (FX == 2) {
                const uint32_t bh0 = i8_high_limbs(bf.x), bh1 = i8_high_limbs(bf.y);
#pragma unroll
                for (int i = 0; i < MT; ++i) imma3(iacc[i], ah[i], bf, bh0, bh1);
            } else {
#pragma unroll
                for (int i = 0; i < MT; ++i) mma16816(acc[i], ah[i][0], ah[i][1], ah[i][2], ah[i][3], bf.x, bf.y);
#pragma unroll
                for (int i = 0; i < MT; ++i) mma16816(acc[i], ah[i][0], ah[i][1], ah[i][2], ah[i][3], bf.z, bf.w);
#pragma unroll
                for (int i = 0; i < MT; ++i) mma16816(acc[i], al[i][0], al[i][1], al[i][2], al[i][3], bf.x, bf.y);
            }
        }
#pragma unroll
        for (int i = 0; i < MT; ++i) {
#pragma unroll
            for (int r = 0; r < 2; ++r) {
                const int v = (tile0 + i) * 16 + g + 8 * r;
                if (v < nvis) {
                    const int t = tstep(v), c = v - t * nc;
                    if constexpr (FX == 2) {
                        vis0[int64_t(t) * row + c * 4 + q] = make_float2(i8_out(iacc[i], 2 * r, ioff0, double(inv)),
                                                                         i8_out(iacc[i], 2 * r + 1, ioff1, double(inv)));
                    } else {
                        vis0[int64_t(t) * row + c * 4 + q] =
                            make_float2((acc[i][2 * r] - off0) * inv, (acc[i][2 * r + 1] - off1) * inv);
                    }
                }
            }
        }
    }
}

// ------------------------------------------------------------------------------------------------
// Tensor-core degridder with phasor rotation across channel groups (uniform channels, C~ % 32 == 0).
// A warp takes 32 channels of one timestep as two m-tiles, so each thread's four A rows are the
// channels c0 + g + 8r (r = 0..3) of the same timestep.  With the phase linear in frequency,
//     Phi(t, c + 8r, p) = Phi(t, c, p) E_tp^r,    E_tp = exp(i 8 dnu/c Q_t(p))
// so per pixel slot the thread evaluates two sincos (row 0 and E) instead of four and forms rows
// 1..3 by complex products (fp32, on the FMA pipe) before the operand split.  Exact in exact
// arithmetic; the rounding is that of up to three extra complex products per phasor.
// ------------------------------------------------------------------------------------------------
// SCH (R = 8, 16): issue schedule of the k-block loop.  0: per tile, its rows' rotation + split, then its
// three products.  2: two independent rotation chains (rows 0..R/2-1 from row 0, rows R/2..R-1 from row
// R/2, which gets its own sincos) advanced in alternation: half the dependent-chain length for one more
// sincos pair per k-block (measured: N~ = 32 SKA 2140 -> 2186 MVis/s, predict +0.5%; N~ = 24 LOFAR -3.7%,
// so it is the default for N~ = 32 only).  A one-tile software pipeline of the HMMAs (tried as SCH = 1)
// compiles to the same SASS as 0: ptxas already spaces the HMMAs 5-12 instructions apart.
// FX: the A operand.  1: fixed-point f16 split by byte permutation (split_fx; N~ = 32 SKA loop 7.8 -> 8.8
// pairs/clk/SM against the f16 hi/lo split2 in scripts/split_probe.cu); 2 (the default for 16-row units): the
// integer form (split_i8, three m16n8k32 u8 x s8 mma per tile into s32 accumulators).
template <int NS, int WARPS, int MINB, int UNR, int CPT = 0, int R = 4, int SCH = 0, int FX = 1>
__global__ void __launch_bounds__(WARPS * 32, MINB) degridder_rot_kernel(const KernelArgs a) {
    constexpr int NPIX = NS * NS;
    constexpr int NKB = NPIX / 8;
    extern __shared__ __align__(16) unsigned char smem[];
    const DegridSmem<NS> sm(smem, a.max_timesteps_in_item);
    const uint4 *frag_s = sm.frag_s;
    const float4 *lmn_s = sm.lmn_s, *bq_s = sm.bq_s;
    const float *df_s = sm.df_s;
    static_assert(FX == 1 || FX == 2, "A operand form");
    __shared__ float red_s[WARPS];
    __shared__ __align__(16) float off_s[FX == 2 ? 16 * (WARPS + 1) : 8 * (WARPS + 1)];

    const int item = a.order[blockIdx.x];
    const ItemSetup s = dev::item_setup(a, item, NS);
    const idg_metadata &md = s.md;
    const int nc = s.nc;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, g = lane >> 2, q = lane & 3;
    const float inv0 = degridder_setup_tc<NS, WARPS, FX == 2 ? 1 : 0>(a, s, sm, red_s, off_s);
    // output = (acc - off) inv: the fixed-point operand's gain and per-column offset removed
    const float inv = FX == 1 ? inv0 * (1.0f / kFxGain) : inv0;
    const float off0 = FX == 1 ? off_s[2 * q] : 0.0f, off1 = FX == 1 ? off_s[2 * q + 1] : 0.0f;
    const double *offd = reinterpret_cast<const double *>(off_s);   // FX = 2
    const double ioff0 = FX == 2 ? offd[2 * q] : 0.0, ioff1 = FX == 2 ? offd[2 * q + 1] : 0.0;
    auto split = [](f2p C, f2p S, uint32_t &hq, uint32_t &lq, uint32_t &hq4, uint32_t &lq4) {
        if constexpr (FX == 2) {
            split_i8(C, S, hq, hq4);
        } else {
            split_fx(C, S, hq, lq, hq4, lq4);
        }
    };

    // A warp unit is 8 R visibilities = R channel rows (stride CS) for each of the 8 lane groups g, as R / 2
    // m-tiles (lane group g owns rows g and g+8 of every tile):
    //   CPT = 0 (C~ % 32 == 0, R = 4): one timestep, 32-channel block, lane base channel g, CS = 8;
    //   CPT > 0 (every item exactly CPT channels): CPT / R lane groups per timestep, 8 R / CPT timesteps per
    //   unit, lane base channel g % (CPT / R), CS = CPT / R.
    static_assert(R == 4 || R == 8 || R == 16, "channel rows per lane");
    static_assert(CPT == 0 ? R == 4 : (CPT % R == 0 && (8 * R) % CPT == 0), "channels per timestep");
    constexpr int NTL = R / 2;                        // m-tiles per unit
    constexpr int CS = CPT ? CPT / R : 8;             // channel stride of a lane's rows
    const int blocks = CPT ? 1 : nc >> 5;              // units per timestep (CPT = 0)
    const int nblk = CPT ? (md.nr_timesteps * CPT + 8 * R - 1) / (8 * R) : md.nr_timesteps * blocks;
    const float estep = float(CS) * a.channel_step;
    const int64_t row = int64_t(a.nr_channels) * 4;
    float2 *vis0 = a.vis + (int64_t(md.baseline) * a.nr_timesteps + md.time_offset) * row +
                   int64_t(md.channel_begin) * 4;
    for (int bk = warp; bk < nblk; bk += WARPS) {
        int t, c0;
        if constexpr (CPT) {
            t = bk * (8 * R / CPT) + g / CS;
            c0 = g % CS;
        } else {
            t = bk / blocks;
            c0 = (bk - t * blocks) * 32 + g;
        }
        const bool valid = t < md.nr_timesteps;
        const int tc = valid ? t : md.nr_timesteps - 1;
        const float4 cB = bq_s[2 * tc], cQ = bq_s[2 * tc + 1];
        const float df = df_s[c0];
        // row 0 (channel c0) coefficients, and the coefficients of the E phase
        const f2p cu = dup(fmaf(df, cQ.x, cB.x)), cv = dup(fmaf(df, cQ.y, cB.y)), cw = dup(fmaf(df, cQ.z, cB.z));
        const f2p eu = dup(estep * cQ.x), ev = dup(estep * cQ.y), ew = dup(estep * cQ.z);
        float acc[FX == 2 ? 1 : NTL][4];
        int iacc[FX == 2 ? NTL : 1][3][4];   // FX = 2: the s32 sums of the three weight classes
#pragma unroll
        for (int i = 0; i < NTL; ++i)
#pragma unroll
            for (int j = 0; j < 4; ++j) {
                if constexpr (FX == 2) {
                    iacc[i][0][j] = iacc[i][1][j] = iacc[i][2][j] = 0;
                } else {
                    acc[i][j] = 0.0f;
                }
            }
        static_assert(NKB % UNR == 0, "k-block unroll");
#pragma unroll UNR
        for (int kb = 0; kb < NKB; ++kb) {
            const uint4 bf = frag_s[kb * 32 + lane];
            const uint32_t bh0 = FX == 2 ? i8_high_limbs(bf.x) : 0u, bh1 = FX == 2 ? i8_high_limbs(bf.y) : 0u;
            const float4 lm = lmn_s[(kb * 4 + q) * 2], nn = lmn_s[(kb * 4 + q) * 2 + 1];
            const f2p l2 = pk(lm.x, lm.y), m2 = pk(lm.z, lm.w), n2 = pk(nn.x, nn.y);
            const float2 p = unpk(fma2(cu, l2, fma2(cv, m2, mul2(cw, n2))));   // row 0 at slots q, q+4
            const float2 e = unpk(fma2(eu, l2, fma2(ev, m2, mul2(ew, n2))));   // E phase at slots q, q+4
            float s0, c0q, s1, c1q, es0, ec0, es1, ec1;
            __sincosf(p.x, &s0, &c0q);
            __sincosf(p.y, &s1, &c1q);
            __sincosf(e.x, &es0, &ec0);
            __sincosf(e.y, &es1, &ec1);
            // rows r = 0..R-1 at slots (q, q+4), packed: C = (cos, cos), S = (sin, sin)
            f2p C = pk(c0q, c1q), S = pk(s0, s1);
            const f2p EC = pk(ec0, ec1), ES = pk(es0, es1), NES = pk(-es0, -es1);
            if constexpr (R == 4) {
                uint32_t ah[2][4], al[2][4];
#pragma unroll
                for (int r = 0; r < 4; ++r) {
                    if (r > 0) {
                        const f2p Cn = fma2(C, EC, mul2(S, NES));
                        S = fma2(C, ES, mul2(S, EC));
                        C = Cn;
                    }
                    // tile r >> 1, row g (r even) / g+8 (r odd): A regs {(row, q), (row+8, q), (row, q+4), (row+8, q+4)}
                    split(C, S, ah[r >> 1][r & 1], al[r >> 1][r & 1], ah[r >> 1][2 + (r & 1)], al[r >> 1][2 + (r & 1)]);
                }
                if constexpr (FX == 2) {
#pragma unroll
                    for (int i = 0; i < 2; ++i) imma3(iacc[i], ah[i], bf, bh0, bh1);
                } else {
#pragma unroll
                    for (int i = 0; i < 2; ++i) mma16816(acc[i], ah[i][0], ah[i][1], ah[i][2], ah[i][3], bf.x, bf.y);
#pragma unroll
                    for (int i = 0; i < 2; ++i) mma16816(acc[i], ah[i][0], ah[i][1], ah[i][2], ah[i][3], bf.z, bf.w);
#pragma unroll
                    for (int i = 0; i < 2; ++i) mma16816(acc[i], al[i][0], al[i][1], al[i][2], al[i][3], bf.x, bf.y);
                }
            } else if constexpr (SCH == 2) {
                // R = 8, 16, two rotation chains: tiles i (rows 2i, 2i+1) and i + NTL/2 (rows R/2 + 2i, ...)
                constexpr int H = NTL / 2;
                const f2p ph8 = fma2(dup(float(R / 2)), pk(e.x, e.y), pk(p.x, p.y));
                const float2 p8 = unpk(ph8);
                float s8a, c8a, s8b, c8b;
                __sincosf(p8.x, &s8a, &c8a);
                __sincosf(p8.y, &s8b, &c8b);
                f2p C2 = pk(c8a, c8b), S2 = pk(s8a, s8b);
#pragma unroll
                for (int i = 0; i < H; ++i) {
                    uint32_t ah[4], al[4], bh[4], bl[4];
#pragma unroll
                    for (int h2 = 0; h2 < 2; ++h2) {
                        if (i > 0 || h2 > 0) {
                            const f2p Cn = fma2(C, EC, mul2(S, NES));
                            S = fma2(C, ES, mul2(S, EC));
                            C = Cn;
                            const f2p Cm = fma2(C2, EC, mul2(S2, NES));
                            S2 = fma2(C2, ES, mul2(S2, EC));
                            C2 = Cm;
                        }
                        split(C, S, ah[h2], al[h2], ah[2 + h2], al[2 + h2]);
                        split(C2, S2, bh[h2], bl[h2], bh[2 + h2], bl[2 + h2]);
                    }
                    if constexpr (FX == 2) {
                        imma3(iacc[i], ah, bf, bh0, bh1);
                        imma3(iacc[i + H], bh, bf, bh0, bh1);
                    } else {
                        mma3(acc[i], ah, al, bf);
                        mma3(acc[i + H], bh, bl, bf);
                    }
                }
            } else {
                // R = 8, 16: each tile's three products issued as soon as its two rows are split
#pragma unroll
                for (int i = 0; i < NTL; ++i) {
                    uint32_t ah[4], al[4];
#pragma unroll
                    for (int h2 = 0; h2 < 2; ++h2) {
                        if (i > 0 || h2 > 0) {
                            const f2p Cn = fma2(C, EC, mul2(S, NES));
                            S = fma2(C, ES, mul2(S, EC));
                            C = Cn;
                        }
                        split(C, S, ah[h2], al[h2], ah[2 + h2], al[2 + h2]);
                    }
                    if constexpr (FX == 2) {
                        imma3(iacc[i], ah, bf, bh0, bh1);
                    } else {
                        mma3(acc[i], ah, al, bf);
                    }
                }
            }
        }
        if (valid) {
            float2 *vt = vis0 + int64_t(t) * row + int64_t(c0) * 4 + q;
#pragma unroll
            for (int r = 0; r < R; ++r) {
                if constexpr (FX == 2) {
                    vt[r * CS * 4] = make_float2(i8_out(iacc[r >> 1], 2 * (r & 1), ioff0, double(inv)),
                                                 i8_out(iacc[r >> 1], 2 * (r & 1) + 1, ioff1, double(inv)));
                } else {
                    vt[r * CS * 4] = make_float2((acc[r >> 1][2 * (r & 1)] - off0) * inv,
                                                 (acc[r >> 1][2 * (r & 1) + 1] - off1) * inv);
                }
            }
        }
    }
}

// Host: the DFT B-fragment tables of g_dft_tab (fp64 cos/sin, split into f16 hi + lo), uploaded once per
// device before the first tensor-core gridder / degridder launch on it.
uint32_t h2_pack(double x, double y, bool low_part) {
    auto part = [&](double v) {
        const __half hi = __float2half_rn(float(v));
        const __half h = low_part ? __float2half_rn(float(v - double(__half2float(hi)))) : hi;
        return uint32_t(__half_raw(h).x);
    };
    return part(x) | (part(y) << 16);
}

cudaError_t ensure_dft_tables() {
    static std::mutex mu;
    static std::vector<char> done;
    int dev = 0;
    cudaError_t err = cudaGetDevice(&dev);
    if (err != cudaSuccess) return err;
    std::lock_guard<std::mutex> lock(mu);
    if (size_t(dev) < done.size() && done[dev]) return cudaSuccess;
    std::vector<uint4> tab(2 * size_t(kDftTabEntries));
    for (int sgn = 0; sgn < 2; ++sgn) {
        const double sign = sgn == 0 ? -1.0 : 1.0;
        for (int ns : {16, 24, 32}) {
            const int ntl = ns / 4, kst = ns / 8, h = ns / 2;
            for (int e = 0; e < kst * ntl * 32; ++e) {
                const int ln = e & 31, t = e >> 5, ks = t / ntl, nt = t - ks * ntl;
                const int gg = ln >> 2, qq = ln & 3;
                const int k = nt * 4 + (gg >> 1), im = gg & 1;
                double bx[2], by[2];
                for (int r = 0; r < 2; ++r) {
                    const int x = ks * 8 + qq + 4 * r;
                    int ex = ((k - h) * (x - h)) % ns;
                    ex += ex < 0 ? ns : 0;
                    const double ang = 2.0 * 3.14159265358979323846 * double(ex) / double(ns);
                    const double cs = std::cos(ang), sn = sign * std::sin(ang);
                    bx[r] = im ? sn : cs;
                    by[r] = im ? cs : -sn;
                }
                tab[size_t(sgn) * kDftTabEntries + dft_tab_offset(ns) + e] =
                    make_uint4(h2_pack(bx[0], by[0], false), h2_pack(bx[1], by[1], false),
                               h2_pack(bx[0], by[0], true), h2_pack(bx[1], by[1], true));
            }
        }
    }
    err = cudaMemcpyToSymbol(g_dft_tab, tab.data(), tab.size() * sizeof(uint4));
    if (err != cudaSuccess) return err;
    // a pageable upload may return before its DMA has finished, and kernels launched on non-blocking
    // streams are not ordered after it: wait for it once per device before any kernel reads the table
    err = cudaDeviceSynchronize();
    if (err != cudaSuccess) return err;
    if (done.size() <= size_t(dev)) done.resize(size_t(dev) + 1, 0);
    done[dev] = 1;
    return cudaSuccess;
}

// ------------------------------------------------------------------------------------------------
// Launchers and the variant tables.  Each variant names its dynamic shared memory (smem_*), so the
// dispatcher can skip variants a plan's items do not fit (idg_kernels.cu: eligible()).
// ------------------------------------------------------------------------------------------------
template <typename K>
cudaError_t launch_tc(K kernel, const char *name, size_t smem, int threads, const KernelArgs &a, cudaStream_t st) {
    cudaError_t err = ensure_dft_tables();
    if (err != cudaSuccess) return err;
    if ((err = dev::prepare(kernel, smem)) != cudaSuccess) return err;
    LaunchScope scope(name, st);
    kernel<<<unsigned(a.nr_items), threads, smem, st>>>(a);
    return cudaGetLastError();
}

template <int NS, int WARPS, int MT, int MINB, int KBB = kTcBatchKB>
size_t smem_gridder_tc(const KernelArgs &a) { return gridder_tc_smem_bytes(NS, a.max_channels_in_item, KBB); }
template <int NS, int WARPS, int MT, int MINB, int KBB = kTcBatchKB>
cudaError_t launch_gridder_tc(const KernelArgs &a, cudaStream_t st) {
    return launch_tc(gridder_tc_kernel<NS, WARPS, MT, MINB, KBB>, "gridder", smem_gridder_tc<NS, WARPS, MT, MINB, KBB>(a),
                     WARPS * 32, a, st);
}

template <int NS, int WARPS, int MT, int MINB, int KPT, int GP, int KBB = kTcBatchKB, int NSM = 0>
size_t smem_gridder_rot2(const KernelArgs &) {
    return gridder_rot_smem_bytes(NS, KBB) + size_t(NSM) * NS * NS * 4 + (NSM == 2 ? size_t(NS) * NS * 4 : 0);
}
template <int NS, int WARPS, int MT, int MINB, int KPT, int GP, int KBB = kTcBatchKB, int NSM = 0, int PKR = 0,
          int HOR = 0>
cudaError_t launch_gridder_rot2(const KernelArgs &a, cudaStream_t st) {
    return launch_tc(gridder_rot2_kernel<NS, WARPS, MT, MINB, KPT, GP, KBB, 1, NSM, PKR, HOR>, "gridder",
                     smem_gridder_rot2<NS, WARPS, MT, MINB, KPT, GP, KBB, NSM>(a), WARPS * 32, a, st);
}

template <int NS>
size_t smem_degridder_tc(const KernelArgs &a) {
    return degridder_tc_smem_bytes(NS, a.max_timesteps_in_item, a.max_channels_in_item);
}
template <int NS, int WARPS, int MT, int MINB, int FX = 1>
cudaError_t launch_degridder_tc(const KernelArgs &a, cudaStream_t st) {
    return launch_tc(degridder_tc_kernel<NS, WARPS, MT, MINB, FX>, "degridder", smem_degridder_tc<NS>(a), WARPS * 32, a, st);
}
template <int NS, int WARPS, int MINB, int UNR, int CPT = 0, int R = 4, int SCH = 0, int FX = 1>
cudaError_t launch_degridder_rot(const KernelArgs &a, cudaStream_t st) {
    return launch_tc(degridder_rot_kernel<NS, WARPS, MINB, UNR, CPT, R, SCH, FX>, "degridder", smem_degridder_tc<NS>(a),
                     WARPS * 32, a, st);
}

// Gridders.  First eligible entry is the default: the rotation gridder when every item has exactly 8 KPT
// uniformly spaced channels (nsm / lmnsm: pixel coordinates re-read from shared memory, N~ = 32), else
// the direct kernel (one sincos per pair; any channel table with C~ % 8 == 0), else the SIMT kernel.
#include "idg_kernels_umma.cuh"   // the tcgen05 rotation gridder (gridder_umma_rot), in this namespace

#define GUR(KPT) \
    {32, 8 * KPT, kTensor, 1, "gridder_umma_rot<32,KPT" #KPT ",pair>", launch_gridder_umma_rot<KPT>, 8 * KPT, \
     smem_gridder_umma_rot<KPT>}
#define TGROT2(NS, W, MT, MB, KPT) \
    {NS, 8 * KPT, kTensor, 1, "gridder_rot2<" #NS ",W" #W ",MT" #MT ",minB" #MB ",KPT" #KPT ">", \
     launch_gridder_rot2<NS, W, MT, MB, KPT, KPT, 128>, 8 * KPT, smem_gridder_rot2<NS, W, MT, MB, KPT, KPT, 128>}
#define TGROT2N(NS, W, MT, MB, KPT, GP, NSM, TAG) \
    {NS, 8 * KPT, kTensor, 1, "gridder_rot2<" #NS ",W" #W ",MT" #MT ",minB" #MB ",KPT" #KPT ",GP" #GP "," TAG ">", \
     launch_gridder_rot2<NS, W, MT, MB, KPT, GP, 128, NSM>, 8 * KPT, smem_gridder_rot2<NS, W, MT, MB, KPT, GP, 128, NSM>}
#define TG(NS, W, MT, MB) \
    {NS, 8, kTensor, 0, "gridder_tc<" #NS ",W" #W ",MT" #MT ",minB" #MB ">", launch_gridder_tc<NS, W, MT, MB>, 0, \
     smem_gridder_tc<NS, W, MT, MB>}
#define TGROT2H(NS, W, MT, MB, KPT, GP, NSM, TAG) \
    {NS, 8 * KPT, kTensor, 1, "gridder_rot2h<" #NS ",W" #W ",MT" #MT ",minB" #MB ",KPT" #KPT ",GP" #GP "," TAG ">", \
     launch_gridder_rot2<NS, W, MT, MB, KPT, GP, 128, NSM, 0, 1>, 8 * KPT, smem_gridder_rot2<NS, W, MT, MB, KPT, GP, 128, NSM>}
#define TGROT2P(NS, W, MT, MB, KPT, GP, NSM, TAG) \
    {NS, 8 * KPT, kTensor, 1, "gridder_rot2p<" #NS ",W" #W ",MT" #MT ",minB" #MB ",KPT" #KPT ",GP" #GP "," TAG ">", \
     launch_gridder_rot2<NS, W, MT, MB, KPT, GP, 128, NSM, 1>, 8 * KPT, smem_gridder_rot2<NS, W, MT, MB, KPT, GP, 128, NSM>}
const Variant kTcGridder[] = {
    TGROT2(24, 12, 3, 2, 2), TGROT2(24, 12, 3, 2, 4), TGROT2(24, 12, 3, 2, 1),
    TGROT2H(32, 8, 8, 2, 4, 4, 0, "r"), TGROT2N(32, 8, 8, 2, 2, 2, 0, "r"), TGROT2(32, 16, 4, 2, 1),
    TGROT2(16, 8, 2, 2, 2), TGROT2(16, 8, 2, 2, 4), TGROT2(16, 8, 2, 2, 1),
    TG(24, 12, 3, 2), TG(32, 16, 4, 2), TG(16, 4, 4, 4),
    // alternates kept for measurement (selected by name only): the packed rotation (slower: spills), the
    // E^j form for N~ = 32 (the default before the Horner form), Horner with n only in shared memory.
    // Measured and dropped (r02i / r02o, SKA-T1024, against 135.7 ms): group passes of 1 / 4 in the E^j
    // form, Horner at 16 warps x 4 tiles with 128 registers (138.0), 32 warps of 2 tiles (147.4).  Default
    // since r02zq: 8 warps x 8 tiles at 128 registers (16 warps / SM), pixel coordinates in registers (no
    // spills): SKA-T1024 136.3 -> 124.7 ms (with lmnsm 130.3; 4 warps x 16 tiles 138.1), predict-T256 (KPT 2)
    // 251.5 -> 244.0 ms; LOFAR (N~ = 24) keeps 12 warps x 3 tiles (6 x 6: 36.7, 4 x 9: 38.1 against 32.3 ms).
    // The fixed-point phasor split in the gridders measured 131.7 ms (r02zo) and is not used there.
    TGROT2P(24, 12, 3, 2, 2, 2, 0, "r"), TGROT2N(32, 16, 4, 2, 4, 2, 1, "nsm"), TGROT2H(32, 16, 4, 2, 4, 4, 1, "nsm"),
    // the defaults before r02zo / r02zq (32 warps x 4 tiles at 64 registers, pixel coordinates re-read from
    // shared memory to limit the spills)
    TGROT2H(32, 16, 4, 2, 4, 4, 2, "lmnsm"), TGROT2N(32, 16, 4, 2, 2, 2, 2, "lmnsm"),
    // tcgen05 / TMEM rotation gridder (selected by name while measured)
    GUR(4), GUR(2),
};
#undef GUR
#undef TGROT2H
#undef TGROT2P
#undef TGROT2
#undef TGROT2N
#undef TG

// Degridders.  Default: the phasor-rotation kernel for the item's channel layout (16 channel rows per lane
// for 16- / 32-channel items, 8 for 8, 4 for 4 and for any multiple of 32), else the direct kernel, else
// the SIMT kernel.
#define TDROTC(NS, W, MB, U, CPT, R, TAG) \
    {NS, CPT, kTensor, 1, TAG "<" #NS ",W" #W ",minB" #MB ",U" #U ",C" #CPT ">", \
     launch_degridder_rot<NS, W, MB, U, CPT, R>, CPT, smem_degridder_tc<NS>}
// short items (the plan's mean T~ <= 64): 8 channel rows per lane, 4-timestep warp units (finer than the 8 of
// R = 16, so ragged item tails leave fewer warps idle): lofar_short 3081 -> 3203 MVis/s, LOFAR -7% (r02i); the
// integer form (FX = 2) 34.7 -> 33.9 ms on lofar_short (r02zm), at unroll 4 33.1 ms (r02zz)
#define TDROTS(NS, W, MB, U, CPT, R, FX, TAG) \
    {NS, CPT, kTensor, 1, TAG "<" #NS ",W" #W ",minB" #MB ",U" #U ",C" #CPT ">", \
     launch_degridder_rot<NS, W, MB, U, CPT, R, 0, FX>, CPT, smem_degridder_tc<NS>, 64}
#define TDROTX(NS, W, MB, U, CPT, R, SCH) \
    {NS, CPT, kTensor, 1, "degridder_rot16s" #SCH "<" #NS ",W" #W ",minB" #MB ",U" #U ",C" #CPT ">", \
     launch_degridder_rot<NS, W, MB, U, CPT, R, SCH>, CPT, smem_degridder_tc<NS>}
#define TDROTI(NS, W, MB, U, CPT, R) \
    {NS, CPT, kTensor, 1, "degridder_rot" #R "i<" #NS ",W" #W ",minB" #MB ",U" #U ",C" #CPT ">", \
     launch_degridder_rot<NS, W, MB, U, CPT, R, 0, 2>, CPT, smem_degridder_tc<NS>}
#define TDROTI4(NS, W, MB, U, CPT) \
    {NS, CPT ? CPT : 32, kTensor, 1, "degridder_roti<" #NS ",W" #W ",minB" #MB ",U" #U ",C" #CPT ">", \
     launch_degridder_rot<NS, W, MB, U, CPT, 4, 0, 2>, CPT, smem_degridder_tc<NS>}
#define TDROT(NS, W, MB, U) \
    {NS, 32, kTensor, 1, "degridder_rot<" #NS ",W" #W ",minB" #MB ",U" #U ">", launch_degridder_rot<NS, W, MB, U>, 0, \
     smem_degridder_tc<NS>}
#define TDI(NS, W, MT, MB) \
    {NS, 0, kTensor, 0, "degridder_tci<" #NS ",W" #W ",MT" #MT ",minB" #MB ">", launch_degridder_tc<NS, W, MT, MB, 2>, 0, \
     smem_degridder_tc<NS>}
#define TD(NS, W, MT, MB) \
    {NS, 0, kTensor, 0, "degridder_tc<" #NS ",W" #W ",MT" #MT ",minB" #MB ">", launch_degridder_tc<NS, W, MT, MB>, 0, \
     smem_degridder_tc<NS>}
const Variant kTcDegridder[] = {
    // 16-row integer units at k-block unroll 8 (r02zz: against U4 SKA-T1024 140.7 -> 138.8 ms, predict-T256
    // 214.2 -> 212.1, LOFAR 27.53 -> 27.30)
    TDROTS(24, 4, 3, 4, 16, 8, 2, "degridder_rot8i"), TDROTI(24, 4, 3, 8, 16, 16), TDROTI(32, 4, 2, 8, 32, 16), TDROTI(32, 4, 2, 8, 16, 16),
    TDROTC(24, 4, 3, 4, 16, 16, "degridder_rot16"), TDROTX(32, 8, 2, 2, 32, 16, 2),
    TDROTX(32, 8, 2, 1, 16, 16, 2), TDROTC(16, 8, 2, 1, 16, 16, "degridder_rot16"),
    TDROTC(16, 8, 2, 1, 32, 16, "degridder_rot16"),
    TDROTI(24, 8, 2, 1, 8, 8), TDROTI(32, 8, 2, 1, 8, 8), TDROTI(16, 8, 2, 1, 8, 8),   // 8-channel items
    TDROTC(24, 8, 2, 1, 8, 8, "degridder_rot8"), TDROTC(32, 16, 2, 1, 8, 8, "degridder_rot8"),
    TDROTC(16, 8, 2, 1, 8, 8, "degridder_rot8"),
    // 4-row units (C~ a multiple of 32 other than 32; 4 channels): integer form, then the f16 fixed-point form
    TDROTI4(32, 8, 2, 2, 0), TDROTI4(24, 8, 3, 1, 0), TDROTI4(16, 8, 3, 1, 0),
    TDROTI4(24, 8, 3, 1, 4), TDROTI4(32, 8, 2, 1, 4), TDROTI4(16, 8, 3, 1, 4),
    TDROT(32, 16, 2, 2), TDROT(24, 8, 4, 1), TDROT(16, 8, 4, 1),
    TDROTC(24, 8, 4, 1, 4, 4, "degridder_rot"), TDROTC(32, 16, 2, 1, 4, 4, "degridder_rot"),
    TDROTC(16, 8, 4, 1, 4, 4, "degridder_rot"),
    // the direct kernel (any channel table) in the integer form (r02zu: LOFAR-T2048 10.35 -> 9.72 ms, SKA-T256
    // 53.6 -> 49.6 ms, parity 3.2e-5 -> 1.4e-5), then in the f16 fixed-point form
    TDI(24, 8, 2, 3), TDI(32, 8, 2, 2), TDI(16, 8, 2, 2), TD(24, 8, 2, 4), TD(32, 8, 4, 2), TD(16, 8, 4, 2),
    // the single-chain N~ = 32 kernels, and 8-row units for 16-channel items (finer work units for short
    // items) -- selected by name only
    TDROTC(32, 8, 2, 2, 32, 16, "degridder_rot16"), TDROTC(32, 8, 2, 2, 16, 16, "degridder_rot16"),
    TDROTC(24, 8, 2, 1, 16, 8, "degridder_rot8"), TDROTS(24, 4, 3, 2, 16, 8, 1, "degridder_rot8"),
};
#undef TDROTC
#undef TDROTI
#undef TDROTI4
#undef TDI
#undef TDROTS
#undef TDROTX
#undef TDROT
#undef TD

}  // namespace

const Variant *tc_gridder_variants(int *n) {
    *n = int(sizeof(kTcGridder) / sizeof(kTcGridder[0]));
    return kTcGridder;
}

const Variant *tc_degridder_variants(int *n) {
    *n = int(sizeof(kTcDegridder) / sizeof(kTcDegridder[0]));
    return kTcDegridder;
}

}  // namespace idg
