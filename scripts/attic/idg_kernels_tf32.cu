// idg_kernels_tf32.cu -- tensor-core gridder/degridder with a 3-pass tf32 split (Veenboer et al. 2017).
//
// Same contraction as idg_kernels_tc.cu (16 multiply-adds per (pixel, visibility) pair on the tensor
// cores), but the operands are split as x = hi + lo with hi = x with the low 13 mantissa bits
// cleared (exactly a tf32 value) and lo = x - hi (exact in fp32; the mma reads its top 11 bits), and
// the product is hi*hi + hi*lo + lo*hi in mma.m16n8k8.tf32 with fp32 accumulation (~21-bit operands).
// Compared with the f16 split this needs no conversion instructions (2 LOP3 + 1 FADD2 per phasor
// instead of 2 F2FP + 2 HADD2 + 1 FADD2), no range scaling (tf32 keeps the fp32 exponent) and a
// shorter dependency chain behind each MUFU result; the price is 6 instead of 3 mma per 16x8 tile of
// 8 visibilities (tf32 runs at half the f16 rate), which stays below the sincos (XU) bound.
//
// tf32 m16n8k8 layouts (g = lane/4, q = lane%4); a k8 block = 4 visibilities (or pixels) with the
// k order [cos v0..v3, sin v0..v3]:
//   A: a0 = A[g][q] = cos(row g, v_q), a1 = A[g+8][q] = cos(row g+8, v_q), a2 = sin(row g, v_q),
//      a3 = sin(row g+8, v_q)
//   B: b0 = B[q][g] (cos-row of v_q, column g), b1 = B[q+4][g] (sin-row of v_q, column g)
//   D: d0,d1 = D[g][2q..2q+1], d2,d3 = D[g+8][2q..2q+1]  (column 2 pol + re/im, pol = q)
// An 8-visibility k-block is two k8 halves: visibilities (q) and (q+4) of the block for thread q.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>

#include "idg_device.cuh"
#include "idg_internal.h"

namespace idg {
namespace {

using dev::ItemSetup;
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
__device__ __forceinline__ uint32_t hi_bits(float x) { return __float_as_uint(x) & 0xffffe000u; }

// (x, y) -> hi (tf32-exact bit patterns) and lo = (x, y) - hi (one FADD2)
__device__ __forceinline__ void split_tf32(float x, float y, uint32_t &hx, uint32_t &hy, uint32_t &lx,
                                           uint32_t &ly) {
    hx = hi_bits(x);
    hy = hi_bits(y);
    const float2 d = unpk(sub2(pk(x, y), pk(__uint_as_float(hx), __uint_as_float(hy))));
    lx = __float_as_uint(d.x);
    ly = __float_as_uint(d.y);
}

__device__ __forceinline__ void mma1688(float (&d)[4], uint32_t a0, uint32_t a1, uint32_t a2, uint32_t a3,
                                        uint32_t b0, uint32_t b1) {
    asm("mma.sync.aligned.m16n8k8.row.col.f32.tf32.tf32.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, "
        "{%0,%1,%2,%3};"
        : "+f"(d[0]), "+f"(d[1]), "+f"(d[2]), "+f"(d[3])
        : "r"(a0), "r"(a1), "r"(a2), "r"(a3), "r"(b0), "r"(b1));
}

// One k8 half for one tile: D += Ahi Bhi + Ahi Blo + Alo Bhi.
struct Frag4 {
    uint32_t c0, c1, s0, s1;  // cos(row g), cos(row g+8), sin(row g), sin(row g+8)
};
__device__ __forceinline__ void mma3_tf32(float (&d)[4], const Frag4 &ah, const Frag4 &al, uint32_t bh0,
                                          uint32_t bh1, uint32_t bl0, uint32_t bl1) {
    mma1688(d, ah.c0, ah.c1, ah.s0, ah.s1, bh0, bh1);
    mma1688(d, ah.c0, ah.c1, ah.s0, ah.s1, bl0, bl1);
    mma1688(d, al.c0, al.c1, al.s0, al.s1, bh0, bh1);
}

// phasors (cs, sn) of rows g and g+8 -> hi/lo A fragments
__device__ __forceinline__ void make_frags(float c0, float s0, float c1, float s1, Frag4 &ah, Frag4 &al) {
    split_tf32(c0, c1, ah.c0, ah.c1, al.c0, al.c1);
    split_tf32(s0, s1, ah.s0, ah.s1, al.s0, al.s1);
}

// ------------------------------------------------------------------------------------------------
// Gridder (tf32).  Batch of KBB k-blocks (8 visibilities each, one timestep); B fragments are stored
// split: per (k-block, lane) uint4 hi = {b0, b1 of half 0, b0, b1 of half 1} and uint4 lo likewise.
// ------------------------------------------------------------------------------------------------
constexpr int kTf32BatchKB = 32;  // 256 visibilities per batch

inline size_t gridder_tf32_smem_bytes(int NS, int max_channels) {
    const size_t kbb = kTf32BatchKB;
    const size_t main = kbb * 8 * 32 /*raw*/ + kbb * 32 * 32 /*frag hi+lo*/ + kbb * 4 * 16 /*df*/ +
                        (kbb + 1) * 32 /*coef*/ + size_t(max_channels) * 4;
    const size_t epi = size_t(2) * 4 * NS * NS * sizeof(float2);
    return std::max(main, epi) + 16;
}

template <int NS, int WARPS, int MT, int MINB, int REC>
__global__ void __launch_bounds__(WARPS * 32, MINB) gridder_tf32_kernel(const KernelArgs a) {
    constexpr int NT = WARPS * 32;
    constexpr int NPIX = NS * NS;
    static_assert(WARPS * MT * 16 == NPIX, "warps x m-tiles x 16 must cover the subgrid");
    constexpr int h = NS / 2;
    constexpr int KBB = kTf32BatchKB;
    constexpr int VB = KBB * 8;
    extern __shared__ __align__(16) unsigned char smem[];
    float4 *raw_s = reinterpret_cast<float4 *>(smem);                // [VB][2]
    uint4 *frag_s = reinterpret_cast<uint4 *>(raw_s + 2 * VB);       // [KBB][32][2] (hi, lo)
    float4 *dfk_s = reinterpret_cast<float4 *>(frag_s + KBB * 64);   // [KBB][4]
    float4 *coef_s = reinterpret_cast<float4 *>(dfk_s + KBB * 4);    // [KBB+1][2]
    float *df_s = reinterpret_cast<float *>(coef_s + 2 * (KBB + 1)); // [nc]
    __shared__ float2 tw[NS];

    const int item = a.order[blockIdx.x];
    const ItemSetup s = dev::item_setup(a, item, NS);
    const idg_metadata &md = s.md;
    const int nc = s.nc;
    const int kpt = nc >> 3;
    const int nkb = md.nr_timesteps * kpt;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, g = lane >> 2, q = lane & 3;

    for (int c = threadIdx.x; c < nc; c += NT)
        df_s[c] = float((a.frequencies[md.channel_begin + c] / kSpeedOfLight) - s.f_ref);

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

    const int64_t row = int64_t(a.nr_channels) * 4;
    const float2 *vis0 = a.vis + (int64_t(md.baseline) * a.nr_timesteps + md.time_offset) * row +
                         int64_t(md.channel_begin) * 4;

    for (int kb0 = 0; kb0 < nkb; kb0 += KBB) {
        const int kb1 = min(kb0 + KBB, nkb);
        const int nvb = (kb1 - kb0) * 8;
        const int t_first = kb0 / kpt, t_last = (kb1 - 1) / kpt;
        __syncthreads();
        for (int i = threadIdx.x; i < 2 * nvb; i += NT) {
            const int j = i >> 1;
            const int kb = kb0 + (j >> 3);
            const int t = kb / kpt;
            const int c = (kb - t * kpt) * 8 + (j & 7);
            raw_s[i] = dev::ld_stream(reinterpret_cast<const float4 *>(vis0 + int64_t(t) * row + c * 4) + (i & 1));
        }
        for (int t = t_first + int(threadIdx.x); t <= t_last; t += NT) {
            float4 cB, cQ;
            dev::timestep_coefficients(a, s, md.time_offset + t, cB, cQ);
            coef_s[2 * (t - t_first)] = cB;
            coef_s[2 * (t - t_first) + 1] = cQ;
        }
        for (int i = threadIdx.x; i < (kb1 - kb0) * 4; i += NT) {
            const int kb = kb0 + (i >> 2);
            const int c = (kb % kpt) * 8 + (i & 3);
            dfk_s[i] = make_float4(df_s[c], df_s[c], df_s[c + 4], df_s[c + 4]);
        }
        __syncthreads();
        // B fragments, split: column g = 2 pol + im; cos-row (Vre | Vim), sin-row (-Vim | Vre)
        for (int i = threadIdx.x; i < (kb1 - kb0) * 32; i += NT) {
            const int kbl = i >> 5, ln = i & 31, gg = ln >> 2, qq = ln & 3;
            const int pol = gg >> 1, im = gg & 1;
            uint32_t hv[4], lv[4];
#pragma unroll
            for (int hh = 0; hh < 2; ++hh) {
                const float4 v4 = raw_s[2 * (kbl * 8 + qq + 4 * hh) + (pol >> 1)];
                const float vr = (pol & 1) ? v4.z : v4.x;
                const float vi = (pol & 1) ? v4.w : v4.y;
                split_tf32(im ? vi : vr, im ? vr : -vi, hv[2 * hh], hv[2 * hh + 1], lv[2 * hh], lv[2 * hh + 1]);
            }
            frag_s[2 * i] = make_uint4(hv[0], hv[1], hv[2], hv[3]);
            frag_s[2 * i + 1] = make_uint4(lv[0], lv[1], lv[2], lv[3]);
        }
        __syncthreads();
        float part[MT][4];
#pragma unroll
        for (int i = 0; i < MT; ++i)
#pragma unroll
            for (int j = 0; j < 4; ++j) part[i][j] = 0.0f;
        for (int t = t_first; t <= t_last; ++t) {
            const float4 cB = coef_s[2 * (t - t_first)], cQ = coef_s[2 * (t - t_first) + 1];
            f2p Bv[MT], Qv[MT];
            float stc[REC ? MT : 1][2], sts[REC ? MT : 1][2];
#pragma unroll
            for (int i = 0; i < MT; ++i) {
                Bv[i] = fma2(dup(cB.x), pl[i], fma2(dup(cB.y), pm[i], mul2(dup(cB.z), pn[i])));
                Qv[i] = fma2(dup(cQ.x), pl[i], fma2(dup(cQ.y), pm[i], mul2(dup(cQ.z), pn[i])));
                if (REC) {
                    const float2 st = unpk(mul2(dup(4.0f * a.channel_step), Qv[i]));
                    __sincosf(st.x, &sts[i][0], &stc[i][0]);
                    __sincosf(st.y, &sts[i][1], &stc[i][1]);
                }
            }
            const int k_begin = max(kb0, t * kpt), k_end = min(kb1, (t + 1) * kpt);
#pragma unroll 1
            for (int kb = k_begin; kb < k_end; ++kb) {
                const uint4 bh = frag_s[2 * ((kb - kb0) * 32 + lane)];
                const uint4 bl = frag_s[2 * ((kb - kb0) * 32 + lane) + 1];
                const float4 df = dfk_s[(kb - kb0) * 4 + q];
                const f2p dq = pk(df.x, df.y), dq4 = pk(df.z, df.w);
                Frag4 ah[MT][2], al[MT][2];
#pragma unroll
                for (int i = 0; i < MT; ++i) {
                    float sn[4], cs[4];
                    const float2 ph0 = unpk(fma2(dq, Qv[i], Bv[i]));  // rows (g, g+8) at slot q
                    __sincosf(ph0.x, &sn[0], &cs[0]);
                    __sincosf(ph0.y, &sn[1], &cs[1]);
                    if (REC) {
#pragma unroll
                        for (int r = 0; r < 2; ++r) {
                            cs[2 + r] = fmaf(cs[r], stc[i][r], -sn[r] * sts[i][r]);
                            sn[2 + r] = fmaf(cs[r], sts[i][r], sn[r] * stc[i][r]);
                        }
                    } else {
                        const float2 ph1 = unpk(fma2(dq4, Qv[i], Bv[i]));  // rows at slot q+4
                        __sincosf(ph1.x, &sn[2], &cs[2]);
                        __sincosf(ph1.y, &sn[3], &cs[3]);
                    }
                    make_frags(cs[0], sn[0], cs[1], sn[1], ah[i][0], al[i][0]);
                    make_frags(cs[2], sn[2], cs[3], sn[3], ah[i][1], al[i][1]);
                }
                // pass-major issue: independent accumulators between dependent mma
#pragma unroll
                for (int hh = 0; hh < 2; ++hh) {
                    const uint32_t bh0 = hh ? bh.z : bh.x, bh1 = hh ? bh.w : bh.y;
                    const uint32_t bl0 = hh ? bl.z : bl.x, bl1 = hh ? bl.w : bl.y;
#pragma unroll
                    for (int i = 0; i < MT; ++i)
                        mma1688(part[i], ah[i][hh].c0, ah[i][hh].c1, ah[i][hh].s0, ah[i][hh].s1, bh0, bh1);
#pragma unroll
                    for (int i = 0; i < MT; ++i)
                        mma1688(part[i], ah[i][hh].c0, ah[i][hh].c1, ah[i][hh].s0, ah[i][hh].s1, bl0, bl1);
#pragma unroll
                    for (int i = 0; i < MT; ++i)
                        mma1688(part[i], al[i][hh].c0, al[i][hh].c1, al[i][hh].s0, al[i][hh].s1, bh0, bh1);
                }
            }
        }
#pragma unroll
        for (int i = 0; i < MT; ++i)
#pragma unroll
            for (int j = 0; j < 4; ++j) acc[i][j] += part[i][j];
    }

    __syncthreads();
    float2 *sub_s = reinterpret_cast<float2 *>(smem);
    float2 *tmp_s = sub_s + 4 * NPIX;
#pragma unroll
    for (int i = 0; i < MT; ++i) {
        const int p0 = (warp * MT + i) * 16 + g;
        sub_s[q * NPIX + p0] = make_float2(acc[i][0], acc[i][1]);
        sub_s[q * NPIX + p0 + 8] = make_float2(acc[i][2], acc[i][3]);
    }
    __syncthreads();
    dev::gridder_epilogue<NS>(a, s, sub_s, tmp_s, tw);
}

// ------------------------------------------------------------------------------------------------
// Degridder (tf32).  The corrected subgrid is stored as fp32 B fragments (per (k-block, lane):
// {b0, b1 of half 0, b0, b1 of half 1}); the hi/lo split of B is done on the fly per k-block and
// shared by the MT tiles of the warp.
// ------------------------------------------------------------------------------------------------
inline size_t degridder_tf32_smem_bytes(int NS) {
    const size_t npix = size_t(NS) * NS;
    return npix * 64 /*sub+tmp | frag*/ + npix * 16 /*lmn slot pairs*/ + 16;
}

template <int NS, int WARPS, int MT, int MINB>
__global__ void __launch_bounds__(WARPS * 32, MINB) degridder_tf32_kernel(const KernelArgs a) {
    constexpr int NT = WARPS * 32;
    constexpr int NPIX = NS * NS;
    constexpr int NKB = NPIX / 8;
    constexpr int PPT = (NPIX + NT - 1) / NT;
    constexpr int h = NS / 2;
    extern __shared__ __align__(16) unsigned char smem[];
    float2 *sub_s = reinterpret_cast<float2 *>(smem);
    float2 *tmp_s = sub_s + 4 * NPIX;
    float4 *frag_s = reinterpret_cast<float4 *>(smem);                     // [NKB][32] after prologue
    float4 *lmn_s = reinterpret_cast<float4 *>(smem + size_t(NPIX) * 64);  // [NKB][4][2]
    __shared__ float2 tw[NS];

    const int item = a.order[blockIdx.x];
    const ItemSetup s = dev::item_setup(a, item, NS);
    const idg_metadata &md = s.md;
    const int nc = s.nc;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, g = lane >> 2, q = lane & 3;

    dev::degridder_split_columns<NS>(a, s, sub_s, tmp_s, tw);
    float2 rr[PPT][4];
#pragma unroll
    for (int i = 0; i < PPT; ++i) {
        const int pix = threadIdx.x + i * NT;
        if (pix < NPIX) {
            dev::degridder_pixel<NS>(a, s, tmp_s, tw, pix, rr[i]);
            const int y = pix / NS, x = pix - y * NS;
            const float l = float(x - h) * a.cell_l, m = float(y - h) * a.cell_l;
            const int kb = pix >> 3, slot = pix & 7, half = slot >> 2;
            float *rec = reinterpret_cast<float *>(lmn_s + (kb * 4 + (slot & 3)) * 2);
            rec[half] = l;
            rec[2 + half] = m;
            rec[4 + half] = dev::w_term_n(l, m);
            rec[6 + half] = 0.0f;
        }
    }
    __syncthreads();  // every read of tmp_s is done before frag_s (aliasing sub_s/tmp_s) is written
    float *frag_w = reinterpret_cast<float *>(frag_s);
#pragma unroll
    for (int i = 0; i < PPT; ++i) {
        const int pix = threadIdx.x + i * NT;
        if (pix < NPIX) {
            const int kb = pix >> 3, slot = pix & 7, qq = slot & 3, half = slot >> 2;
#pragma unroll
            for (int gg = 0; gg < 8; ++gg) {
                const int pol = gg >> 1;
                const float sr = rr[i][pol].x, si = rr[i][pol].y;
                // V += S exp(-i phi): column 2pol: cos-row Sre, sin-row Sim; column 2pol+1: Sim, -Sre
                const int e = (kb * 32 + gg * 4 + qq) * 4 + 2 * half;
                frag_w[e] = (gg & 1) ? si : sr;
                frag_w[e + 1] = (gg & 1) ? -sr : si;
            }
        }
    }
    __syncthreads();

    const int nvis = md.nr_timesteps * nc;
    const int ntiles = (nvis + 15) >> 4;
    const int64_t row = int64_t(a.nr_channels) * 4;
    float2 *vis0 = a.vis + (int64_t(md.baseline) * a.nr_timesteps + md.time_offset) * row +
                   int64_t(md.channel_begin) * 4;
    for (int tile0 = warp * MT; tile0 < ntiles; tile0 += WARPS * MT) {
        f2p cu[MT][2], cv[MT][2], cw[MT][2];
        float acc[MT][4];
#pragma unroll
        for (int i = 0; i < MT; ++i) {
#pragma unroll
            for (int r = 0; r < 2; ++r) {
                const int v = (tile0 + i) * 16 + g + 8 * r;
                float fu = 0.0f, fv = 0.0f, fw = 0.0f;
                if (v < nvis) {
                    const int t = v / nc, c = v - t * nc;
                    const float *p = a.uvw + (int64_t(md.baseline) * a.nr_timesteps + md.time_offset + t) * 3;
                    const double f = a.frequencies[md.channel_begin + c] / kSpeedOfLight;
                    fu = float(dev::kTwoPi * (double(p[0]) * f - s.u0));
                    fv = float(dev::kTwoPi * (double(p[1]) * f - s.v0));
                    fw = float(dev::kTwoPi * (double(p[2]) * f - s.w0));
                }
                cu[i][r] = dup(fu);
                cv[i][r] = dup(fv);
                cw[i][r] = dup(fw);
            }
#pragma unroll
            for (int j = 0; j < 4; ++j) acc[i][j] = 0.0f;
        }
#pragma unroll 1
        for (int kb = 0; kb < NKB; ++kb) {
            const float4 b = frag_s[kb * 32 + lane];
            uint32_t bh[4], bl[4];
            split_tf32(b.x, b.y, bh[0], bh[1], bl[0], bl[1]);
            split_tf32(b.z, b.w, bh[2], bh[3], bl[2], bl[3]);
            const float4 lm = lmn_s[(kb * 4 + q) * 2], nn = lmn_s[(kb * 4 + q) * 2 + 1];
            const f2p l2 = pk(lm.x, lm.y), m2 = pk(lm.z, lm.w), n2 = pk(nn.x, nn.y);
            Frag4 ah[MT][2], al[MT][2];
#pragma unroll
            for (int i = 0; i < MT; ++i) {
                const float2 p0 = unpk(fma2(cu[i][0], l2, fma2(cv[i][0], m2, mul2(cw[i][0], n2))));  // row g
                const float2 p1 = unpk(fma2(cu[i][1], l2, fma2(cv[i][1], m2, mul2(cw[i][1], n2))));  // row g+8
                float sn[4], cs[4];
                __sincosf(p0.x, &sn[0], &cs[0]);  // row g,   pixel slot q
                __sincosf(p1.x, &sn[1], &cs[1]);  // row g+8, pixel slot q
                __sincosf(p0.y, &sn[2], &cs[2]);  // row g,   pixel slot q+4
                __sincosf(p1.y, &sn[3], &cs[3]);  // row g+8, pixel slot q+4
                make_frags(cs[0], sn[0], cs[1], sn[1], ah[i][0], al[i][0]);
                make_frags(cs[2], sn[2], cs[3], sn[3], ah[i][1], al[i][1]);
            }
#pragma unroll
            for (int hh = 0; hh < 2; ++hh) {
#pragma unroll
                for (int i = 0; i < MT; ++i)
                    mma1688(acc[i], ah[i][hh].c0, ah[i][hh].c1, ah[i][hh].s0, ah[i][hh].s1, bh[2 * hh], bh[2 * hh + 1]);
#pragma unroll
                for (int i = 0; i < MT; ++i)
                    mma1688(acc[i], ah[i][hh].c0, ah[i][hh].c1, ah[i][hh].s0, ah[i][hh].s1, bl[2 * hh], bl[2 * hh + 1]);
#pragma unroll
                for (int i = 0; i < MT; ++i)
                    mma1688(acc[i], al[i][hh].c0, al[i][hh].c1, al[i][hh].s0, al[i][hh].s1, bh[2 * hh], bh[2 * hh + 1]);
            }
        }
#pragma unroll
        for (int i = 0; i < MT; ++i) {
#pragma unroll
            for (int r = 0; r < 2; ++r) {
                const int v = (tile0 + i) * 16 + g + 8 * r;
                if (v < nvis) {
                    const int t = v / nc, c = v - t * nc;
                    vis0[int64_t(t) * row + c * 4 + q] = make_float2(acc[i][2 * r], acc[i][2 * r + 1]);
                }
            }
        }
    }
}

template <int NS, int WARPS, int MT, int MINB, int REC>
cudaError_t launch_gridder_tf32(const KernelArgs &a, cudaStream_t st) {
    const size_t smem = gridder_tf32_smem_bytes(NS, a.max_channels_in_item);
    cudaError_t err = dev::prepare(gridder_tf32_kernel<NS, WARPS, MT, MINB, REC>, smem);
    if (err != cudaSuccess) return err;
    LaunchScope scope("gridder", st);
    gridder_tf32_kernel<NS, WARPS, MT, MINB, REC><<<unsigned(a.nr_items), WARPS * 32, smem, st>>>(a);
    return cudaGetLastError();
}

template <int NS, int WARPS, int MT, int MINB>
cudaError_t launch_degridder_tf32(const KernelArgs &a, cudaStream_t st) {
    const size_t smem = degridder_tf32_smem_bytes(NS);
    cudaError_t err = dev::prepare(degridder_tf32_kernel<NS, WARPS, MT, MINB>, smem);
    if (err != cudaSuccess) return err;
    LaunchScope scope("degridder", st);
    degridder_tf32_kernel<NS, WARPS, MT, MINB><<<unsigned(a.nr_items), WARPS * 32, smem, st>>>(a);
    return cudaGetLastError();
}

#define G32(NS, W, MT, MB, R) \
    {NS, 8, kTensor, R, "gridder_tf32" #R "<" #NS ",W" #W ",MT" #MT ",minB" #MB ">", launch_gridder_tf32<NS, W, MT, MB, R>}
const Variant kTf32Gridder[] = {
    G32(24, 12, 3, 2, 1), G32(24, 6, 6, 2, 1), G32(24, 9, 4, 2, 1), G32(24, 18, 2, 1, 1),
    G32(24, 12, 3, 2, 0), G32(24, 6, 6, 2, 0), G32(24, 9, 4, 2, 0), G32(24, 18, 2, 1, 0),
    G32(32, 16, 4, 2, 1), G32(32, 8, 8, 2, 1), G32(32, 16, 4, 2, 0), G32(32, 8, 8, 2, 0),
    G32(16, 4, 4, 4, 1), G32(16, 8, 2, 3, 1), G32(16, 4, 4, 4, 0), G32(16, 8, 2, 3, 0),
};
#undef G32
#define D32(NS, W, MT, MB) \
    {NS, 0, kTensor, 0, "degridder_tf32<" #NS ",W" #W ",MT" #MT ",minB" #MB ">", launch_degridder_tf32<NS, W, MT, MB>}
const Variant kTf32Degridder[] = {
    D32(24, 8, 2, 3), D32(24, 8, 4, 2), D32(24, 4, 4, 4), D32(24, 16, 2, 1), D32(24, 8, 2, 4),
    D32(32, 8, 4, 2), D32(32, 8, 2, 3), D32(32, 16, 2, 1),
    D32(16, 8, 4, 2), D32(16, 8, 2, 3),
};
#undef D32

}  // namespace

const Variant *tf32_gridder_variants(int *n) {
    *n = int(sizeof(kTf32Gridder) / sizeof(kTf32Gridder[0]));
    return kTf32Gridder;
}

const Variant *tf32_degridder_variants(int *n) {
    *n = int(sizeof(kTf32Degridder) / sizeof(kTf32Degridder[0]));
    return kTf32Degridder;
}

}  // namespace idg
