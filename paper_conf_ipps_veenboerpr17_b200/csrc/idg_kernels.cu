// idg_kernels.cu -- sm_100a kernels of the IDG hot path (Veenboer, Petschow, Romein, IPDPS 2017).
//
//   gridder_kernel    one CTA per work item: Alg. 1 (pixel = direct sum of phase-
//                     shifted visibilities) -> A-term + taper (a3) -> centred subgrid DFT (a4)
//                     -> atomic adder into the grid (a5).  Fused: no subgrid round trip.
//   degridder_kernel  one CTA per work item: splitter (a6) -> centred inverse DFT (a7) ->
//                     taper + A-term (Alg. 2 lines 2-3) -> Alg. 2 over the item's visibilities (a9).
//
// Phases.  For visibility (t,c) of an item at subgrid pixel (l,m,n) (R-2, R-3):
//     phi = 2 pi [ (u_t f_c - u0) l + (v_t f_c - v0) m + (w_t f_c - w0) n ],  f_c = nu_c / c.
// fp32 cannot hold u_t f_c - u0 accurately when u_t f_c ~ N/(2L) (SURVEY 7 "hard parts"), so the
// phase is split around a reference frequency f_r of the item's channel block:
//     phi = B_t(l,m,n) + (f_c - f_r) Q_t(l,m,n)
//     B_t = 2 pi [(u_t f_r - u0) l + (v_t f_r - v0) m + (w_t f_r - w0) n]   (coefficients in fp64)
//     Q_t = 2 pi [ u_t l + v_t m + w_t n ]
// The small coefficients are formed in fp64 once per (item, timestep) and stored as fp32; per
// (pixel, visibility) pair the kernels then spend 1 FMA on the phase, one sincos (MUFU sin + cos
// after the FMUL range reduction) and 16 FMAs on the 2x2 complex multiply-accumulate: the paper's
// "17 real-valued FMA per sincos".
//
// n = 1 - sqrt(1 - l^2 - m^2) is evaluated as r^2 / (1 + sqrt(1 - r^2)) to avoid the fp32
// cancellation of the literal form (same value in exact arithmetic).
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdlib>
#include <cstring>
#include <string>

#include "idg_internal.h"

namespace idg {
namespace {

constexpr double kTwoPi = 6.283185307179586476925286766559;

__device__ __forceinline__ float2 cmul(float2 a, float2 b) {
    return make_float2(a.x * b.x - a.y * b.y, a.x * b.y + a.y * b.x);
}
__device__ __forceinline__ float2 cmulc(float2 a, float2 b) {  // conj(a) * b
    return make_float2(a.x * b.x + a.y * b.y, a.x * b.y - a.y * b.x);
}
__device__ __forceinline__ float2 cmul_conj_b(float2 a, float2 b) {  // a * conj(b)
    return make_float2(a.x * b.x + a.y * b.y, a.y * b.x - a.x * b.y);
}
__device__ __forceinline__ float2 cadd(float2 a, float2 b) { return make_float2(a.x + b.x, a.y + b.y); }
__device__ __forceinline__ float2 cscale(float2 a, float s) { return make_float2(a.x * s, a.y * s); }

__device__ __forceinline__ float w_term_n(float l, float m) {
    const float r2 = l * l + m * m;
    return r2 / (1.0f + sqrtf(1.0f - r2));  // == 1 - sqrt(1 - r2)
}

// Streaming 16-byte load that does not allocate in L1 (visibilities are read once per item).
__device__ __forceinline__ float4 ld_stream(const float4 *p) {
    float4 v;
    asm volatile("ld.global.nc.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];"
                 : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w)
                 : "l"(p));
    return v;
}

// Vector fp32 atomic add of one complex value (sm_90+: red.global.add.v2.f32).
__device__ __forceinline__ void red_add(float2 *addr, float2 v) {
    asm volatile("red.global.add.v2.f32 [%0], {%1, %2};" ::"l"(addr), "f"(v.x), "f"(v.y)
                 : "memory");
}

// Centred-DFT twiddle table tw[r] = exp(sign 2 pi i r / N~), r = 0..N~-1 (R-5).
template <int NS>
__device__ __forceinline__ void init_twiddles(float2 *tw, float sign) {
    for (int r = threadIdx.x; r < NS; r += blockDim.x) {
        float s, c;
        sincospif(2.0f * float(r) / float(NS), &s, &c);
        tw[r] = make_float2(c, sign * s);
    }
}

// exponent index ((k - N~/2) (x - N~/2)) mod N~ at x = 0, and its increment per x
template <int NS>
__device__ __forceinline__ void dft_index(int k, int &idx0, int &step) {
    constexpr int h = NS / 2;
    int e = (k - h) * (-h);
    idx0 = ((e % NS) + NS) % NS;
    step = ((k - h) % NS + NS) % NS;
}

struct ItemSetup {
    idg_metadata md;
    int nc;                 // channels in the item
    int st1, st2;           // stations of the baseline (A_p, A_q)
    double u0, v0, w0;      // uv(w) of the subgrid centre cell, wavelengths
    double f_ref;           // reference nu / c of the channel block, 1/m
};

__device__ __forceinline__ ItemSetup item_setup(const KernelArgs &a, int item, int NS) {
    ItemSetup s;
    s.md = a.items[item];
    s.nc = s.md.channel_end - s.md.channel_begin;
    s.st1 = a.baselines[2 * s.md.baseline];
    s.st2 = a.baselines[2 * s.md.baseline + 1];
    s.u0 = double(s.md.x + NS / 2 - a.grid_size / 2) * a.inv_image_size;
    s.v0 = double(s.md.y + NS / 2 - a.grid_size / 2) * a.inv_image_size;
    s.w0 = a.w_offset;
    s.f_ref = a.frequencies[s.md.channel_begin + s.nc / 2] / kSpeedOfLight;
    return s;
}

// B_t and Q_t coefficients (2 pi x wavelengths) of one timestep, formed in fp64.
__device__ __forceinline__ void timestep_coefficients(const KernelArgs &a, const ItemSetup &s,
                                                      int t, float4 &cB, float4 &cQ) {
    const float *p = a.uvw + (int64_t(s.md.baseline) * a.nr_timesteps + t) * 3;
    const float u = p[0], v = p[1], w = p[2];
    cB = make_float4(float(kTwoPi * (double(u) * s.f_ref - s.u0)),
                     float(kTwoPi * (double(v) * s.f_ref - s.v0)),
                     float(kTwoPi * (double(w) * s.f_ref - s.w0)), 0.0f);
    cQ = make_float4(float(kTwoPi * double(u)), float(kTwoPi * double(v)),
                     float(kTwoPi * double(w)), 0.0f);
}

// ------------------------------------------------------------------------------------------------
// Gridder: thread -> P pixels (strided by the CTA size so every pixel row is written coalesced);
// the item's visibilities stream through shared memory in batches of VB and are read back as
// warp-broadcasts; each thread accumulates its pixels in registers (P:216 items (1)-(3)).
// ------------------------------------------------------------------------------------------------
constexpr int kGridderBatch = 512;  // visibilities per shared-memory batch (16 KiB)

inline size_t gridder_smem_bytes(int NS, int max_channels) {
    const size_t main_loop = size_t(kGridderBatch) * 32 + size_t(kGridderBatch + 1) * 32 +
                             size_t(max_channels) * 4;
    const size_t epi = size_t(2) * 4 * NS * NS * sizeof(float2);
    return std::max(main_loop, epi) + 16;
}

template <int NS, int P, int MINB>
__global__ void __launch_bounds__(NS *NS / P, MINB) gridder_kernel(const KernelArgs a) {
    constexpr int NT = NS * NS / P;
    constexpr int NPIX = NS * NS;
    constexpr int h = NS / 2;
    constexpr int VB = kGridderBatch;
    extern __shared__ __align__(16) unsigned char smem[];
    float4 *vis_s = reinterpret_cast<float4 *>(smem);              // [2*VB]
    float4 *coef_s = vis_s + 2 * VB;                                 // [2*(VB+1)]
    float *df_s = reinterpret_cast<float *>(coef_s + 2 * (VB + 1));  // [nc]

    const int item = a.order[blockIdx.x];
    const ItemSetup s = item_setup(a, item, NS);
    const idg_metadata &md = s.md;
    const int nc = s.nc;
    const int nvis = md.nr_timesteps * nc;

    for (int c = threadIdx.x; c < nc; c += NT)
        df_s[c] = float((a.frequencies[md.channel_begin + c] / kSpeedOfLight) - s.f_ref);

    float l[P], m[P], n[P];
    float acc[P][8];
#pragma unroll
    for (int k = 0; k < P; ++k) {
        const int pix = threadIdx.x + k * NT;
        const int x = pix % NS, y = pix / NS;
        l[k] = float(x - h) * a.cell_l;
        m[k] = float(y - h) * a.cell_l;
        n[k] = w_term_n(l[k], m[k]);
#pragma unroll
        for (int j = 0; j < 8; ++j) acc[k][j] = 0.0f;
    }

    const int64_t row = int64_t(a.nr_channels) * 4;  // float2 per timestep
    const float2 *vis0 = a.vis + (int64_t(md.baseline) * a.nr_timesteps + md.time_offset) * row;
    const bool contiguous = (nc == a.nr_channels);

    for (int e0 = 0; e0 < nvis; e0 += VB) {
        const int e1 = min(e0 + VB, nvis);
        const int t_first = e0 / nc, t_last = (e1 - 1) / nc;
        __syncthreads();
        if (contiguous) {
            const float4 *src = reinterpret_cast<const float4 *>(vis0) + 2 * int64_t(e0);
            for (int i = threadIdx.x; i < 2 * (e1 - e0); i += NT) vis_s[i] = ld_stream(src + i);
        } else {
            for (int i = threadIdx.x; i < 2 * (e1 - e0); i += NT) {
                const int e = e0 + (i >> 1);
                const int t = e / nc, c = e - t * nc;
                const float4 *src = reinterpret_cast<const float4 *>(
                    vis0 + int64_t(t) * row + int64_t(md.channel_begin + c) * 4);
                vis_s[i] = ld_stream(src + (i & 1));
            }
        }
        for (int t = t_first + int(threadIdx.x); t <= t_last; t += NT) {
            float4 cB, cQ;
            timestep_coefficients(a, s, md.time_offset + t, cB, cQ);
            coef_s[2 * (t - t_first)] = cB;
            coef_s[2 * (t - t_first) + 1] = cQ;
        }
        __syncthreads();

        int e = e0;
        while (e < e1) {
            const int t = e / nc;
            const int c_begin = e - t * nc;
            const int c_end = min(nc, e1 - t * nc);
            const float4 cB = coef_s[2 * (t - t_first)];
            const float4 cQ = coef_s[2 * (t - t_first) + 1];
            float B[P], Q[P];
#pragma unroll
            for (int k = 0; k < P; ++k) {
                B[k] = fmaf(cB.x, l[k], fmaf(cB.y, m[k], cB.z * n[k]));
                Q[k] = fmaf(cQ.x, l[k], fmaf(cQ.y, m[k], cQ.z * n[k]));
            }
            const float4 *vrow = vis_s + 2 * (t * nc - e0);
#pragma unroll 2
            for (int c = c_begin; c < c_end; ++c) {
                const float4 va = vrow[2 * c];      // XX re, XX im, XY re, XY im
                const float4 vb = vrow[2 * c + 1];  // YX re, YX im, YY re, YY im
                const float df = df_s[c];
#pragma unroll
                for (int k = 0; k < P; ++k) {
                    const float ph = fmaf(df, Q[k], B[k]);
                    float sn, cs;
                    __sincosf(ph, &sn, &cs);
                    // S += V * exp(+i phi)  (Alg. 1, R-1)
                    acc[k][0] = fmaf(va.x, cs, acc[k][0]);
                    acc[k][1] = fmaf(va.x, sn, acc[k][1]);
                    acc[k][2] = fmaf(va.z, cs, acc[k][2]);
                    acc[k][3] = fmaf(va.z, sn, acc[k][3]);
                    acc[k][4] = fmaf(vb.x, cs, acc[k][4]);
                    acc[k][5] = fmaf(vb.x, sn, acc[k][5]);
                    acc[k][6] = fmaf(vb.z, cs, acc[k][6]);
                    acc[k][7] = fmaf(vb.z, sn, acc[k][7]);
                    acc[k][0] = fmaf(-va.y, sn, acc[k][0]);
                    acc[k][1] = fmaf(va.y, cs, acc[k][1]);
                    acc[k][2] = fmaf(-va.w, sn, acc[k][2]);
                    acc[k][3] = fmaf(va.w, cs, acc[k][3]);
                    acc[k][4] = fmaf(-vb.y, sn, acc[k][4]);
                    acc[k][5] = fmaf(vb.y, cs, acc[k][5]);
                    acc[k][6] = fmaf(-vb.w, sn, acc[k][6]);
                    acc[k][7] = fmaf(vb.w, cs, acc[k][7]);
                }
            }
            e = t * nc + c_end;
        }
    }

    // ---- epilogue: A-term + taper (a3), centred forward DFT (a4), adder (a5) -------------------
    __syncthreads();
    float2 *sub_s = reinterpret_cast<float2 *>(smem);  // [4][NS][NS]
    float2 *tmp_s = sub_s + 4 * NPIX;                  // [4][NS][NS]
    __shared__ float2 tw[NS];
    init_twiddles<NS>(tw, -1.0f);
    const float2 *Ap_base = a.aterms + ((int64_t(md.aterm_index) * a.nr_stations + s.st1) * NPIX) * 4;
    const float2 *Aq_base = a.aterms + ((int64_t(md.aterm_index) * a.nr_stations + s.st2) * NPIX) * 4;
#pragma unroll
    for (int k = 0; k < P; ++k) {
        const int pix = threadIdx.x + k * NT;
        const float4 *ap4 = reinterpret_cast<const float4 *>(Ap_base + int64_t(pix) * 4);
        const float4 *aq4 = reinterpret_cast<const float4 *>(Aq_base + int64_t(pix) * 4);
        const float4 ap01 = ap4[0], ap23 = ap4[1], aq01 = aq4[0], aq23 = aq4[1];
        const float2 p0 = make_float2(ap01.x, ap01.y), p1 = make_float2(ap01.z, ap01.w);
        const float2 p2 = make_float2(ap23.x, ap23.y), p3 = make_float2(ap23.z, ap23.w);
        const float2 q0 = make_float2(aq01.x, aq01.y), q1 = make_float2(aq01.z, aq01.w);
        const float2 q2 = make_float2(aq23.x, aq23.y), q3 = make_float2(aq23.z, aq23.w);
        const float2 s0 = make_float2(acc[k][0], acc[k][1]), s1 = make_float2(acc[k][2], acc[k][3]);
        const float2 s2 = make_float2(acc[k][4], acc[k][5]), s3 = make_float2(acc[k][6], acc[k][7]);
        // M = A_p^H S
        const float2 m0 = cadd(cmulc(p0, s0), cmulc(p2, s2));
        const float2 m1 = cadd(cmulc(p0, s1), cmulc(p2, s3));
        const float2 m2 = cadd(cmulc(p1, s0), cmulc(p3, s2));
        const float2 m3 = cadd(cmulc(p1, s1), cmulc(p3, s3));
        // R = sph * M A_q   (R-6: adjoint A-term in gridding)
        const float sph = a.taper[pix];
        sub_s[0 * NPIX + pix] = cscale(cadd(cmul(m0, q0), cmul(m1, q2)), sph);
        sub_s[1 * NPIX + pix] = cscale(cadd(cmul(m0, q1), cmul(m1, q3)), sph);
        sub_s[2 * NPIX + pix] = cscale(cadd(cmul(m2, q0), cmul(m3, q2)), sph);
        sub_s[3 * NPIX + pix] = cscale(cadd(cmul(m2, q1), cmul(m3, q3)), sph);
    }
    __syncthreads();
    // rows: tmp[pol][y][kx] = sum_x sub[pol][y][x] exp(-2 pi i (kx-h)(x-h)/N~)
    for (int o = threadIdx.x; o < 4 * NPIX; o += NT) {
        const int pol = o / NPIX, rem = o - pol * NPIX, y = rem / NS, kx = rem - y * NS;
        int idx, step;
        dft_index<NS>(kx, idx, step);
        const float2 *src = sub_s + pol * NPIX + y * NS;
        float2 sum = make_float2(0.0f, 0.0f);
#pragma unroll
        for (int x = 0; x < NS; ++x) {
            const float2 w = tw[idx];
            const float2 v = src[x];
            sum.x = fmaf(v.x, w.x, fmaf(-v.y, w.y, sum.x));
            sum.y = fmaf(v.x, w.y, fmaf(v.y, w.x, sum.y));
            idx += step;
            idx -= (idx >= NS) ? NS : 0;
        }
        tmp_s[o] = sum;
    }
    __syncthreads();
    // columns + adder: G[pol][y_j+ky][x_j+kx] += sum_y tmp[pol][y][kx] exp(-2 pi i (ky-h)(y-h)/N~)
    for (int o = threadIdx.x; o < 4 * NPIX; o += NT) {
        const int pol = o / NPIX, rem = o - pol * NPIX, ky = rem / NS, kx = rem - ky * NS;
        int idx, step;
        dft_index<NS>(ky, idx, step);
        const float2 *src = tmp_s + pol * NPIX + kx;
        float2 sum = make_float2(0.0f, 0.0f);
#pragma unroll
        for (int y = 0; y < NS; ++y) {
            const float2 w = tw[idx];
            const float2 v = src[y * NS];
            sum.x = fmaf(v.x, w.x, fmaf(-v.y, w.y, sum.x));
            sum.y = fmaf(v.x, w.y, fmaf(v.y, w.x, sum.y));
            idx += step;
            idx -= (idx >= NS) ? NS : 0;
        }
        float2 *dst = a.grid + (int64_t(pol) * a.grid_size + md.y + ky) * a.grid_size + md.x + kx;
        red_add(dst, sum);
    }
}

// ------------------------------------------------------------------------------------------------
// Degridder: thread -> V channels of one timestep (one visibility slot); all pixels of the
// (split, inverse-transformed, corrected) subgrid sit in shared memory as {l,m,n} + 4 complex and
// are read as warp broadcasts (the thread's "first mapping" = visibilities, the
// "second mapping" = pixels in the prologue).
// ------------------------------------------------------------------------------------------------
inline size_t degridder_smem_bytes(int NS, int max_channels) {
    const size_t npix = size_t(NS) * NS;
    const size_t region_a = std::max(npix * 48, npix * 4 * sizeof(float2));  // pixels | split sub
    const size_t region_b = npix * 4 * sizeof(float2);                         // row-pass buffer
    return region_a + region_b + size_t(max_channels) * 4 + 16;
}

template <int NS, int V, int NT, int MINB>
__global__ void __launch_bounds__(NT, MINB) degridder_kernel(const KernelArgs a) {
    constexpr int NPIX = NS * NS;
    constexpr int h = NS / 2;
    extern __shared__ __align__(16) unsigned char smem[];
    float4 *pix_s = reinterpret_cast<float4 *>(smem);                // [NPIX][3]   (region A)
    float2 *sub_s = reinterpret_cast<float2 *>(smem);                // [4][NS][NS] (region A)
    float2 *tmp_s = reinterpret_cast<float2 *>(smem + NPIX * 48);    // [4][NS][NS] (region B)
    float *df_s = reinterpret_cast<float *>(smem + NPIX * 48 + NPIX * 4 * sizeof(float2));
    __shared__ float2 tw[NS];

    const int item = a.order[blockIdx.x];
    const ItemSetup s = item_setup(a, item, NS);
    const idg_metadata &md = s.md;
    const int nc = s.nc;

    // a6 splitter: sub[pol][ky][kx] = G[pol][y_j+ky][x_j+kx]
    for (int o = threadIdx.x; o < 4 * NPIX; o += NT) {
        const int pol = o / NPIX, rem = o - pol * NPIX, ky = rem / NS, kx = rem - ky * NS;
        sub_s[o] = a.grid[(int64_t(pol) * a.grid_size + md.y + ky) * a.grid_size + md.x + kx];
    }
    for (int c = threadIdx.x; c < nc; c += NT)
        df_s[c] = float((a.frequencies[md.channel_begin + c] / kSpeedOfLight) - s.f_ref);
    init_twiddles<NS>(tw, +1.0f);
    __syncthreads();
    // a7 columns: tmp[pol][y][kx] = sum_ky sub[pol][ky][kx] exp(+2 pi i (ky-h)(y-h)/N~)
    for (int o = threadIdx.x; o < 4 * NPIX; o += NT) {
        const int pol = o / NPIX, rem = o - pol * NPIX, y = rem / NS, kx = rem - y * NS;
        int idx, step;
        dft_index<NS>(y, idx, step);
        const float2 *src = sub_s + pol * NPIX + kx;
        float2 sum = make_float2(0.0f, 0.0f);
#pragma unroll
        for (int ky = 0; ky < NS; ++ky) {
            const float2 w = tw[idx];
            const float2 v = src[ky * NS];
            sum.x = fmaf(v.x, w.x, fmaf(-v.y, w.y, sum.x));
            sum.y = fmaf(v.x, w.y, fmaf(v.y, w.x, sum.y));
            idx += step;
            idx -= (idx >= NS) ? NS : 0;
        }
        tmp_s[o] = sum;
    }
    __syncthreads();
    // a7 rows + Alg. 2 lines 2-3 (taper, A_p S A_q^H) -> pixel records {l, m, n, -}, S
    const float2 *Ap_base = a.aterms + ((int64_t(md.aterm_index) * a.nr_stations + s.st1) * NPIX) * 4;
    const float2 *Aq_base = a.aterms + ((int64_t(md.aterm_index) * a.nr_stations + s.st2) * NPIX) * 4;
    for (int pix = threadIdx.x; pix < NPIX; pix += NT) {
        const int y = pix / NS, x = pix - y * NS;
        int idx0, step;
        dft_index<NS>(x, idx0, step);
        float2 sv[4];
#pragma unroll
        for (int pol = 0; pol < 4; ++pol) {
            const float2 *src = tmp_s + pol * NPIX + y * NS;
            float2 sum = make_float2(0.0f, 0.0f);
            int idx = idx0;
#pragma unroll
            for (int kx = 0; kx < NS; ++kx) {
                const float2 w = tw[idx];
                const float2 v = src[kx];
                sum.x = fmaf(v.x, w.x, fmaf(-v.y, w.y, sum.x));
                sum.y = fmaf(v.x, w.y, fmaf(v.y, w.x, sum.y));
                idx += step;
                idx -= (idx >= NS) ? NS : 0;
            }
            sv[pol] = sum;
        }
        const float4 *ap4 = reinterpret_cast<const float4 *>(Ap_base + int64_t(pix) * 4);
        const float4 *aq4 = reinterpret_cast<const float4 *>(Aq_base + int64_t(pix) * 4);
        const float4 ap01 = ap4[0], ap23 = ap4[1], aq01 = aq4[0], aq23 = aq4[1];
        const float2 p0 = make_float2(ap01.x, ap01.y), p1 = make_float2(ap01.z, ap01.w);
        const float2 p2 = make_float2(ap23.x, ap23.y), p3 = make_float2(ap23.z, ap23.w);
        const float2 q0 = make_float2(aq01.x, aq01.y), q1 = make_float2(aq01.z, aq01.w);
        const float2 q2 = make_float2(aq23.x, aq23.y), q3 = make_float2(aq23.z, aq23.w);
        // M = A_p S ; R = sph * M A_q^H   (Eq. 1: A_p B A_q^H)
        const float2 m0 = cadd(cmul(p0, sv[0]), cmul(p1, sv[2]));
        const float2 m1 = cadd(cmul(p0, sv[1]), cmul(p1, sv[3]));
        const float2 m2 = cadd(cmul(p2, sv[0]), cmul(p3, sv[2]));
        const float2 m3 = cadd(cmul(p2, sv[1]), cmul(p3, sv[3]));
        const float sph = a.taper[pix];
        const float2 r0 = cscale(cadd(cmul_conj_b(m0, q0), cmul_conj_b(m1, q1)), sph);
        const float2 r1 = cscale(cadd(cmul_conj_b(m0, q2), cmul_conj_b(m1, q3)), sph);
        const float2 r2 = cscale(cadd(cmul_conj_b(m2, q0), cmul_conj_b(m3, q1)), sph);
        const float2 r3 = cscale(cadd(cmul_conj_b(m2, q2), cmul_conj_b(m3, q3)), sph);
        const float l = float(x - h) * a.cell_l, m = float(y - h) * a.cell_l;
        // region A is rewritten: sub_s is dead after the column pass (barrier above)
        pix_s[3 * pix + 0] = make_float4(l, m, w_term_n(l, m), 0.0f);
        pix_s[3 * pix + 1] = make_float4(r0.x, r0.y, r1.x, r1.y);
        pix_s[3 * pix + 2] = make_float4(r2.x, r2.y, r3.x, r3.y);
    }
    __syncthreads();

    // Alg. 2 lines 4-19: visibility slots = (timestep, group of V channels)
    const int groups = nc / V;
    const int nslots = md.nr_timesteps * groups;
    const int64_t row = int64_t(a.nr_channels) * 4;
    float2 *vis0 = a.vis + (int64_t(md.baseline) * a.nr_timesteps + md.time_offset) * row;
    for (int slot = threadIdx.x; slot < nslots; slot += NT) {
        const int t = slot / groups;
        const int c0 = (slot - t * groups) * V;
        float4 cB, cQ;
        timestep_coefficients(a, s, md.time_offset + t, cB, cQ);
        float df[V];
        float acc[V][8];
#pragma unroll
        for (int j = 0; j < V; ++j) {
            df[j] = df_s[c0 + j];
#pragma unroll
            for (int q = 0; q < 8; ++q) acc[j][q] = 0.0f;
        }
#pragma unroll 2
        for (int p = 0; p < NPIX; ++p) {
            const float4 lmn = pix_s[3 * p + 0];
            const float4 s01 = pix_s[3 * p + 1];
            const float4 s23 = pix_s[3 * p + 2];
            const float B = fmaf(cB.x, lmn.x, fmaf(cB.y, lmn.y, cB.z * lmn.z));
            const float Q = fmaf(cQ.x, lmn.x, fmaf(cQ.y, lmn.y, cQ.z * lmn.z));
#pragma unroll
            for (int j = 0; j < V; ++j) {
                const float ph = fmaf(df[j], Q, B);
                float sn, cs;
                __sincosf(ph, &sn, &cs);
                // V += S * exp(-i phi)  (alpha = -f.g)
                acc[j][0] = fmaf(s01.x, cs, acc[j][0]);
                acc[j][1] = fmaf(s01.y, cs, acc[j][1]);
                acc[j][2] = fmaf(s01.z, cs, acc[j][2]);
                acc[j][3] = fmaf(s01.w, cs, acc[j][3]);
                acc[j][4] = fmaf(s23.x, cs, acc[j][4]);
                acc[j][5] = fmaf(s23.y, cs, acc[j][5]);
                acc[j][6] = fmaf(s23.z, cs, acc[j][6]);
                acc[j][7] = fmaf(s23.w, cs, acc[j][7]);
                acc[j][0] = fmaf(s01.y, sn, acc[j][0]);
                acc[j][1] = fmaf(-s01.x, sn, acc[j][1]);
                acc[j][2] = fmaf(s01.w, sn, acc[j][2]);
                acc[j][3] = fmaf(-s01.z, sn, acc[j][3]);
                acc[j][4] = fmaf(s23.y, sn, acc[j][4]);
                acc[j][5] = fmaf(-s23.x, sn, acc[j][5]);
                acc[j][6] = fmaf(s23.w, sn, acc[j][6]);
                acc[j][7] = fmaf(-s23.z, sn, acc[j][7]);
            }
        }
        float4 *dst = reinterpret_cast<float4 *>(vis0 + int64_t(t) * row +
                                                 int64_t(md.channel_begin + c0) * 4);
#pragma unroll
        for (int j = 0; j < V; ++j) {
            dst[2 * j + 0] = make_float4(acc[j][0], acc[j][1], acc[j][2], acc[j][3]);
            dst[2 * j + 1] = make_float4(acc[j][4], acc[j][5], acc[j][6], acc[j][7]);
        }
    }
}

template <typename K>
cudaError_t prepare(K kernel, size_t smem) {
    cudaError_t err = cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
    if (err != cudaSuccess) return err;
    return cudaFuncSetAttribute(kernel, cudaFuncAttributePreferredSharedMemoryCarveout,
                                int(cudaSharedmemCarveoutMaxShared));
}

template <int NS, int P, int MINB>
cudaError_t launch_gridder_t(const KernelArgs &a, cudaStream_t st) {
    constexpr int NT = NS * NS / P;
    static_assert(NS * NS % (P * 32) == 0, "pixels per thread must give whole warps");
    const size_t smem = gridder_smem_bytes(NS, a.max_channels_in_item);
    cudaError_t err = prepare(gridder_kernel<NS, P, MINB>, smem);
    if (err != cudaSuccess) return err;
    LaunchScope scope("gridder", st);
    gridder_kernel<NS, P, MINB><<<unsigned(a.nr_items), NT, smem, st>>>(a);
    return cudaGetLastError();
}

template <int NS, int V, int NT, int MINB>
cudaError_t launch_degridder_t(const KernelArgs &a, cudaStream_t st) {
    const size_t smem = degridder_smem_bytes(NS, a.max_channels_in_item);
    cudaError_t err = prepare(degridder_kernel<NS, V, NT, MINB>, smem);
    if (err != cudaSuccess) return err;
    LaunchScope scope("degridder", st);
    degridder_kernel<NS, V, NT, MINB><<<unsigned(a.nr_items), NT, smem, st>>>(a);
    return cudaGetLastError();
}

using Launcher = cudaError_t (*)(const KernelArgs &, cudaStream_t);
struct Variant {
    int ns, v;            // subgrid size; pixels (gridder) or channels (degridder) per thread
    const char *name;
    Launcher fn;
};

// Launch-shape variants (tuned on B200 with scripts/tune.py; the first entry per (NS, V) is the default).
#define GV(NS, P, MB) {NS, 0, "gridder<" #NS ",P" #P ",minB" #MB ">", launch_gridder_t<NS, P, MB>}
const Variant kGridderVariants[] = {
    GV(24, 6, 4), GV(24, 6, 5), GV(24, 6, 6), GV(24, 3, 3), GV(24, 3, 4), GV(24, 2, 4), GV(24, 9, 3),
    GV(32, 4, 2), GV(32, 8, 3), GV(32, 8, 4), GV(32, 4, 3), GV(32, 16, 4),
    GV(16, 4, 4), GV(16, 4, 6), GV(16, 2, 4), GV(16, 8, 6),
};
#undef GV
#define DV(NS, V, NT, MB) {NS, V, "degridder<" #NS ",V" #V ",T" #NT ",minB" #MB ">", launch_degridder_t<NS, V, NT, MB>}
#define DV_ALL(NS) DV(NS, 8, 128, 4), DV(NS, 8, 128, 3), DV(NS, 8, 256, 1), DV(NS, 8, 256, 2), \
    DV(NS, 8, 64, 6), DV(NS, 8, 64, 8), DV(NS, 4, 128, 4), DV(NS, 4, 256, 3), DV(NS, 4, 128, 6), \
    DV(NS, 2, 128, 6), DV(NS, 1, 128, 6)
const Variant kDegridderVariants[] = {DV_ALL(24), DV_ALL(32), DV_ALL(16)};
#undef DV_ALL
#undef DV

// Variant choice: default = first match; env IDG_GRIDDER_VARIANT / IDG_DEGRIDDER_VARIANT = name
// overrides (tuning only).
template <size_t K>
const Variant *pick(const Variant (&table)[K], int ns, int v, const char *env) {
    const char *want = std::getenv(env);
    const Variant *first = nullptr;
    for (const Variant &var : table) {
        if (var.ns != ns) continue;
        // an override may use fewer channels per thread than the default, as long as it divides it
        const bool valid = (v == 0) ? var.v == 0 : (var.v > 0 && v % var.v == 0);
        if (valid && want && std::strcmp(want, var.name) == 0) return &var;
        if (!first && var.v == v) first = &var;
    }
    return first;
}

}  // namespace

cudaError_t launch_gridder(const KernelArgs &a, cudaStream_t s) {
    if (a.nr_items == 0) return cudaSuccess;
    const Variant *var = pick(kGridderVariants, a.subgrid_size, 0, "IDG_GRIDDER_VARIANT");
    return var ? var->fn(a, s) : cudaErrorInvalidValue;
}

// The channel count of every item must be a multiple of V (the host picks V from the plan).
int degridder_channels_per_thread(int channel_gcd) {
    if (channel_gcd % 8 == 0) return 8;
    if (channel_gcd % 4 == 0) return 4;
    if (channel_gcd % 2 == 0) return 2;
    return 1;
}

cudaError_t launch_degridder_v(const KernelArgs &a, int V, cudaStream_t s) {
    if (a.nr_items == 0) return cudaSuccess;
    const Variant *var = pick(kDegridderVariants, a.subgrid_size, V, "IDG_DEGRIDDER_VARIANT");
    return var ? var->fn(a, s) : cudaErrorInvalidValue;
}

const char *variant_names(int which) {
    static std::string g, d;
    if (g.empty()) {
        for (const Variant &v : kGridderVariants) g += std::string(v.name) + "\n";
        for (const Variant &v : kDegridderVariants) d += std::string(v.name) + "\n";
    }
    return which == 0 ? g.c_str() : d.c_str();
}

}  // namespace idg
