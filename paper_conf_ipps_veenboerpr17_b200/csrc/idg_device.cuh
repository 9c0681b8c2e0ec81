// idg_device.cuh -- device helpers shared by the SIMT kernels (idg_kernels.cu) and the tensor-core
// kernels (idg_kernels_tc.cu): complex arithmetic, phase coefficients, centred subgrid DFT passes,
// the gridder epilogue (a3 A-term + taper, a4 subgrid DFT, a5 adder) and the degridder prologue
// (a6 splitter, a7 inverse subgrid DFT, a8 taper + A-term).  See idg_kernels.cu for the phase model.
#pragma once

#include <cuda_runtime.h>

#include <cstdint>

#include "idg_internal.h"

namespace idg {
namespace dev {

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

// Grid element (plane z, pol, row y, column x): in the device-resident grid, or -- banded grid -- in the band
// of its owner, bands[y / R] (rows [r R, (r+1) R) of every [plane][pol], stored [planes][4][R][N]).
__device__ __forceinline__ float2 *grid_elem(const KernelArgs &a, int z, int pol, int y, int x) {
    if (a.bands) {
        const int r = y / a.band_rows, ly = y - r * a.band_rows;
        return a.bands[r] + ((int64_t(z) * 4 + pol) * a.band_rows + ly) * a.grid_size + x;
    }
    return a.grid + ((int64_t(z) * 4 + pol) * a.grid_size + y) * a.grid_size + x;
}
// The adder for one grid element.  Banded: the owner's band may be another GPU's memory (CUDA IPC over
// NVLink / NVSwitch), so the sum uses scalar fp32 reductions, which peer memory supports everywhere.
__device__ __forceinline__ void grid_add(const KernelArgs &a, int z, int pol, int y, int x, float2 v) {
    float2 *p = grid_elem(a, z, pol, y, x);
    if (a.bands) {
        asm volatile("red.global.add.f32 [%0], %1;" ::"l"(&p->x), "f"(v.x) : "memory");
        asm volatile("red.global.add.f32 [%0], %1;" ::"l"(&p->y), "f"(v.y) : "memory");
    } else {
        red_add(p, v);
    }
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
    s.w0 = a.w_offset + (double(s.md.z) - double(a.nr_w_planes - 1) / 2.0) * a.w_step;  // W-plane (R-21)
    s.f_ref = a.frequencies[s.md.channel_begin + s.nc / 2] / kSpeedOfLight;
    return s;
}

// B_t and Q_t coefficients (2 pi x wavelengths) of one timestep, formed in fp64.
__device__ __forceinline__ void timestep_coefficients_uvw(const ItemSetup &s, float u, float v, float w,
                                                          float4 &cB, float4 &cQ) {
    cB = make_float4(float(kTwoPi * (double(u) * s.f_ref - s.u0)),
                     float(kTwoPi * (double(v) * s.f_ref - s.v0)),
                     float(kTwoPi * (double(w) * s.f_ref - s.w0)), 0.0f);
    cQ = make_float4(float(kTwoPi * double(u)), float(kTwoPi * double(v)),
                     float(kTwoPi * double(w)), 0.0f);
}
__device__ __forceinline__ void timestep_coefficients(const KernelArgs &a, const ItemSetup &s,
                                                      int t, float4 &cB, float4 &cQ) {
    const float *p = a.uvw + (int64_t(s.md.baseline) * a.nr_timesteps + t) * 3;
    timestep_coefficients_uvw(s, p[0], p[1], p[2], cB, cQ);
}


// a3 for one pixel, in place: sub_s[pol][pix] <- sph * A_p^H S A_q (R-6).  Returns max |component|.
template <int NS>
__device__ __forceinline__ float gridder_aterm_pixel(const KernelArgs &a, const ItemSetup &s, float2 *sub_s, int pix) {
    constexpr int NPIX = NS * NS;
    const idg_metadata &md = s.md;
    const float2 *Ap_base = a.aterms + ((int64_t(md.aterm_index) * a.nr_stations + s.st1) * NPIX) * 4;
    const float2 *Aq_base = a.aterms + ((int64_t(md.aterm_index) * a.nr_stations + s.st2) * NPIX) * 4;
    const float4 *ap4 = reinterpret_cast<const float4 *>(Ap_base + int64_t(pix) * 4);
    const float4 *aq4 = reinterpret_cast<const float4 *>(Aq_base + int64_t(pix) * 4);
    const float4 ap01 = ap4[0], ap23 = ap4[1], aq01 = aq4[0], aq23 = aq4[1];
    const float2 p0 = make_float2(ap01.x, ap01.y), p1 = make_float2(ap01.z, ap01.w);
    const float2 p2 = make_float2(ap23.x, ap23.y), p3 = make_float2(ap23.z, ap23.w);
    const float2 q0 = make_float2(aq01.x, aq01.y), q1 = make_float2(aq01.z, aq01.w);
    const float2 q2 = make_float2(aq23.x, aq23.y), q3 = make_float2(aq23.z, aq23.w);
    const float2 s0 = sub_s[0 * NPIX + pix], s1 = sub_s[1 * NPIX + pix];
    const float2 s2 = sub_s[2 * NPIX + pix], s3 = sub_s[3 * NPIX + pix];
    // M = A_p^H S
    const float2 m0 = cadd(cmulc(p0, s0), cmulc(p2, s2));
    const float2 m1 = cadd(cmulc(p0, s1), cmulc(p2, s3));
    const float2 m2 = cadd(cmulc(p1, s0), cmulc(p3, s2));
    const float2 m3 = cadd(cmulc(p1, s1), cmulc(p3, s3));
    // R = sph * M A_q
    const float sph = a.taper[pix];
    const float2 r0 = cscale(cadd(cmul(m0, q0), cmul(m1, q2)), sph);
    const float2 r1 = cscale(cadd(cmul(m0, q1), cmul(m1, q3)), sph);
    const float2 r2 = cscale(cadd(cmul(m2, q0), cmul(m3, q2)), sph);
    const float2 r3 = cscale(cadd(cmul(m2, q1), cmul(m3, q3)), sph);
    sub_s[0 * NPIX + pix] = r0;
    sub_s[1 * NPIX + pix] = r1;
    sub_s[2 * NPIX + pix] = r2;
    sub_s[3 * NPIX + pix] = r3;
    return fmaxf(fmaxf(fmaxf(fabsf(r0.x), fabsf(r0.y)), fmaxf(fabsf(r1.x), fabsf(r1.y))),
                 fmaxf(fmaxf(fabsf(r2.x), fabsf(r2.y)), fmaxf(fabsf(r3.x), fabsf(r3.y))));
}

// ------------------------------------------------------------------------------------------------
// a3 + a4 + a5 (gridder epilogue).  On entry (after a barrier) sub_s[pol][pix] holds the raw image-
// domain sums S of the item.  Applies sph * A_p^H S A_q per pixel (R-6), the centred forward DFT
// (rows, then columns, R-5) and adds the transformed subgrid to the grid with vector fp32 atomics.
// ------------------------------------------------------------------------------------------------
template <int NS>
__device__ __forceinline__ void gridder_epilogue(const KernelArgs &a, const ItemSetup &s, float2 *sub_s,
                                                 float2 *tmp_s, float2 *tw) {
    constexpr int NPIX = NS * NS;
    const int nt = blockDim.x;
    const idg_metadata &md = s.md;
    init_twiddles<NS>(tw, -1.0f);
    for (int pix = threadIdx.x; pix < NPIX; pix += nt) gridder_aterm_pixel<NS>(a, s, sub_s, pix);
    __syncthreads();
    // rows: tmp[pol][y][kx] = sum_x sub[pol][y][x] exp(-2 pi i (kx-h)(x-h)/N~)
    for (int o = threadIdx.x; o < 4 * NPIX; o += nt) {
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
    for (int o = threadIdx.x; o < 4 * NPIX; o += nt) {
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
        if (a.subgrids) {   // host adder: store into the item's slot of the subgrid buffer
            a.subgrids[int64_t(blockIdx.x) * 4 * NPIX + o] = sum;
            continue;
        }
        grid_add(a, md.z, pol, md.y + ky, md.x + kx, sum);
    }
    if (a.bands) __threadfence_system();   // the peer-memory adds are visible before the kernel completes
}

// ------------------------------------------------------------------------------------------------
// a6 + a7 (first half): splitter into sub_s, inverse-DFT columns into tmp_s.  Ends with a barrier.
// ------------------------------------------------------------------------------------------------
template <int NS>
__device__ __forceinline__ void degridder_split_columns(const KernelArgs &a, const ItemSetup &s,
                                                        float2 *sub_s, float2 *tmp_s, float2 *tw) {
    constexpr int NPIX = NS * NS;
    const int nt = blockDim.x;
    const idg_metadata &md = s.md;
    for (int o = threadIdx.x; o < 4 * NPIX; o += nt) {
        const int pol = o / NPIX, rem = o - pol * NPIX, ky = rem / NS, kx = rem - ky * NS;
        sub_s[o] = a.subgrids ? a.subgrids[int64_t(blockIdx.x) * 4 * NPIX + o]   // host splitter
                              : *grid_elem(a, md.z, pol, md.y + ky, md.x + kx);
    }
    init_twiddles<NS>(tw, +1.0f);
    __syncthreads();
    // tmp[pol][y][kx] = sum_ky sub[pol][ky][kx] exp(+2 pi i (ky-h)(y-h)/N~)
    for (int o = threadIdx.x; o < 4 * NPIX; o += nt) {
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
}

template <int NS>
__device__ __forceinline__ void degridder_aterm_pixel(const KernelArgs &a, const ItemSetup &s, const float2 sv[4],
                                                      int pix, float2 r[4]);

// a7 (second half) + a8 for one pixel: inverse-DFT row, then sph * A_p S A_q^H (Alg. 2 lines 2-3).
template <int NS>
__device__ __forceinline__ void degridder_pixel(const KernelArgs &a, const ItemSetup &s, const float2 *tmp_s,
                                                const float2 *tw, int pix, float2 r[4]) {
    constexpr int NPIX = NS * NS;
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
    degridder_aterm_pixel<NS>(a, s, sv, pix, r);
}

// a8 for one pixel: r = sph * A_p S A_q^H (Alg. 2 lines 2-3; Eq. 1: A_p B A_q^H).
template <int NS>
__device__ __forceinline__ void degridder_aterm_pixel(const KernelArgs &a, const ItemSetup &s, const float2 sv[4],
                                                      int pix, float2 r[4]) {
    constexpr int NPIX = NS * NS;
    const idg_metadata &md = s.md;
    const float2 *Ap_base = a.aterms + ((int64_t(md.aterm_index) * a.nr_stations + s.st1) * NPIX) * 4;
    const float2 *Aq_base = a.aterms + ((int64_t(md.aterm_index) * a.nr_stations + s.st2) * NPIX) * 4;
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
    r[0] = cscale(cadd(cmul_conj_b(m0, q0), cmul_conj_b(m1, q1)), sph);
    r[1] = cscale(cadd(cmul_conj_b(m0, q2), cmul_conj_b(m1, q3)), sph);
    r[2] = cscale(cadd(cmul_conj_b(m2, q0), cmul_conj_b(m3, q1)), sph);
    r[3] = cscale(cadd(cmul_conj_b(m2, q2), cmul_conj_b(m3, q3)), sph);
}

template <typename K>
inline cudaError_t prepare(K kernel, size_t smem) {
    cudaError_t err = cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
    if (err != cudaSuccess) return err;
    return cudaFuncSetAttribute(kernel, cudaFuncAttributePreferredSharedMemoryCarveout,
                                int(cudaSharedmemCarveoutMaxShared));
}

}  // namespace dev
}  // namespace idg
