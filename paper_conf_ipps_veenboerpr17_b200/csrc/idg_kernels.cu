// idg_kernels.cu -- SIMT sm_100a kernels of the IDG hot path (Veenboer, Petschow, Romein, IPDPS 2017)
// and the launch-variant dispatch (SIMT + tensor-core kernels of idg_kernels_tc.cu).
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
#include <atomic>
#include <cstdlib>
#include <cstring>
#include <string>
#include <vector>

#include "idg_device.cuh"
#include "idg_internal.h"

namespace idg {
namespace {

constexpr double kTwoPi = dev::kTwoPi;

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
    const dev::ItemSetup s = dev::item_setup(a, item, NS);
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
        n[k] = dev::w_term_n(l[k], m[k]);
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
            for (int i = threadIdx.x; i < 2 * (e1 - e0); i += NT) vis_s[i] = dev::ld_stream(src + i);
        } else {
            for (int i = threadIdx.x; i < 2 * (e1 - e0); i += NT) {
                const int e = e0 + (i >> 1);
                const int t = e / nc, c = e - t * nc;
                const float4 *src = reinterpret_cast<const float4 *>(
                    vis0 + int64_t(t) * row + int64_t(md.channel_begin + c) * 4);
                vis_s[i] = dev::ld_stream(src + (i & 1));
            }
        }
        for (int t = t_first + int(threadIdx.x); t <= t_last; t += NT) {
            float4 cB, cQ;
            dev::timestep_coefficients(a, s, md.time_offset + t, cB, cQ);
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
#pragma unroll
    for (int k = 0; k < P; ++k) {
        const int pix = threadIdx.x + k * NT;
#pragma unroll
        for (int pol = 0; pol < 4; ++pol) sub_s[pol * NPIX + pix] = make_float2(acc[k][2 * pol], acc[k][2 * pol + 1]);
    }
    __syncthreads();
    dev::gridder_epilogue<NS>(a, s, sub_s, tmp_s, tw);
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
    const dev::ItemSetup s = dev::item_setup(a, item, NS);
    const idg_metadata &md = s.md;
    const int nc = s.nc;

    for (int c = threadIdx.x; c < nc; c += NT)
        df_s[c] = float((a.frequencies[md.channel_begin + c] / kSpeedOfLight) - s.f_ref);
    dev::degridder_split_columns<NS>(a, s, sub_s, tmp_s, tw);
    // a7 rows + Alg. 2 lines 2-3 -> pixel records {l, m, n, -}, S (region A: sub_s is dead now)
    for (int pix = threadIdx.x; pix < NPIX; pix += NT) {
        float2 r[4];
        dev::degridder_pixel<NS>(a, s, tmp_s, tw, pix, r);
        const int y = pix / NS, x = pix - y * NS;
        const float l = float(x - h) * a.cell_l, m = float(y - h) * a.cell_l;
        pix_s[3 * pix + 0] = make_float4(l, m, dev::w_term_n(l, m), 0.0f);
        pix_s[3 * pix + 1] = make_float4(r[0].x, r[0].y, r[1].x, r[1].y);
        pix_s[3 * pix + 2] = make_float4(r[2].x, r[2].y, r[3].x, r[3].y);
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
        dev::timestep_coefficients(a, s, md.time_offset + t, cB, cQ);
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

template <int NS>
size_t smem_gridder_t(const KernelArgs &a) { return gridder_smem_bytes(NS, a.max_channels_in_item); }
template <int NS>
size_t smem_degridder_t(const KernelArgs &a) { return degridder_smem_bytes(NS, a.max_channels_in_item); }

template <int NS, int P, int MINB>
cudaError_t launch_gridder_t(const KernelArgs &a, cudaStream_t st) {
    constexpr int NT = NS * NS / P;
    static_assert(NS * NS % (P * 32) == 0, "pixels per thread must give whole warps");
    const size_t smem = gridder_smem_bytes(NS, a.max_channels_in_item);
    cudaError_t err = dev::prepare(gridder_kernel<NS, P, MINB>, smem);
    if (err != cudaSuccess) return err;
    LaunchScope scope("gridder", st);
    gridder_kernel<NS, P, MINB><<<unsigned(a.nr_items), NT, smem, st>>>(a);
    return cudaGetLastError();
}

template <int NS, int V, int NT, int MINB>
cudaError_t launch_degridder_t(const KernelArgs &a, cudaStream_t st) {
    const size_t smem = degridder_smem_bytes(NS, a.max_channels_in_item);
    cudaError_t err = dev::prepare(degridder_kernel<NS, V, NT, MINB>, smem);
    if (err != cudaSuccess) return err;
    LaunchScope scope("degridder", st);
    degridder_kernel<NS, V, NT, MINB><<<unsigned(a.nr_items), NT, smem, st>>>(a);
    return cudaGetLastError();
}

// SIMT variants (the paper's kernel structure on the CUDA cores; launch shapes tuned with scripts/tune.py).
// v = channels per thread for the degridder (every item's channel count must be a multiple of v).
#define GV(NS, P, MB) {NS, 0, kSimt, 0, "gridder<" #NS ",P" #P ",minB" #MB ">", launch_gridder_t<NS, P, MB>, 0, \
                       smem_gridder_t<NS>}
const Variant kGridderVariants[] = {GV(24, 6, 4), GV(32, 4, 2), GV(16, 4, 4)};
#undef GV
#define DV(NS, V, NT, MB) {NS, V, kSimt, 0, "degridder<" #NS ",V" #V ",T" #NT ",minB" #MB ">", \
                           launch_degridder_t<NS, V, NT, MB>, 0, smem_degridder_t<NS>}
#define DV_ALL(NS) DV(NS, 8, 128, 4), DV(NS, 4, 128, 4), DV(NS, 2, 128, 6), DV(NS, 1, 128, 6)
const Variant kDegridderVariants[] = {DV_ALL(24), DV_ALL(32), DV_ALL(16)};
#undef DV_ALL
#undef DV

// Opt-in dynamic shared memory limit of the current device (cached per device).
size_t max_dynamic_smem() {
    static std::atomic<int> cache[64];
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) return 0;
    int v = cache[dev].load();
    if (v == 0) {
        if (cudaDeviceGetAttribute(&v, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev) != cudaSuccess) return 0;
        cache[dev].store(v);
    }
    return size_t(v);
}

bool eligible(const Variant &var, const KernelArgs &a) {
    if (var.ns != a.subgrid_size) return false;
    if (var.needs_uniform && !a.channels_uniform) return false;
    if (var.max_channels > 0 && a.max_channels_in_item > var.max_channels) return false;
    if (var.v != 0 && a.channel_gcd % var.v != 0) return false;
    if (var.max_mean_timesteps > 0 && a.mean_timesteps_in_item > float(var.max_mean_timesteps)) return false;
    // shared memory grows with the plan's largest item (T~ for the degridders, C~ for the gridders): a
    // variant whose launch would not fit is skipped, so a kernel that fits (ultimately SIMT) runs instead
    if (var.smem) {
        const size_t lim = max_dynamic_smem();
        if (lim > 0 && var.smem(a) > lim) return false;
    }
    return true;
}

// Variant choice.  Default: the first eligible tensor-core variant, else the first eligible SIMT
// variant (for the SIMT degridder: the one with the largest channels-per-thread).  The environment
// variable `env` (IDG_GRIDDER_VARIANT / IDG_DEGRIDDER_VARIANT) may name any eligible variant (tuning).
const Variant *pick(const Variant *simt, int nsimt, const std::vector<const Variant *> &tc, const KernelArgs &a,
                    const char *env) {
    const char *want = std::getenv(env);
    if (want && *want) {
        // exact name, or a prefix ending in '*' (first eligible match)
        const size_t len = std::strlen(want);
        const bool prefix = want[len - 1] == '*';
        auto match = [&](const char *name) {
            return prefix ? std::strncmp(want, name, len - 1) == 0 : std::strcmp(want, name) == 0;
        };
        for (const Variant *v : tc)
            if (eligible(*v, a) && match(v->name)) return v;
        for (int i = 0; i < nsimt; ++i)
            if (eligible(simt[i], a) && match(simt[i].name)) return &simt[i];
    }
    // "tc": the direct tensor-core kernel (no channel recurrence); "simt": the CUDA-core kernel
    const bool tc_direct = want && std::strcmp(want, "tc") == 0;
    if (!(want && std::strcmp(want, "simt") == 0))
        for (const Variant *v : tc)
            if (eligible(*v, a) && !(tc_direct && v->needs_uniform)) return v;
    const Variant *best = nullptr;
    for (int i = 0; i < nsimt; ++i)
        if (eligible(simt[i], a) && (!best || simt[i].v > best->v)) best = &simt[i];
    return best;
}

// All tensor-core variants in default-preference order (measured on B200).
const std::vector<const Variant *> &tensor_variants(int which) {
    static const std::vector<const Variant *> lists[2] = {
        [] {
            std::vector<const Variant *> v;
            int n = 0;
            const Variant *t = tc_gridder_variants(&n);
            for (int i = 0; i < n; ++i) v.push_back(&t[i]);
            return v;
        }(),
        [] {
            std::vector<const Variant *> v;
            int n = 0;
            const Variant *t = tc_degridder_variants(&n);
            for (int i = 0; i < n; ++i) v.push_back(&t[i]);
            return v;
        }()};
    return lists[which];
}

}  // namespace

std::atomic<const char *> g_last_variant[2] = {"", ""};

// Dropped visibilities are predicted as 0 (R-12, R-13): one CTA per run (grid-stride), 16-byte stores.
__global__ void __launch_bounds__(256) zero_ranges_kernel(float4 *vis, const int64_t *ranges, int64_t nr,
                                                          int64_t base) {
    for (int64_t r = blockIdx.x; r < nr; r += gridDim.x) {
        float4 *p = vis + 2 * (ranges[2 * r] - base);
        const int64_t n = 2 * ranges[2 * r + 1];   // a visibility is 4 complex64 = 2 float4
        for (int64_t i = threadIdx.x; i < n; i += blockDim.x) p[i] = make_float4(0.0f, 0.0f, 0.0f, 0.0f);
    }
}

cudaError_t launch_zero_ranges(float2 *vis, const int64_t *ranges, int64_t nr, int64_t base, cudaStream_t s) {
    if (nr <= 0) return cudaSuccess;
    LaunchScope scope("zero_dropped", s);
    const unsigned blocks = unsigned(std::min<int64_t>(nr, 148 * 16));
    zero_ranges_kernel<<<blocks, 256, 0, s>>>(reinterpret_cast<float4 *>(vis), ranges, nr, base);
    return cudaGetLastError();
}

cudaError_t launch_gridder(const KernelArgs &a, cudaStream_t s) {
    if (a.nr_items == 0) return cudaSuccess;
    const Variant *var = pick(kGridderVariants, int(std::size(kGridderVariants)), tensor_variants(0), a,
                              "IDG_GRIDDER_VARIANT");
    if (!var) return cudaErrorInvalidValue;
    g_last_variant[0].store(var->name);
    return var->fn(a, s);
}

cudaError_t launch_degridder(const KernelArgs &a, cudaStream_t s) {
    if (a.nr_items == 0) return cudaSuccess;
    const Variant *var = pick(kDegridderVariants, int(std::size(kDegridderVariants)), tensor_variants(1), a,
                              "IDG_DEGRIDDER_VARIANT");
    if (!var) return cudaErrorInvalidValue;
    g_last_variant[1].store(var->name);
    return var->fn(a, s);
}

const char *last_variant(int which) { return g_last_variant[which == 0 ? 0 : 1].load(); }

const char *variant_names(int which) {
    static std::string names[2];
    if (names[0].empty()) {
        for (const Variant *v : tensor_variants(0)) names[0] += std::string(v->name) + "\n";
        for (const Variant &v : kGridderVariants) names[0] += std::string(v.name) + "\n";
        for (const Variant *v : tensor_variants(1)) names[1] += std::string(v->name) + "\n";
        for (const Variant &v : kDegridderVariants) names[1] += std::string(v.name) + "\n";
    }
    return names[which == 0 ? 0 : 1].c_str();
}

}  // namespace idg
