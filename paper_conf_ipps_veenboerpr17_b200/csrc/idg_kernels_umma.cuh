// idg_kernels_umma.cuh -- the rotation gridder on the 5th-generation tensor cores (tcgen05 / TMEM), sm_100a.
// Veenboer et al. 2017, Alg. 1 + the channel-group rotation of gridder_rot2 (idg_kernels_tc.cu).
//
// Per work item and timestep t, with channels c = 8j + s (group j = 0..J-1, slot s = 0..7, uniform spacing):
//     S(pixel) += sum_j E_t^j D_j,   D_j = sum_s Phi(t, s) V(t, 8j + s),   E_t = exp(i 8 dnu/c Q_t(pixel))
// (exact in exact arithmetic; R-1, R-2).  All J products D_j share the same A operand (the 8 slot phasors of
// every pixel), so they are ONE tensor-core product with N = 8 J columns (4 pols x re/im per group): N = 32
// for the SKA-shaped items (J = 4), N = 16 for predict (J = 2).
//
//   * A cluster of two CTAs per item (see below), 512 threads = 4 tiles of 128 pixel rows each, one row per
//     thread.  Per timestep every thread forms its pixel's 8 slot phasors (phase FMA, MUFU sincos), splits
//     them into f16 hi + lo (x = hi + lo to ~22 bits, as the mma.sync kernels) and stores the two A rows into
//     a 2-stage shared-memory ring in the canonical K-major no-swizzle layout (8 x 16 B core matrices).
//   * The first thread of each tile waits for its 128 rows (mbarrier), issues 3 UMMAs
//     (M = 128, N = 8 J, K = 16; A and B from shared memory): D = A_hi B_hi, D += A_hi B_lo, D += A_lo B_hi
//     into the tile's TMEM stage, and commits them to the stage's mbarrier (issue distributed over the tiles).
//   * One timestep later each thread reads its row of D back (tcgen05.ld) and sums the groups in Horner form,
//     D_0 + E (D_1 + E (D_2 + E D_3)) (FFMA2, complex multiply-add per pol), into fp32 registers.
//   * Visibilities: one power-of-two f16 range scale per item (a pre-pass over its visibilities), batches of
//     kUrTpb timesteps prefetched into registers two batches ahead and staged (split B tiles + the timestep's
//     uvw coefficients) one batch ahead into a 4-slot ring guarded by ready / empty mbarriers -- no CTA-wide
//     barrier inside the loop.
//   * Epilogue: a3 per pixel, the halves exchange polarisations over distributed shared memory, each CTA runs
//     the tensor-core subgrid DFT (a4) and the atomic adder (a5) -- or the host adder's subgrid buffer -- for
//     two polarisations.
// Measured (SKA-T1024, r02t-r02w): 140.3 ms against 135.7 ms for gridder_rot2h (mma.sync), so it is selected
// by name only.  The loop runs at ~2600 clk per (SM, timestep) -- the probe's ceiling for this structure;
// tcgen05.ld of the 32 D columns of every pixel and timestep (128 KB per SM-timestep) bounds it.
// Included by idg_kernels_tc.cu inside namespace idg::{anonymous}: it shares that translation unit's split /
// scale helpers, the tensor-core DFT, the DFT tables and the f32x2 helpers.
#pragma once

__device__ __forceinline__ uint32_t smem_u32(const void *p) { return static_cast<uint32_t>(__cvta_generic_to_shared(p)); }

// K-major, no-swizzle UMMA shared-memory descriptor: element (row, k) at
// (row/8)*SBO + (k/8)*LBO + (row%8)*16 + (k%8)*2 bytes from the start address.
__device__ __forceinline__ uint64_t umma_desc(uint32_t saddr) {
    constexpr uint32_t lbo = 128, sbo = 256;
    return uint64_t((saddr >> 4) & 0x3fff) | (uint64_t((lbo >> 4) & 0x3fff) << 16) |
           (uint64_t((sbo >> 4) & 0x3fff) << 32) | (uint64_t(1) << 46);
}

template <int N>
__device__ __forceinline__ void umma_f16(uint32_t tmem_d, uint64_t da, uint64_t db, uint32_t accumulate) {
    // kind::f16 instruction descriptor: D f32, A/B f16, both K-major, N, M = 128
    constexpr uint32_t idesc = (1u << 4) | (uint32_t(N >> 3) << 17) | (uint32_t(128 >> 4) << 24);
    asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\n"
                 "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}" ::"r"(tmem_d),
                 "l"(da), "l"(db), "r"(idesc), "r"(accumulate));
}

__device__ __forceinline__ void mbar_wait(uint64_t *bar, uint32_t parity) {
    const uint32_t addr = smem_u32(bar);
    uint32_t done = 0;
    do {
        asm volatile("{\n.reg .pred P;\nmbarrier.try_wait.parity.shared::cta.b64 P, [%1], %2;\nselp.u32 %0, 1, 0, P;\n}"
                     : "=r"(done) : "r"(addr), "r"(parity) : "memory");
    } while (!done);
}

// 16 TMEM columns of this thread's lane -> registers (no wait)
__device__ __forceinline__ void tmem_ld16(uint32_t taddr, uint32_t (&r)[16]) {
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
                 : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
                   "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
                 : "r"(taddr));
}
__device__ __forceinline__ void tmem_wait_ld() { asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory"); }

__device__ __forceinline__ f2p pk_u(uint32_t lo, uint32_t hi) {
    f2p r;
    asm("mov.b64 %0, {%1, %2};" : "=l"(r) : "r"(lo), "r"(hi));
    return r;
}
__device__ __forceinline__ f2p swp(f2p v) {   // (x, y) -> (y, x)
    f2p r;
    asm("{\n.reg .b32 x, y;\nmov.b64 {x, y}, %1;\nmov.b64 %0, {y, x};\n}" : "=l"(r) : "l"(v));
    return r;
}

// h <- D + E h for the 4 pols, packed (re, im): (er hr + dr, er hi + di) then + (-ei hi, ei hr)
// (two FFMA2 per pol; e = (er, er), ne = (-ei, ei))
__device__ __forceinline__ void horner_step2(f2p (&h)[4], const uint32_t *d, f2p e, f2p ne) {
#pragma unroll
    for (int p = 0; p < 4; ++p) h[p] = fma2(ne, swp(h[p]), fma2(e, h[p], pk_u(d[2 * p], d[2 * p + 1])));
}

// A cluster of two CTAs per item, 4 tiles (512 pixel rows) each: 256 TMEM columns and ~105 KB of shared
// memory per CTA, so two CTAs (of different items) share an SM and one's pre-pass / epilogue overlaps the
// other's loop.  (One 1024-thread CTA per item holds all 512 TMEM columns and ~193 KB, one CTA per SM: its
// per-item work is exposed -- measured 151.6 against 140.3 ms, r02v / r02w.)  The halves meet in the
// epilogue through distributed shared memory: after a3, which mixes the polarisations of a pixel, each CTA
// sends the other the two polarisations that one transforms and adds (a4 + a5).
constexpr int kUrTiles = 4;                  // 128-row tiles per CTA
constexpr int kUrThreads = kUrTiles * 128;   // one pixel row per thread
constexpr int kUrTpb = 5;                    // timesteps per visibility batch (r02w: 4 -> 5: 143.5 -> 140.3 ms)
constexpr int kUrBufs = 4;                   // batch ring: staged one batch ahead, reused three batches later
constexpr int kUrStages = 2;                 // A (shared) and D (TMEM) stages

inline size_t gridder_umma_rot_smem_bytes(int kpt) {
    const size_t a_ring = size_t(kUrStages) * kUrTiles * 8192;                 // hi 4 KB + lo 4 KB / tile, stage
    const size_t b = size_t(kUrBufs) * kUrTpb * 2 * (size_t(8 * kpt) * 32);    // [buf][t] B_hi, B_lo
    const size_t coef = size_t(kUrBufs) * kUrTpb * 32;
    return a_ring + b + coef;
}

__device__ __forceinline__ uint32_t cluster_rank() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
    return r;
}
__device__ __forceinline__ void cluster_sync() {
    asm volatile("barrier.cluster.arrive.release.aligned;\nbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
// store to the same shared-memory offset in CTA `rank` of the cluster
__device__ __forceinline__ void st_cluster_f2(const void *local, uint32_t rank, float2 v) {
    uint32_t remote;
    asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(remote) : "r"(smem_u32(local)), "r"(rank));
    asm volatile("st.shared::cluster.v2.f32 [%0], {%1, %2};" ::"r"(remote), "f"(v.x), "f"(v.y) : "memory");
}

// KPT = channel groups of 8 per item (exactly 8 KPT uniformly spaced channels per item); N~ = 32.
template <int KPT>
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(kUrThreads, 2) gridder_umma_rot_kernel(const KernelArgs a) {
    constexpr int kCols = kUrStages * kUrTiles * 8 * KPT;   // TMEM columns (a power of two)
    constexpr int NS = 32;
    constexpr int NPIX = NS * NS;
    constexpr int h = NS / 2;
    constexpr int N = 8 * KPT;               // UMMA N: 4 pols x (re, im) per channel group
    constexpr int NC = 8 * KPT;              // channels per item
    constexpr int BT = N * 32;               // bytes of one B tile (N rows x K = 16 f16)
    constexpr int VPB = kUrTpb * NC * 2;     // float4 (2 complex values) per batch
    constexpr int PER = (VPB + kUrThreads - 1) / kUrThreads;
    static_assert(KPT == 2 || KPT == 4, "N = 16 or 32");
    static_assert(kUrStages * kUrTiles * N <= 512, "TMEM columns");

    // the no-swizzle K-major operands need 16-byte alignment only
    extern __shared__ __align__(16) unsigned char smem[];
    unsigned char *a_ring = smem;                                                   // [stage][tile][hi | lo]
    unsigned char *b_s = a_ring + size_t(kUrStages) * kUrTiles * 8192;              // [buf][t][hi | lo] BT each
    float4 *coef_s = reinterpret_cast<float4 *>(b_s + size_t(kUrBufs * kUrTpb) * 2 * BT);   // [buf][t][cB, cQ]
    __shared__ __align__(8) uint64_t full_bar[kUrStages][kUrTiles], dfull_bar[kUrStages][kUrTiles];
    __shared__ __align__(8) uint64_t ready_bar[kUrBufs], empty_bar[kUrBufs];
    __shared__ uint32_t tmem_base_s;
    __shared__ float red_s[kUrThreads / 32];
    __shared__ float df_s[8];

    const int slot = int(blockIdx.x >> 1);    // position of the item in the order
    const int item = a.order[slot];
    const uint32_t rank = cluster_rank();     // which half of the subgrid
    const ItemSetup s = dev::item_setup(a, item, NS);
    const idg_metadata &md = s.md;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int tile = warp >> 2, quarter = warp & 3;
    const int row = quarter * 32 + lane;                      // row of the tile = TMEM lane
    const bool leader = quarter == 0 && lane == 0;            // issues the tile's UMMAs

    if (warp == 0) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(&tmem_base_s)),
                     "r"(kCols));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    if (threadIdx.x == 0) {
        for (int st = 0; st < kUrStages; ++st)
            for (int t = 0; t < kUrTiles; ++t) {
                asm volatile("mbarrier.init.shared::cta.b64 [%0], 128;" ::"r"(smem_u32(&full_bar[st][t])));
                asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&dfull_bar[st][t])));
            }
        for (int b = 0; b < kUrBufs; ++b) {
            asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(&ready_bar[b])), "r"(kUrThreads));
            asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(&empty_bar[b])), "r"(kUrTiles));
        }
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    if (threadIdx.x < 8)   // slot offsets of group 0 from the reference frequency
        df_s[threadIdx.x] = float(a.frequencies[md.channel_begin + threadIdx.x] / kSpeedOfLight - s.f_ref);

    const int T = md.nr_timesteps;
    const int nb = (T + kUrTpb - 1) / kUrTpb;
    const int64_t vrow = int64_t(a.nr_channels) * 4;   // float2 per timestep
    const float2 *vis0 = a.vis + (int64_t(md.baseline) * a.nr_timesteps + md.time_offset) * vrow +
                         int64_t(md.channel_begin) * 4;
    const float *uvw0 = a.uvw + (int64_t(md.baseline) * a.nr_timesteps + md.time_offset) * 3;

    // f16 range: one power-of-two scale for the item from its largest visibility component (a pre-pass over
    // the item's visibilities; they stay in L2 for the batches below)
    float mx = 0.0f;
    for (int i0 = threadIdx.x; i0 < T * NC * 2; i0 += 4 * kUrThreads) {
        float4 q[4];
#pragma unroll
        for (int u = 0; u < 4; ++u) {   // four independent loads in flight
            const int i = i0 + u * kUrThreads;
            q[u] = make_float4(0.0f, 0.0f, 0.0f, 0.0f);
            if (i < T * NC * 2) {
                const int t = i / (NC * 2), r = i - t * NC * 2;
                q[u] = __ldg(reinterpret_cast<const float4 *>(vis0 + int64_t(t) * vrow) + r);
            }
        }
#pragma unroll
        for (int u = 0; u < 4; ++u)
            mx = fmaxf(mx, fmaxf(fmaxf(fabsf(q[u].x), fabsf(q[u].y)), fmaxf(fabsf(q[u].z), fabsf(q[u].w))));
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) mx = fmaxf(mx, __shfl_xor_sync(0xffffffffu, mx, o));
    if (lane == 0) red_s[warp] = mx;

    // prefetch registers of one batch: float4 i = (t, c, half) and the uvw of timestep threadIdx.x
    float4 v[PER];
    float pu = 0.0f, pv = 0.0f, pw = 0.0f;
    auto load_batch = [&](int b) {
        const int t0 = b * kUrTpb, nt = min(kUrTpb, T - t0);
#pragma unroll
        for (int k = 0; k < PER; ++k) {
            const int i = threadIdx.x + k * kUrThreads;
            if (i < nt * NC * 2) {
                const int t = i / (NC * 2), r = i - t * NC * 2;
                v[k] = dev::ld_stream(reinterpret_cast<const float4 *>(vis0 + int64_t(t0 + t) * vrow) + r);
            }
        }
        if (int(threadIdx.x) < nt) {
            const float *p = uvw0 + int64_t(t0 + threadIdx.x) * 3;
            pu = __ldg(p);
            pv = __ldg(p + 1);
            pw = __ldg(p + 2);
        }
    };
    if (T > 0) load_batch(0);
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;");
    const uint32_t tmem = tmem_base_s;
    float bmax = 0.0f;
#pragma unroll 8
    for (int w = 0; w < kUrThreads / 32; ++w) bmax = fmaxf(bmax, red_s[w]);
    const float scale = pow2_scale(bmax);   // 1 for an all-zero (flagged) item

    // stage the prefetched batch b into its ring slot: B tiles and timestep coefficients, then arrive on the
    // slot's ready barrier.  The slot's previous batch (b - kUrBufs) must have been consumed by every tile's
    // UMMAs (empty barrier: one tcgen05.commit per tile after its last UMMA of that batch).
    auto stage_batch = [&](int b) {
        const int buf = b % kUrBufs;
        if (b >= kUrBufs) mbar_wait(&empty_bar[buf], uint32_t((b / kUrBufs - 1) & 1));
        const int t0 = b * kUrTpb, nt = min(kUrTpb, T - t0);
        if (int(threadIdx.x) < nt) {
            float4 cB, cQ;
            dev::timestep_coefficients_uvw(s, pu, pv, pw, cB, cQ);
            coef_s[2 * (buf * kUrTpb + threadIdx.x)] = cB;
            coef_s[2 * (buf * kUrTpb + threadIdx.x) + 1] = cQ;
        }
        // B tiles: element (n, k) at (n/8)*256 + (k/8)*128 + (n%8)*16 + (k%8)*2; column n = 8 j + 2 pol
        // (+1: im), rows k = 2 s (cos), 2 s + 1 (sin); column 2pol: (Vre, -Vim), 2pol+1: (Vim, Vre)
#pragma unroll
        for (int k = 0; k < PER; ++k) {
            const int i = threadIdx.x + k * kUrThreads;
            if (i < nt * NC * 2) {
                const int t = i / (NC * 2), r = i - t * NC * 2, c = r >> 1, pol0 = (r & 1) * 2;
                const int j = c >> 3, sl = c & 7;
                unsigned char *bt = b_s + size_t(buf * kUrTpb + t) * 2 * BT;
#pragma unroll
                for (int q = 0; q < 2; ++q) {
                    const int pol = pol0 + q;
                    const float vr = (q ? v[k].z : v[k].x) * scale, vi = (q ? v[k].w : v[k].y) * scale;
#pragma unroll
                    for (int im = 0; im < 2; ++im) {
                        const int n = 8 * j + 2 * pol + im;
                        uint32_t hi, lo;
                        split2(im ? vi : vr, im ? vr : -vi, hi, lo);
                        const int off = (n >> 3) * 256 + (sl >> 2) * 128 + (n & 7) * 16 + (sl & 3) * 4;
                        *reinterpret_cast<uint32_t *>(bt + off) = hi;
                        *reinterpret_cast<uint32_t *>(bt + BT + off) = lo;
                    }
                }
            }
        }
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(&ready_bar[buf])) : "memory");
    };

    // this thread's pixel
    const int pix = int(rank) * kUrThreads + tile * 128 + row;
    const float pl = float(pix % NS - h) * a.cell_l, pm = float(pix / NS - h) * a.cell_l;
    const float pn = dev::w_term_n(pl, pm);
    float df[8];
#pragma unroll
    for (int q = 0; q < 8; ++q) df[q] = df_s[q];
    // shared-memory addresses / descriptors: A stage st at + st * 64 KB (desc + 4096), lo half + 4 KB
    // (desc + 256); B of (buf, t) at + (buf TPB + t) 2 BT, lo half + BT
    unsigned char *a_row = a_ring + tile * 8192 + (row >> 3) * 256 + (row & 7) * 16;
    const uint64_t da0 = umma_desc(smem_u32(a_ring + tile * 8192));
    const uint64_t db0 = umma_desc(smem_u32(b_s));
    const uint32_t td0 = tmem + uint32_t(tile * N);
    const uint32_t tr0 = tmem + (uint32_t(quarter * 32) << 16) + uint32_t(tile * N);

    if (T > 0) {
        stage_batch(0);
        if (nb > 1) load_batch(1);
    }
    f2p acc[4];
#pragma unroll
    for (int p = 0; p < 4; ++p) acc[p] = 0;
    f2p e_p = 0, ne_p = 0;
    int t = 0;
    for (int b = 0; b < nb; ++b) {
        const int buf = b % kUrBufs;
        // stage the next batch one batch ahead, prefetch the one after
        if (b + 1 < nb) {
            stage_batch(b + 1);
            if (b + 2 < nb) load_batch(b + 2);
        }
        mbar_wait(&ready_bar[buf], uint32_t((b / kUrBufs) & 1));
        const int t1 = min(T, (b + 1) * kUrTpb);
        for (int tl = 0; t < t1; ++t, ++tl) {
            const int st = t & 1;
            const float4 cB = coef_s[2 * (buf * kUrTpb + tl)], cQ = coef_s[2 * (buf * kUrTpb + tl) + 1];
            const float bv = fmaf(cB.x, pl, fmaf(cB.y, pm, cB.z * pn));
            const float qv = fmaf(cQ.x, pl, fmaf(cQ.y, pm, cQ.z * pn));
            uint32_t hi[8], lo[8];
            float c0 = 1.0f, s0 = 0.0f, c4 = 1.0f, s4 = 0.0f;
#pragma unroll
            for (int sl = 0; sl < 8; ++sl) {
                float sn, cs;
                __sincosf(fmaf(df[sl], qv, bv), &sn, &cs);
                split2(cs, sn, hi[sl], lo[sl]);
                if (sl == 0) { c0 = cs; s0 = sn; }
                if (sl == 4) { c4 = cs; s4 = sn; }
            }
            // E4 = Phi(4) conj(Phi(0)) = exp(i 4 dnu/c Q), E = E4^2
            const float r4 = fmaf(c4, c0, s4 * s0), i4 = fmaf(s4, c0, -c4 * s0);
            const float er = fmaf(r4, r4, -i4 * i4), ei = 2.0f * r4 * i4;
            // A rows of stage st (its previous UMMAs, timestep t - 2, were waited for one timestep ago)
            unsigned char *ta = a_row + st * (kUrTiles * 8192);
            *reinterpret_cast<uint4 *>(ta) = make_uint4(hi[0], hi[1], hi[2], hi[3]);
            *reinterpret_cast<uint4 *>(ta + 128) = make_uint4(hi[4], hi[5], hi[6], hi[7]);
            *reinterpret_cast<uint4 *>(ta + 4096) = make_uint4(lo[0], lo[1], lo[2], lo[3]);
            *reinterpret_cast<uint4 *>(ta + 4096 + 128) = make_uint4(lo[4], lo[5], lo[6], lo[7]);
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            asm volatile("tcgen05.fence::before_thread_sync;");
            asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(&full_bar[st][tile])) : "memory");
            if (leader) {
                mbar_wait(&full_bar[st][tile], uint32_t((t >> 1) & 1));
                asm volatile("tcgen05.fence::after_thread_sync;");
                const uint64_t da = da0 + uint64_t(st * (kUrTiles * 8192 / 16));
                const uint64_t db = db0 + uint64_t((buf * kUrTpb + tl) * (2 * BT / 16));
                const uint32_t td = td0 + uint32_t(st * kUrTiles * N);
                umma_f16<N>(td, da, db, 0u);                         // A_hi B_hi (fresh)
                umma_f16<N>(td, da, db + BT / 16, 1u);               // + A_hi B_lo
                umma_f16<N>(td, da + 4096 / 16, db, 1u);             // + A_lo B_hi
                asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];"
                             ::"r"(smem_u32(&dfull_bar[st][tile])) : "memory");
                if (t + 1 == t1)   // the tile's last UMMA reading this batch slot
                    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];"
                                 ::"r"(smem_u32(&empty_bar[buf])) : "memory");
            }
            // D of the previous timestep, rotated into the accumulators (Horner over the groups)
            if (t > 0) {
                const int ps = st ^ 1;
                mbar_wait(&dfull_bar[ps][tile], uint32_t(((t - 1) >> 1) & 1));
                asm volatile("tcgen05.fence::after_thread_sync;");
                const uint32_t tdr = tr0 + uint32_t(ps * kUrTiles * N);
                f2p hh[4];
                uint32_t d[16];
                if constexpr (KPT == 4) {
                    tmem_ld16(tdr + 16, d);                   // groups 2, 3
                    tmem_wait_ld();
#pragma unroll
                    for (int p = 0; p < 4; ++p) hh[p] = pk_u(d[8 + 2 * p], d[9 + 2 * p]);
                    horner_step2(hh, d, e_p, ne_p);           // D_2 + E D_3
                    tmem_ld16(tdr, d);                        // groups 0, 1
                    tmem_wait_ld();
                    horner_step2(hh, d + 8, e_p, ne_p);       // D_1 + E h
                    horner_step2(hh, d, e_p, ne_p);           // D_0 + E h
                } else {
                    tmem_ld16(tdr, d);
                    tmem_wait_ld();
#pragma unroll
                    for (int p = 0; p < 4; ++p) hh[p] = pk_u(d[8 + 2 * p], d[9 + 2 * p]);
                    horner_step2(hh, d, e_p, ne_p);           // D_0 + E D_1
                }
                asm volatile("tcgen05.fence::before_thread_sync;");
#pragma unroll
                for (int p = 0; p < 4; ++p) acc[p] = add2(acc[p], hh[p]);
            }
            e_p = pk(er, er);
            ne_p = pk(-ei, ei);
        }
    }
    // D of the last timestep
    if (T > 0) {
        const int ps = (T - 1) & 1;
        mbar_wait(&dfull_bar[ps][tile], uint32_t(((T - 1) >> 1) & 1));
        asm volatile("tcgen05.fence::after_thread_sync;");
        const uint32_t tdr = tr0 + uint32_t(ps * kUrTiles * N);
        f2p hh[4];
        uint32_t d[16];
        if constexpr (KPT == 4) {
            tmem_ld16(tdr + 16, d);
            tmem_wait_ld();
#pragma unroll
            for (int p = 0; p < 4; ++p) hh[p] = pk_u(d[8 + 2 * p], d[9 + 2 * p]);
            horner_step2(hh, d, e_p, ne_p);
            tmem_ld16(tdr, d);
            tmem_wait_ld();
            horner_step2(hh, d + 8, e_p, ne_p);
            horner_step2(hh, d, e_p, ne_p);
        } else {
            tmem_ld16(tdr, d);
            tmem_wait_ld();
#pragma unroll
            for (int p = 0; p < 4; ++p) hh[p] = pk_u(d[8 + 2 * p], d[9 + 2 * p]);
            horner_step2(hh, d, e_p, ne_p);
        }
#pragma unroll
        for (int p = 0; p < 4; ++p) acc[p] = add2(acc[p], hh[p]);
        asm volatile("tcgen05.fence::before_thread_sync;");
    }

    // ---- epilogue: registers -> sub_s[pol][pixel], then a3 + a4 + a5 ------------------------------
    __syncthreads();
    if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(kCols));
    float2 *sub_s = reinterpret_cast<float2 *>(smem);
    float2 *tmp_s = sub_s + 4 * NPIX;
    const float inv = 1.0f / scale;
#pragma unroll
    for (int pol = 0; pol < 4; ++pol) {
        const float2 r = unpk(acc[pol]);
        sub_s[pol * NPIX + pix] = make_float2(r.x * inv, r.y * inv);
    }
    {
        // CTA `rank` transforms and adds polarisations 2 rank, 2 rank + 1 of the whole subgrid
        uint4 *tab = reinterpret_cast<uint4 *>(tmp_s + 2 * NPIX);
        dft_tab_to_smem<NS>(tab, -1);
        cluster_sync();   // both halves are out of their loops: the peer's shared memory is free for our writes
        dev::gridder_aterm_pixel<NS>(a, s, sub_s, pix);               // a3 of this thread's pixel (all 4 pols)
        const uint32_t peer = rank ^ 1u;
#pragma unroll
        for (int q = 0; q < 2; ++q) {
            const int pol = 2 * int(peer) + q;
            st_cluster_f2(&sub_s[pol * NPIX + pix], peer, sub_s[pol * NPIX + pix]);
        }
        cp_async_wait_all();
        cluster_sync();   // the peer's half of our polarisations has landed
        const float2 *own = sub_s + 2 * int(rank) * NPIX;
        float mx = 0.0f;
        for (int i = threadIdx.x; i < 2 * NPIX; i += kUrThreads)
            mx = fmaxf(mx, fmaxf(fabsf(own[i].x), fabsf(own[i].y)));
        const float sc = pow2_scale(block_max<kUrThreads / 32>(mx, red_s));
        // a4 rows: T[pol][y][kx] -> tmp_s[pol][kx][y], kept scaled by sc / 32 (|T| <= N~ max|S|)
        dft_pass_tc<NS, kUrThreads / 32, 2>(own, NS, 1, tab, sc, 1.0f / 32.0f, [&](int pol, int y, int kx, float2 v) {
            tmp_s[pol * NPIX + kx * NS + y] = v;
        });
        __syncthreads();
        const int pol0 = 2 * int(rank);
        if (a.subgrids) {   // host adder: the transformed subgrid goes to its slot of the subgrid buffer
            float2 *sp = a.subgrids + int64_t(slot) * 4 * NPIX;
            dft_pass_tc<NS, kUrThreads / 32, 2>(tmp_s, NS, 1, tab, 1.0f, 32.0f / sc,
                                                [&](int pol, int kx, int ky, float2 v) {
                                                    sp[((pol0 + pol) * NS + ky) * NS + kx] = v;
                                                });
            return;
        }
        if (a.bands) {   // banded grid: each element goes to its owner's band (peer memory)
            dft_pass_tc<NS, kUrThreads / 32, 2>(tmp_s, NS, 1, tab, 1.0f, 32.0f / sc,
                                                [&](int pol, int kx, int ky, float2 v) {
                                                    dev::grid_add(a, md.z, pol0 + pol, md.y + ky, md.x + kx, v);
                                                });
            __threadfence_system();
            return;
        }
        const int64_t gs = a.grid_size;
        float2 *gp = a.grid + (int64_t(md.z) * 4 * gs + md.y) * gs + md.x;
        dft_pass_tc<NS, kUrThreads / 32, 2>(tmp_s, NS, 1, tab, 1.0f, 32.0f / sc, [&](int pol, int kx, int ky, float2 v) {
            dev::red_add(gp + (int64_t(pol0 + pol) * gs + ky) * gs + kx, v);
        });
    }
}

template <int KPT>
size_t smem_gridder_umma_rot(const KernelArgs &) { return gridder_umma_rot_smem_bytes(KPT); }

template <int KPT>
cudaError_t launch_gridder_umma_rot(const KernelArgs &a, cudaStream_t st) {
    constexpr auto kernel = gridder_umma_rot_kernel<KPT>;
    const size_t smem = gridder_umma_rot_smem_bytes(KPT);
    cudaError_t err = ensure_dft_tables();
    if (err != cudaSuccess) return err;
    if ((err = dev::prepare(kernel, smem)) != cudaSuccess) return err;
    LaunchScope scope("gridder", st);
    // two CTAs (one cluster, __cluster_dims__) per item
    kernel<<<2u * unsigned(a.nr_items), kUrThreads, smem, st>>>(a);
    return cudaGetLastError();
}
