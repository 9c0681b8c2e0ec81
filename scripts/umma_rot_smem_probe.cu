// umma_rot_smem_probe.cu -- design probe (not part of the product): the rotation gridder's per-timestep loop on
// tcgen05 with the A operand (split phasors) in SHARED memory, so TMEM holds only the D accumulators and a CTA
// can keep all 8 tiles (1024 pixel rows = an N~ = 32 subgrid) in flight with 32 producer warps.  Per timestep
// and tile: producers write A_hi / A_lo rows (canonical K-major layout, 2 x STS.128 each) + fence.proxy.async +
// mbarrier arrive; one thread issues 3 UMMAs (M=128, N=8J, K=16): A_hi B_hi (fresh), + A_hi B_lo, + A_lo B_hi,
// commits to the tile's D barrier; the producers read D of the previous timestep (tcgen05.ld) and sum the groups
// in Horner form into their fp32 accumulators (4 pols per pixel).  Memory-free otherwise (B constant).
#include <cstdint>
#include <cstdio>
#include <cuda_fp16.h>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t smem_u32(const void *p) { return static_cast<uint32_t>(__cvta_generic_to_shared(p)); }
__device__ __forceinline__ uint64_t make_desc(uint32_t saddr, uint32_t lbo, uint32_t sbo) {
    return uint64_t((saddr >> 4) & 0x3fff) | (uint64_t((lbo >> 4) & 0x3fff) << 16) | (uint64_t((sbo >> 4) & 0x3fff) << 32) |
           (uint64_t(1) << 46);
}
__device__ __forceinline__ void mbar_wait(uint64_t *bar, uint32_t parity) {
    uint32_t done = 0;
    do {
        asm volatile("{\n.reg .pred P;\nmbarrier.try_wait.parity.shared::cta.b64 P, [%1], %2;\nselp.u32 %0, 1, 0, P;\n}"
                     : "=r"(done) : "r"(smem_u32(bar)), "r"(parity) : "memory");
    } while (!done);
}
__device__ __forceinline__ uint32_t h2b(__half2 h) { return *reinterpret_cast<uint32_t *>(&h); }
__device__ __forceinline__ void split_mx(float x, float y, uint32_t &hi, uint32_t &lo) {
    hi = h2b(__floats2half2_rn(x, y));
    float lx, ly;
    asm("{\n.reg .f16 a, b, m;\nmov.b32 {a, b}, %2;\nmov.b16 m, 0xBC00;\n"
        "fma.rn.f32.f16 %0, a, m, %3;\nfma.rn.f32.f16 %1, b, m, %4;\n}"
        : "=f"(lx), "=f"(ly) : "r"(hi), "f"(x), "f"(y));
    lo = h2b(__floats2half2_rn(lx, ly));
}

template <int J>
__device__ __forceinline__ void ld_d(uint32_t taddr, float (&d)[8 * J]) {
#pragma unroll
    for (int h = 0; h < (8 * J) / 16; ++h) {
        uint32_t r[16];
        asm volatile("tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
                     : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
                       "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
                     : "r"(taddr + 16 * h));
#pragma unroll
        for (int i = 0; i < 16; ++i) d[16 * h + i] = __uint_as_float(r[i]);
    }
    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
}

// A tile: 128 rows x K=16 f16 (32 B per row) = 4 KB, canonical K-major no swizzle: row r, k-chunk c (8 values)
// at (r / 8) * 256 + c * 128 + (r % 8) * 16 bytes.
// DIST = 1: no MMA warp; lane 0 of each tile's first warp issues that tile's UMMAs once all 128 rows arrived.
template <int NT, int J, int S, int DIST = 0>
__global__ void __launch_bounds__((NT * 4 + (DIST ? 0 : 1)) * 32, 1) loop_umma_rot_smem(float *out, int steps) {
    constexpr int N = 8 * J;
    static_assert(NT * S * N <= 512, "TMEM columns");
    extern __shared__ __align__(1024) uint8_t dsm[];
    uint8_t *a_s = dsm;                                        // [S][NT][hi, lo][4 KB]
    uint8_t *b_s = dsm + S * NT * 2 * 4096;                    // B_hi, B_lo: [K=16][N] K-major
    __shared__ __align__(8) uint64_t full_bar[S][NT], dfull_bar[S][NT];
    __shared__ uint32_t tmem_base;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    for (int i = threadIdx.x; i < 2 * N * 8; i += blockDim.x)
        reinterpret_cast<uint32_t *>(b_s)[i] = 0x2c002c00u ^ (i & 0x00ff00ffu);
    if (warp == 0) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(smem_u32(&tmem_base)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    if (threadIdx.x == 0) {
        for (int s = 0; s < S; ++s)
            for (int t = 0; t < NT; ++t) {
                asm volatile("mbarrier.init.shared::cta.b64 [%0], 128;" ::"r"(smem_u32(&full_bar[s][t])));
                asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&dfull_bar[s][t])));
            }
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    asm volatile("fence.proxy.async.shared::cta;");
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;");
    const uint32_t tmem = tmem_base;
    float result = 0.0f;
    if (warp < NT * 4) {
        const int tile = warp >> 2, quarter = warp & 3;
        const uint32_t lane_off = uint32_t(quarter * 32) << 16;
        const int row = quarter * 32 + lane;
        const uint32_t row_off = uint32_t((row >> 3) * 256 + (row & 7) * 16);
        const float l = 1e-3f * row, m = 2e-3f * tile, n = 1e-6f * row;
        float df[8];
#pragma unroll
        for (int v = 0; v < 8; ++v) df[v] = 1e-4f * v;
        float acc[8];
#pragma unroll
        for (int i = 0; i < 8; ++i) acc[i] = 0.0f;
        float er_prev = 1.0f, ei_prev = 0.0f;
        for (int k = 0; k <= steps; ++k) {
            const int st = k % S;
            float er = 1.0f, ei = 0.0f;
            if (k < steps) {
                const float Bv = fmaf(0.1f + 1e-5f * k, l, fmaf(0.2f, m, 0.3f * n));
                const float Qv = fmaf(1e-3f, l, fmaf(2e-3f, m, (3e-3f + 1e-9f * k) * n));
                uint32_t hi[8], lo[8];
                float c0 = 1, s0 = 0, c4 = 1, s4 = 0;
#pragma unroll
                for (int v = 0; v < 8; ++v) {
                    float sn, cs;
                    __sincosf(fmaf(df[v], Qv, Bv), &sn, &cs);
                    split_mx(cs, sn, hi[v], lo[v]);
                    if (v == 0) { c0 = cs; s0 = sn; }
                    if (v == 4) { c4 = cs; s4 = sn; }
                }
                const float r4 = fmaf(c4, c0, s4 * s0), i4 = fmaf(s4, c0, -c4 * s0);
                er = fmaf(r4, r4, -i4 * i4);
                ei = 2.0f * r4 * i4;
                // the stage's A buffer is free: the MMAs that read it (step k - S) were waited for at step k - S + 1
                uint8_t *ah = a_s + (st * NT + tile) * 2 * 4096;
                const uint32_t ahs = smem_u32(ah) + row_off;
                asm volatile("st.shared.v4.b32 [%0], {%1,%2,%3,%4};" ::"r"(ahs), "r"(hi[0]), "r"(hi[1]), "r"(hi[2]), "r"(hi[3]));
                asm volatile("st.shared.v4.b32 [%0], {%1,%2,%3,%4};" ::"r"(ahs + 128), "r"(hi[4]), "r"(hi[5]), "r"(hi[6]), "r"(hi[7]));
                asm volatile("st.shared.v4.b32 [%0], {%1,%2,%3,%4};" ::"r"(ahs + 4096), "r"(lo[0]), "r"(lo[1]), "r"(lo[2]), "r"(lo[3]));
                asm volatile("st.shared.v4.b32 [%0], {%1,%2,%3,%4};" ::"r"(ahs + 4096 + 128), "r"(lo[4]), "r"(lo[5]), "r"(lo[6]), "r"(lo[7]));
                asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
                asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(&full_bar[st][tile])) : "memory");
                if (DIST && quarter == 0 && lane == 0) {
                    mbar_wait(&full_bar[st][tile], uint32_t((k / S) & 1));
                    asm volatile("tcgen05.fence::after_thread_sync;");
                    const uint32_t idesc = (1u << 4) | (uint32_t(N >> 3) << 17) | (uint32_t(128 >> 4) << 24);
                    const uint64_t dbh = make_desc(smem_u32(b_s), 128, 256), dbl = make_desc(smem_u32(b_s + N * 32), 128, 256);
                    const uint32_t sa = smem_u32(a_s + (st * NT + tile) * 2 * 4096);
                    const uint64_t dah = make_desc(sa, 128, 256), dal = make_desc(sa + 4096, 128, 256);
                    const uint32_t td = tmem + uint32_t((st * NT + tile) * N);
                    asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, 0, 0;\ntcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}"
                                 ::"r"(td), "l"(dah), "l"(dbh), "r"(idesc));
                    asm volatile("{\n.reg .pred p;\nsetp.eq.b32 p, 0, 0;\ntcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}"
                                 ::"r"(td), "l"(dah), "l"(dbl), "r"(idesc));
                    asm volatile("{\n.reg .pred p;\nsetp.eq.b32 p, 0, 0;\ntcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}"
                                 ::"r"(td), "l"(dal), "l"(dbh), "r"(idesc));
                    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];"
                                 ::"r"(smem_u32(&dfull_bar[st][tile])) : "memory");
                }
            }
            if (k > 0) {   // D of the previous timestep: Horner sum of the groups
                const int ps = (k - 1) % S;
                mbar_wait(&dfull_bar[ps][tile], uint32_t(((k - 1) / S) & 1));
                asm volatile("tcgen05.fence::after_thread_sync;");
                float d[N];
                ld_d<J>(tmem + lane_off + uint32_t((ps * NT + tile) * N), d);
                float h[8];
#pragma unroll
                for (int i = 0; i < 8; ++i) h[i] = d[8 * (J - 1) + i];
#pragma unroll
                for (int j = J - 2; j >= 0; --j) {
#pragma unroll
                    for (int p = 0; p < 4; ++p) {
                        const float hr = h[2 * p], hi_ = h[2 * p + 1];
                        h[2 * p] = fmaf(er_prev, hr, fmaf(-ei_prev, hi_, d[8 * j + 2 * p]));
                        h[2 * p + 1] = fmaf(er_prev, hi_, fmaf(ei_prev, hr, d[8 * j + 2 * p + 1]));
                    }
                }
#pragma unroll
                for (int i = 0; i < 8; ++i) acc[i] += h[i];
            }
            er_prev = er;
            ei_prev = ei;
        }
#pragma unroll
        for (int i = 0; i < 8; ++i) result += acc[i];
    } else if (!DIST && lane == 0) {
        const uint32_t idesc = (1u << 4) | (uint32_t(N >> 3) << 17) | (uint32_t(128 >> 4) << 24);
        const uint64_t dbh = make_desc(smem_u32(b_s), 128, 256), dbl = make_desc(smem_u32(b_s + N * 32), 128, 256);
        for (int k = 0; k < steps; ++k) {
            const int st = k % S;
#pragma unroll 1
            for (int t = 0; t < NT; ++t) {
                mbar_wait(&full_bar[st][t], uint32_t((k / S) & 1));
                asm volatile("tcgen05.fence::after_thread_sync;");
                const uint32_t sa = smem_u32(a_s + (st * NT + t) * 2 * 4096);
                const uint64_t dah = make_desc(sa, 128, 256), dal = make_desc(sa + 4096, 128, 256);
                const uint32_t td = tmem + uint32_t((st * NT + t) * N);
                asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, 0, 0;\ntcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}"
                             ::"r"(td), "l"(dah), "l"(dbh), "r"(idesc));
                asm volatile("{\n.reg .pred p;\nsetp.eq.b32 p, 0, 0;\ntcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}"
                             ::"r"(td), "l"(dah), "l"(dbl), "r"(idesc));
                asm volatile("{\n.reg .pred p;\nsetp.eq.b32 p, 0, 0;\ntcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}"
                             ::"r"(td), "l"(dal), "l"(dbh), "r"(idesc));
                asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];"
                             ::"r"(smem_u32(&dfull_bar[st][t])) : "memory");
            }
        }
    }
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tmem));
    out[blockIdx.x * blockDim.x + threadIdx.x] = result;
}

template <int NT, int J, int S, int DIST = 0>
void run(float *out) {
    const int steps = 2048, blocks = 148;
    const size_t smem = size_t(S) * NT * 2 * 4096 + 2 * 8 * J * 32;
    const int threads = (NT * 4 + (DIST ? 0 : 1)) * 32;
    cudaFuncSetAttribute(loop_umma_rot_smem<NT, J, S, DIST>, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0); cudaEventCreate(&e1);
    loop_umma_rot_smem<NT, J, S, DIST><<<blocks, threads, smem>>>(out, 16);
    cudaError_t e = cudaDeviceSynchronize();
    if (e != cudaSuccess) { printf("NT %d J %d: %s\n", NT, J, cudaGetErrorString(e)); return; }
    cudaEventRecord(e0);
    loop_umma_rot_smem<NT, J, S, DIST><<<blocks, threads, smem>>>(out, steps);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    const double pairs = double(blocks) * NT * 128 * 8 * J * steps;
    printf("UMMA-ROT-SMEM-A %s NT %d (%2d producer warps/SM) J %d S %d: %6.2f pairs/clk/SM (at 1965 MHz)  %s\n",
           DIST ? "dist-issue" : "mma-warp  ", NT, NT * 4, J, S, pairs / (ms * 1e-3) / 148 / 1.965e9, cudaGetErrorString(cudaGetLastError()));
}

int main() {
    float *out; cudaMalloc(&out, 148 * 1056 * 4);
    run<7, 4, 2>(out);   // J = 4 (SKA): 7 tiles x 2 stages x 32 columns = 448 (224 producer threads x 4 warps + 1)
    run<4, 4, 2>(out);
    run<7, 2, 2>(out);   // J = 2 (LOFAR)
    run<8, 4, 2, 1>(out);   // distributed issue: all 8 tiles of an N~ = 32 subgrid, 32 warps
    run<4, 4, 2, 1>(out);
    run<8, 2, 2, 1>(out);
    run<4, 4, 3, 1>(out);
    return 0;
}
