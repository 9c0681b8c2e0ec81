// umma_loop_probe.cu -- throughput of the warp-specialised tcgen05 gridder inner loop, no memory:
// PW producer warps each own one 32-row unit (tile = w / 4, TMEM lane quarter = w % 4) and per k-block
// generate 8 phasors per row (phase FMA + sincos + f16 hi/lo split) straight into a TMEM A ring
// (tcgen05.st.32x32b.x8, hi at +0, lo at +8 columns); one MMA warp issues 2 UMMAs per tile
// (M=128, N=16, K=16, A from TMEM, B from shared memory) and commits each stage to its empty barrier.
// Prints pairs per clock per SM (pairs = rows x 8 visibilities per k-block).
#include <cstdio>
#include <cstdint>
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
__device__ __forceinline__ uint32_t h2_bits(__half2 h) { return *reinterpret_cast<uint32_t *>(&h); }

constexpr uint32_t kIdesc = (1u << 4) | (uint32_t(16 >> 3) << 17) | (uint32_t(128 >> 4) << 24);

template <int PW, int NTILES, int S, int MODE>
__global__ void __launch_bounds__((PW + 1) * 32, 1) loop_umma(float *out, int nkb) {
    __shared__ __align__(1024) uint8_t sb[512];
    __shared__ __align__(8) uint64_t full_bar[S], empty_bar[S];
    __shared__ uint32_t tmem_base;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    for (int i = threadIdx.x; i < 128; i += blockDim.x) reinterpret_cast<uint32_t *>(sb)[i] = 0x3c003c00u ^ i;
    if (warp == 0) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(smem_u32(&tmem_base)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    if (threadIdx.x == 0) {
        for (int s = 0; s < S; ++s) {
            asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(&full_bar[s])), "r"(PW));
            asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&empty_bar[s])));
        }
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    asm volatile("fence.proxy.async.shared::cta;");
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;");
    const uint32_t tmem = tmem_base;
    constexpr uint32_t STAGE_COLS = NTILES * 16, D_COL = S * STAGE_COLS;
    static_assert(D_COL + NTILES * 16 <= 512, "TMEM");
    float acc = 0.0f;
    if (warp < PW) {
        const int tile = warp >> 2, q = warp & 3;
        const uint32_t lane_off = uint32_t(q * 32) << 16;
        const float B = 0.1f + (tile * 128 + q * 32 + lane) * 1e-3f, Q = 0.3f + lane * 1e-4f;
        float df[8];
        for (int v = 0; v < 8; ++v) df[v] = v * 0.01f;
        for (int kb = 0; kb < nkb; ++kb) {
            const int st = kb % S;
            if (kb >= S) mbar_wait(&empty_bar[st], uint32_t(((kb / S) - 1) & 1));
            asm volatile("tcgen05.fence::after_thread_sync;");
            uint32_t hi[8], lo[8];
            const float Bk = B + kb * 1e-4f;
            if (MODE == 2) {
#pragma unroll
                for (int v = 0; v < 8; ++v) { hi[v] = __float_as_uint(Bk) + v; lo[v] = hi[v] ^ 7; }
            } else
#pragma unroll
            for (int v = 0; v < 8; v += 2) {
                float s0, c0, s1, c1;
                __sincosf(fmaf(df[v], Q, Bk), &s0, &c0);
                __sincosf(fmaf(df[v + 1], Q, Bk), &s1, &c1);
                const float hc0 = __uint_as_float(__float_as_uint(c0) & 0xffffe000u), hs0 = __uint_as_float(__float_as_uint(s0) & 0xffffe000u);
                const float hc1 = __uint_as_float(__float_as_uint(c1) & 0xffffe000u), hs1 = __uint_as_float(__float_as_uint(s1) & 0xffffe000u);
                hi[v] = h2_bits(__floats2half2_rn(hc0, hs0));
                hi[v + 1] = h2_bits(__floats2half2_rn(hc1, hs1));
                lo[v] = h2_bits(__floats2half2_rn(c0 - hc0, s0 - hs0));
                lo[v + 1] = h2_bits(__floats2half2_rn(c1 - hc1, s1 - hs1));
            }
            const uint32_t ta = tmem + lane_off + uint32_t(st * STAGE_COLS + tile * 16);
            asm volatile("tcgen05.st.sync.aligned.32x32b.x8.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"r"(ta), "r"(hi[0]),
                         "r"(hi[1]), "r"(hi[2]), "r"(hi[3]), "r"(hi[4]), "r"(hi[5]), "r"(hi[6]), "r"(hi[7]));
            asm volatile("tcgen05.st.sync.aligned.32x32b.x8.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"r"(ta + 8), "r"(lo[0]),
                         "r"(lo[1]), "r"(lo[2]), "r"(lo[3]), "r"(lo[4]), "r"(lo[5]), "r"(lo[6]), "r"(lo[7]));
            asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
            asm volatile("tcgen05.fence::before_thread_sync;");
            __syncwarp();
            if (lane == 0) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(&full_bar[st])) : "memory");
        }
        // final D read (keeps the MMAs live)
        mbar_wait(&empty_bar[(nkb - 1) % S], uint32_t(((nkb - 1) / S) & 1));
        asm volatile("tcgen05.fence::after_thread_sync;");
        uint32_t r[8];
        asm volatile("tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                     : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7])
                     : "r"(tmem + lane_off + D_COL + tile * 16));
        asm volatile("tcgen05.wait::ld.sync.aligned;");
        for (int j = 0; j < 8; ++j) acc += __uint_as_float(r[j]);
    } else if (lane == 0) {
        const uint64_t db = make_desc(smem_u32(sb), 128, 256);
        for (int kb = 0; kb < nkb; ++kb) {
            const int st = kb % S;
            mbar_wait(&full_bar[st], uint32_t((kb / S) & 1));
            asm volatile("tcgen05.fence::after_thread_sync;");
            if (MODE == 1) {
                asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(&empty_bar[st])) : "memory");
                continue;
            }
#pragma unroll
            for (int t = 0; t < NTILES; ++t) {
                const uint32_t ta = tmem + uint32_t(st * STAGE_COLS + t * 16), td = tmem + D_COL + uint32_t(t * 16);
                asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\ntcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n}"
                             ::"r"(td), "r"(ta), "l"(db), "r"(kIdesc), "r"(kb > 0 ? 1 : 0));
                asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\ntcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n}"
                             ::"r"(td), "r"(ta + 8), "l"(db), "r"(kIdesc), "r"(1));
            }
            asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(&empty_bar[st]))
                         : "memory");
        }
    }
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tmem));
    out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
}


// raw UMMA issue rate: one thread issues `iters` dependent-accumulator MMAs (M=128, K=16, N given),
// A from TMEM (ATMEM=1) or shared memory, then one commit; clock64 around it.
template <int N, int ATMEM, int NACC = 1>
__global__ void mma_rate(long long *clk, int iters) {
    __shared__ __align__(1024) uint8_t sa[128 * 32];
    __shared__ __align__(1024) uint8_t sb[256 * 32];
    __shared__ __align__(8) uint64_t bar;
    __shared__ uint32_t tmem_base;
    for (int i = threadIdx.x; i < 128 * 8; i += blockDim.x) reinterpret_cast<uint32_t *>(sa)[i] = 0x3c003c00u;
    for (int i = threadIdx.x; i < 256 * 8; i += blockDim.x) reinterpret_cast<uint32_t *>(sb)[i] = 0x3c003c00u;
    if (threadIdx.x < 32) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(smem_u32(&tmem_base)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    if (threadIdx.x == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&bar)));
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    asm volatile("fence.proxy.async.shared::cta;");
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;");
    const uint32_t tmem = tmem_base;
    if (threadIdx.x == 0) {
        const uint32_t idesc = (1u << 4) | (uint32_t(N >> 3) << 17) | (uint32_t(128 >> 4) << 24);
        const uint64_t da = make_desc(smem_u32(sa), 128, 256), db = make_desc(smem_u32(sb), 128, 256);
        const long long t0 = clock64();
        for (int i = 0; i < iters; ++i) {
            if (ATMEM)
                asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\ntcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n}"
                             ::"r"(tmem + uint32_t((i % NACC) * N)), "r"(tmem + 384), "l"(db), "r"(idesc), "r"(uint32_t(i >= NACC)));
            else
                asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\ntcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}"
                             ::"r"(tmem), "l"(da), "l"(db), "r"(idesc), "r"(i));
        }
        asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(&bar)) : "memory");
        mbar_wait(&bar, 0);
        clk[blockIdx.x] = clock64() - t0;
    }
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    if (threadIdx.x < 32) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tmem));
}
template <int N, int ATMEM, int NACC = 1>
void rate(long long *dclk) {
    const int iters = 8192;
    mma_rate<N, ATMEM, NACC><<<148, 128>>>(dclk, 64);
    mma_rate<N, ATMEM, NACC><<<148, 128>>>(dclk, iters);
    cudaError_t e = cudaDeviceSynchronize();
    long long h[148];
    cudaMemcpy(h, dclk, sizeof(h), cudaMemcpyDeviceToHost);
    double m = 0; for (int i = 0; i < 148; ++i) m += h[i]; m /= 148;
    printf("UMMA M128 N%-3d K16 A in %-5s acc x%d: %6.1f clk per MMA = %7.0f MAC/clk/SM  %s\n", N, ATMEM ? "TMEM" : "smem", NACC, m / iters,
           128.0 * N * 16 * iters / m, cudaGetErrorString(e));
}
template <int PW, int NTILES, int S, int MODE = 0>
void run(const char *name, float *out) {
    const int nkb = 4096, blocks = 148 * 4;
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0); cudaEventCreate(&e1);
    loop_umma<PW, NTILES, S, MODE><<<blocks, (PW + 1) * 32>>>(out, 64);
    cudaError_t e = cudaDeviceSynchronize();
    if (e != cudaSuccess) { printf("%s: %s\n", name, cudaGetErrorString(e)); return; }
    cudaEventRecord(e0);
    loop_umma<PW, NTILES, S, MODE><<<blocks, (PW + 1) * 32>>>(out, nkb);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    const double pairs = double(blocks) * PW * 32 * 8 * nkb;
    printf("%-40s %6.2f pairs/clk/SM (at 1.965 GHz)  %s\n", name, pairs / (ms * 1e-3) / 148 / 1.965e9,
           cudaGetErrorString(cudaGetLastError()));
}

int main() {
    float *out; cudaMalloc(&out, 148 * 4 * 1024 * 4);
    long long *dclk; cudaMalloc(&dclk, 148 * 8);
    rate<16, 1>(dclk); rate<16, 1, 8>(dclk); rate<16, 1, 20>(dclk); rate<32, 1, 8>(dclk); rate<16, 0>(dclk); rate<32, 1>(dclk); rate<64, 1>(dclk); rate<128, 1>(dclk); rate<256, 1>(dclk);
    rate<256, 0>(dclk);
    run<18, 5, 4>("PW18 5 tiles S4 full", out);
    run<18, 5, 4, 1>("PW18 5 tiles S4 no MMA", out);
    run<18, 5, 4, 2>("PW18 5 tiles S4 no sincos", out);
    run<24, 6, 3, 2>("PW24 6 tiles S3 no sincos", out);
    run<8, 2, 8, 2>("PW8 2 tiles S8 no sincos", out);
    run<4, 1, 8, 2>("PW4 1 tile S8 no sincos", out);
    run<4, 1, 8, 0>("PW4 1 tile S8 full", out);
    return 0;
}
