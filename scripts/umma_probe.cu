// umma_probe.cu -- validate tcgen05.mma (kind::f16, cta_group::1, M=128, N=16, K=16) with A and B in
// shared memory (K-major, no swizzle, canonical 8x16B core matrices), D in TMEM, read back with
// tcgen05.ld.32x32b.  Design probe for the tcgen05 gridder; prints max error vs a CPU reference.
#include <cstdio>
#include <cstdint>
#include <cmath>
#include <cuda_fp16.h>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t smem_u32(const void *p) { return static_cast<uint32_t>(__cvta_generic_to_shared(p)); }

// K-major no-swizzle operand: element (row, k) at (row/8)*SBO + (k/8)*LBO + (row%8)*16 + (k%8)*2 bytes
__device__ __forceinline__ uint64_t make_desc(uint32_t saddr, uint32_t lbo, uint32_t sbo) {
    uint64_t d = 0;
    d |= uint64_t((saddr >> 4) & 0x3fff);
    d |= uint64_t((lbo >> 4) & 0x3fff) << 16;
    d |= uint64_t((sbo >> 4) & 0x3fff) << 32;
    d |= uint64_t(1) << 46;  // version (sm100)
    return d;                 // base offset 0, lbo mode 0, layout SWIZZLE_NONE (0)
}

__global__ void probe(const __half *A, const __half *B, float *D) {
    constexpr int M = 128, N = 16, K = 16;
    __shared__ __align__(128) uint8_t sa[M * K * 2];
    __shared__ __align__(128) uint8_t sb[N * K * 2];
    __shared__ __align__(8) uint64_t bar;
    __shared__ uint32_t tmem_base;
    const int tid = threadIdx.x;  // 128 threads
    // A row tid
    for (int k = 0; k < K; ++k) {
        const uint32_t off = (tid / 8) * 256 + (k / 8) * 128 + (tid % 8) * 16 + (k % 8) * 2;
        *reinterpret_cast<__half *>(sa + off) = A[tid * K + k];
    }
    if (tid < N)
        for (int k = 0; k < K; ++k) {
            const uint32_t off = (tid / 8) * 256 + (k / 8) * 128 + (tid % 8) * 16 + (k % 8) * 2;
            *reinterpret_cast<__half *>(sb + off) = B[tid * K + k];  // B stored N x K (K-major)
        }
    if (tid < 32) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 32;" ::"r"(smem_u32(&tmem_base)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    if (tid == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&bar)));
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    asm volatile("fence.proxy.async.shared::cta;");
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;");
    const uint32_t tmem = tmem_base;
    if (tid == 0) {
        const uint64_t da = make_desc(smem_u32(sa), 128, 256);
        const uint64_t db = make_desc(smem_u32(sb), 128, 256);
        // instr desc: c_format F32 (bit 4), a/b F16 (0), K-major (0), n_dim = N>>3 at 17, m_dim = M>>4 at 24
        const uint32_t idesc = (1u << 4) | (uint32_t(N >> 3) << 17) | (uint32_t(M >> 4) << 24);
        asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\n"
                     "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}"
                     ::"r"(tmem), "l"(da), "l"(db), "r"(idesc), "r"(0));
        asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(&bar)));
    }
    // wait for the mma
    asm volatile("{\n.reg .pred P1;\nWAIT:\n"
                 "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n"
                 "@!P1 bra WAIT;\n}" ::"r"(smem_u32(&bar)), "r"(0));
    asm volatile("tcgen05.fence::after_thread_sync;");
    uint32_t r[16];
    const uint32_t taddr = tmem + (uint32_t((tid / 32) * 32) << 16);
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
                 : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
                   "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
                 : "r"(taddr));
    asm volatile("tcgen05.wait::ld.sync.aligned;");
    for (int n = 0; n < N; ++n) D[tid * N + n] = __uint_as_float(r[n]);
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    if (tid < 32) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 32;" ::"r"(tmem));
}


// A operand in TMEM: lane = row, 32-bit column j holds (k = 2j, 2j+1) as f16x2 (low half = even k).
// Written by the owning warp with tcgen05.st.32x32b.x8; MMA: tcgen05.mma ... [d], [a], b_desc.
__global__ void probe_tmem_a(const __half *A, const __half *B, float *D, int a_col) {
    constexpr int M = 128, N = 16, K = 16;
    __shared__ __align__(128) uint8_t sb[N * K * 2];
    __shared__ __align__(8) uint64_t bar;
    __shared__ uint32_t tmem_base;
    const int tid = threadIdx.x;
    if (tid < N)
        for (int k = 0; k < K; ++k) {
            const uint32_t off = (tid / 8) * 256 + (k / 8) * 128 + (tid % 8) * 16 + (k % 8) * 2;
            *reinterpret_cast<__half *>(sb + off) = B[tid * K + k];
        }
    if (tid < 32) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 64;" ::"r"(smem_u32(&tmem_base)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    if (tid == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&bar)));
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    asm volatile("fence.proxy.async.shared::cta;");
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;");
    const uint32_t tmem = tmem_base;
    const uint32_t lane_off = uint32_t((tid / 32) * 32) << 16;
    uint32_t w[8];
    for (int j = 0; j < 8; ++j) {
        __half2 h = __halves2half2(A[tid * K + 2 * j], A[tid * K + 2 * j + 1]);
        w[j] = *reinterpret_cast<uint32_t *>(&h);
    }
    asm volatile("tcgen05.st.sync.aligned.32x32b.x8.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};"
                 ::"r"(tmem + lane_off + uint32_t(a_col)), "r"(w[0]), "r"(w[1]), "r"(w[2]), "r"(w[3]), "r"(w[4]), "r"(w[5]),
                   "r"(w[6]), "r"(w[7]));
    asm volatile("tcgen05.wait::st.sync.aligned;");
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;");
    if (tid == 0) {
        const uint64_t db = make_desc(smem_u32(sb), 128, 256);
        const uint32_t idesc = (1u << 4) | (uint32_t(N >> 3) << 17) | (uint32_t(M >> 4) << 24);
        asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\n"
                     "tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n}"
                     ::"r"(tmem), "r"(tmem + uint32_t(a_col)), "l"(db), "r"(idesc), "r"(0));
        asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(&bar)));
    }
    asm volatile("{\n.reg .pred P1;\nWAIT2:\n"
                 "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n"
                 "@!P1 bra WAIT2;\n}" ::"r"(smem_u32(&bar)), "r"(0));
    asm volatile("tcgen05.fence::after_thread_sync;");
    uint32_t r[16];
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
                 : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
                   "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
                 : "r"(tmem + lane_off));
    asm volatile("tcgen05.wait::ld.sync.aligned;");
    for (int n = 0; n < N; ++n) D[tid * N + n] = __uint_as_float(r[n]);
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    if (tid < 32) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 64;" ::"r"(tmem));
}
int main() {
    const int M = 128, N = 16, K = 16;
    __half hA[M * K], hB[N * K];
    float fA[M * K], fB[N * K], hD[M * N];
    for (int i = 0; i < M * K; ++i) { fA[i] = float((i * 37) % 23 - 11) / 8.0f; hA[i] = __float2half(fA[i]); }
    for (int i = 0; i < N * K; ++i) { fB[i] = float((i * 13) % 17 - 8) / 4.0f; hB[i] = __float2half(fB[i]); }
    __half *dA, *dB; float *dD;
    cudaMalloc(&dA, sizeof(hA)); cudaMalloc(&dB, sizeof(hB)); cudaMalloc(&dD, sizeof(hD));
    cudaMemcpy(dA, hA, sizeof(hA), cudaMemcpyHostToDevice); cudaMemcpy(dB, hB, sizeof(hB), cudaMemcpyHostToDevice);
    probe<<<1, 128>>>(dA, dB, dD);
    cudaError_t e = cudaDeviceSynchronize();
    cudaMemcpy(hD, dD, sizeof(hD), cudaMemcpyDeviceToHost);
    double maxerr = 0;
    for (int m = 0; m < M; ++m)
        for (int n = 0; n < N; ++n) {
            double ref = 0;
            for (int k = 0; k < K; ++k) ref += double(fA[m * K + k]) * fB[n * K + k];
            maxerr = fmax(maxerr, fabs(ref - hD[m * N + n]));
        }
    printf("status %s, max |D - A.B^T| = %g (D[0]=%g D[17]=%g)\n", cudaGetErrorString(e), maxerr, hD[0], hD[17]);
    for (int a_col : {16, 24, 40}) {
        cudaMemset(dD, 0, sizeof(hD));
        probe_tmem_a<<<1, 128>>>(dA, dB, dD, a_col);
        e = cudaDeviceSynchronize();
        cudaMemcpy(hD, dD, sizeof(hD), cudaMemcpyDeviceToHost);
        maxerr = 0;
        for (int m = 0; m < M; ++m)
            for (int n = 0; n < N; ++n) {
                double ref = 0;
                for (int k = 0; k < K; ++k) ref += double(fA[m * K + k]) * fB[n * K + k];
                maxerr = fmax(maxerr, fabs(ref - hD[m * N + n]));
            }
        printf("A in TMEM (col %d): status %s, max |D - A.B^T| = %g (D[0]=%g D[17]=%g)\n", a_col, cudaGetErrorString(e),
               maxerr, hD[0], hD[17]);
    }
    return 0;
}
