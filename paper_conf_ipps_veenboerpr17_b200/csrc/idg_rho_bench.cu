// idg_rho_bench.cu -- the FMA:sincos throughput benchmark of the paper (Fig. 12):
// "we benchmarked the performance for various ratios of rho = number of FMAs / number of sincos";
// the value at rho = 17 is the "modified roofline" bound of the gridder and degridder.
//
// Each thread runs U independent units (like U pixels of the gridder).  Per unit and iteration:
// one FMA forms the sincos argument, one __sincosf (FMUL range reduction + MUFU.SIN + MUFU.COS, the
// same black box the kernels use) and rho-1 FMAs accumulate into 8 independent accumulators
// (at rho = 17: exactly the 2x2 complex multiply-accumulate of Alg. 1/2).  The loop-carried
// argument advances by one FADD per iteration, amortised over the U units.
//
// Two forms.  rho_kernel (scalar, the paper's form) issues every FMA as a 3-register FFMA, which sm_100
// issues at half the FP32 lane rate (one per 2 cycles per SMSP); rho_kernel_x2 (the B200-native form)
// runs two units per thread as packed f32x2 pairs, so each FFMA2 carries the FMAs of both units -- the
// FMA-pipe arithmetic the kernels use.  idg_rho_benchmark times the packed form,
// idg_rho_benchmark_scalar the scalar one.
#include <cstdint>

#include <cuda_runtime.h>

#include "idg_internal.h"

namespace idg {
namespace {

constexpr int kRhoUnits = 4;
constexpr int kRhoThreads = 256;

// Per unit and iteration: the argument FMA consumes the previous sin and cos (so neither can be
// dropped, at any rho), then rho-1 accumulate FMAs alternate over cos and sin into 8 accumulators.
template <int RHO>
__global__ void __launch_bounds__(kRhoThreads) rho_kernel(float *out, int iterations) {
    constexpr int U = kRhoUnits;
    const int tid = blockIdx.x * blockDim.x + threadIdx.x;
    float sn[U], cs[U], acc[U][8], coef[8];
#pragma unroll
    for (int j = 0; j < 8; ++j) coef[j] = 0.25f + 0.01f * float((tid + j) & 7);
#pragma unroll
    for (int k = 0; k < U; ++k) {
        sn[k] = 0.1f * float(k) + 1e-6f * float(tid & 1023);
        cs[k] = 0.37f + 0.013f * float(k);
#pragma unroll
        for (int j = 0; j < 8; ++j) acc[k][j] = 0.0f;
    }
    const float x = 0.731f + 1e-7f * float(tid & 255);
#pragma unroll 1
    for (int i = 0; i < iterations; ++i) {
#pragma unroll
        for (int k = 0; k < U; ++k) {
            const float ph = fmaf(x, cs[k], sn[k]);  // FMA #1: the argument f().g()
            __sincosf(ph, &sn[k], &cs[k]);
#pragma unroll
            for (int j = 0; j < RHO - 1; ++j) {       // FMAs #2 .. #rho
                acc[k][j & 7] = fmaf(coef[(j >> 3) & 7], (j & 1) ? sn[k] : cs[k], acc[k][j & 7]);
            }
        }
    }
    float sum = 0.0f;
#pragma unroll
    for (int k = 0; k < U; ++k) {
        sum += sn[k] + cs[k];
#pragma unroll
        for (int j = 0; j < 8; ++j) sum += acc[k][j];
    }
    out[tid] = sum;
}

// rho = 0: sincos throughput alone (the XU/MUFU bound of the tensor-core kernels).  Eight independent
// chains per thread; the next argument is cos * 0.5 + sin (one FMA that is not counted as an op).
template <>
__global__ void __launch_bounds__(kRhoThreads) rho_kernel<0>(float *out, int iterations) {
    constexpr int U = 8;
    const int tid = blockIdx.x * blockDim.x + threadIdx.x;
    float x[U];
#pragma unroll
    for (int k = 0; k < U; ++k) x[k] = 1e-3f * float(tid & 255) + float(k);
#pragma unroll 1
    for (int i = 0; i < iterations; ++i) {
#pragma unroll
        for (int k = 0; k < U; ++k) {
            float sn, cs;
            __sincosf(x[k], &sn, &cs);
            x[k] = fmaf(cs, 0.5f, sn);
        }
    }
    float sum = 0.0f;
#pragma unroll
    for (int k = 0; k < U; ++k) sum += x[k];
    out[tid] = sum;
}

// Packed form: U unit pairs per thread; per pair and iteration one FFMA2 forms both arguments, two
// __sincosf, then rho-1 FFMA2 accumulate (alternating cos / sin pairs) into 8 packed accumulators.  The
// accumulate coefficient is a kernel parameter (a uniform register), so an FFMA2 reads two 64-bit
// register pairs: with three (scripts/rho_forms_probe.cu, B200) rho = 17 reaches 55 TOps/s instead of 61.
using u64 = unsigned long long;
__device__ __forceinline__ u64 pk2(float lo, float hi) {
    u64 r;
    asm("mov.b64 %0, {%1, %2};" : "=l"(r) : "f"(lo), "f"(hi));
    return r;
}
__device__ __forceinline__ float2 up2(u64 v) {
    float2 r;
    asm("mov.b64 {%0, %1}, %2;" : "=f"(r.x), "=f"(r.y) : "l"(v));
    return r;
}
__device__ __forceinline__ u64 ffma2(u64 a, u64 b, u64 c) {
    u64 r;
    asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(r) : "l"(a), "l"(b), "l"(c));
    return r;
}

constexpr int kRhoPairs = 4;   // unit pairs per thread (8 units)

template <int RHO>
__global__ void __launch_bounds__(kRhoThreads) rho_kernel_x2(float *out, int iterations, u64 coef) {
    constexpr int U = kRhoPairs;
    const int tid = blockIdx.x * blockDim.x + threadIdx.x;
    u64 sn[U], cs[U], acc[U][8];
#pragma unroll
    for (int k = 0; k < U; ++k) {
        sn[k] = pk2(0.1f * float(k) + 1e-6f * float(tid & 1023), 0.05f * float(k) + 1e-6f * float(tid & 511));
        cs[k] = pk2(0.37f + 0.013f * float(k), 0.41f + 0.011f * float(k));
#pragma unroll
        for (int j = 0; j < 8; ++j) acc[k][j] = 0ull;
    }
    const u64 x = pk2(0.731f + 1e-7f * float(tid & 255), 0.689f + 1e-7f * float(tid & 127));
#pragma unroll 1
    for (int i = 0; i < iterations; ++i) {
#pragma unroll
        for (int k = 0; k < U; ++k) {
            const float2 ph = up2(ffma2(x, cs[k], sn[k]));   // FMA #1 of both units: the arguments
            float s0, c0, s1, c1;
            __sincosf(ph.x, &s0, &c0);
            __sincosf(ph.y, &s1, &c1);
            sn[k] = pk2(s0, s1);
            cs[k] = pk2(c0, c1);
#pragma unroll
            for (int j = 0; j < RHO - 1; ++j)                  // FMAs #2 .. #rho of both units
                acc[k][j & 7] = ffma2(coef, (j & 1) ? sn[k] : cs[k], acc[k][j & 7]);
        }
    }
    float sum = 0.0f;
#pragma unroll
    for (int k = 0; k < U; ++k) {
        const float2 a = up2(sn[k]), b = up2(cs[k]);
        sum += a.x + a.y + b.x + b.y;
#pragma unroll
        for (int j = 0; j < 8; ++j) {
            const float2 c = up2(acc[k][j]);
            sum += c.x + c.y;
        }
    }
    out[tid] = sum;
}

template <typename K, typename... Extra>
cudaError_t run_kernel(K kernel, int iterations, float *out, cudaStream_t s, int *blocks, Extra... extra) {
    int per_sm = 0, dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceProp prop;
    cudaGetDeviceProperties(&prop, dev);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kernel, kRhoThreads, 0);
    *blocks = prop.multiProcessorCount * (per_sm > 0 ? per_sm : 1) * 4;  // 4 full waves
    LaunchScope scope("rho_benchmark", s);
    kernel<<<*blocks, kRhoThreads, 0, s>>>(out, iterations, extra...);
    return cudaGetLastError();
}

template <int RHO>
cudaError_t run(int iterations, float *out, cudaStream_t s, int *blocks, bool packed, int *units) {
    if (packed && RHO > 0) {
        *units = 2 * kRhoPairs;
        return run_kernel(rho_kernel_x2<RHO>, iterations, out, s, blocks, 0x3e8a00003e800000ull);  // (0.25, 0.27)
    }
    *units = RHO == 0 ? 8 : kRhoUnits;
    return run_kernel(rho_kernel<RHO>, iterations, out, s, blocks);
}

}  // namespace

cudaError_t launch_rho_benchmark(int rho, int iterations, float *d_out, cudaStream_t s, int *blocks,
                                 int *threads, int *units_per_thread, bool packed) {
    *threads = kRhoThreads;
    switch (rho) {
        case 0: return run<0>(iterations, d_out, s, blocks, packed, units_per_thread);
#define IDG_RHO_CASE(R) \
    case R: return run<R>(iterations, d_out, s, blocks, packed, units_per_thread);
        IDG_RHO_CASE(1) IDG_RHO_CASE(2) IDG_RHO_CASE(3) IDG_RHO_CASE(4) IDG_RHO_CASE(6)
        IDG_RHO_CASE(8) IDG_RHO_CASE(12) IDG_RHO_CASE(16) IDG_RHO_CASE(17) IDG_RHO_CASE(20)
        IDG_RHO_CASE(24) IDG_RHO_CASE(32) IDG_RHO_CASE(48) IDG_RHO_CASE(64)
#undef IDG_RHO_CASE
        default: return cudaErrorInvalidValue;
    }
}

}  // namespace idg
