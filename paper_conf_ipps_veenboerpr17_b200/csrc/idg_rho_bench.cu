// idg_rho_bench.cu -- the FMA:sincos throughput benchmark of the paper (Fig. 12):
// "we benchmarked the performance for various ratios of rho = number of FMAs / number of sincos";
// the value at rho = 17 is the "modified roofline" bound of the gridder and degridder.
//
// Each thread runs U independent units (like U pixels of the gridder).  Per unit and iteration:
// one FMA forms the sincos argument, one __sincosf (FMUL range reduction + MUFU.SIN + MUFU.COS, the
// same black box the kernels use) and rho-1 FMAs accumulate into 8 independent accumulators
// (at rho = 17: exactly the 2x2 complex multiply-accumulate of Alg. 1/2).  The loop-carried
// argument advances by one FADD per iteration, amortised over the U units.
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

template <int RHO>
cudaError_t run(int iterations, float *out, cudaStream_t s, int *blocks) {
    int per_sm = 0, dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceProp prop;
    cudaGetDeviceProperties(&prop, dev);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, rho_kernel<RHO>, kRhoThreads, 0);
    *blocks = prop.multiProcessorCount * (per_sm > 0 ? per_sm : 1) * 4;  // 4 full waves
    LaunchScope scope("rho_benchmark", s);
    rho_kernel<RHO><<<*blocks, kRhoThreads, 0, s>>>(out, iterations);
    return cudaGetLastError();
}

}  // namespace

cudaError_t launch_rho_benchmark(int rho, int iterations, float *d_out, cudaStream_t s, int *blocks,
                                 int *threads, int *units_per_thread) {
    *threads = kRhoThreads;
    *units_per_thread = rho == 0 ? 8 : kRhoUnits;
    switch (rho) {
        case 0: return run<0>(iterations, d_out, s, blocks);
#define IDG_RHO_CASE(R) \
    case R: return run<R>(iterations, d_out, s, blocks);
        IDG_RHO_CASE(1) IDG_RHO_CASE(2) IDG_RHO_CASE(3) IDG_RHO_CASE(4) IDG_RHO_CASE(6)
        IDG_RHO_CASE(8) IDG_RHO_CASE(12) IDG_RHO_CASE(16) IDG_RHO_CASE(17) IDG_RHO_CASE(20)
        IDG_RHO_CASE(24) IDG_RHO_CASE(32) IDG_RHO_CASE(48) IDG_RHO_CASE(64)
#undef IDG_RHO_CASE
        default: return cudaErrorInvalidValue;
    }
}

}  // namespace idg
