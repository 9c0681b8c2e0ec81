// idg_internal.h -- structures shared by the host API (idg_api.cpp, idg_plan.cpp) and the sm_100a
// kernels (idg_kernels.cu).  Not part of the public ABI (see include/idg.h).
#pragma once

#include <cstdint>
#include <string>
#include <vector>
#include <cuda_runtime.h>

#include "idg.h"

namespace idg {

constexpr double kSpeedOfLight = 299792458.0;  // m/s; u_lambda = u nu / c

// Host-side result of the plan builder.
struct PlanResult {
    int64_t nr_vis_assigned = 0;
    int64_t nr_vis_dropped = 0;
};

// Builds the work items; `items` is cleared and filled in plan order.  Returns IDG_OK or an error
// (with a message in `err`).
idg_status build_plan(const idg_plan_params &p, int32_t nr_stations, int32_t nbl, int32_t T,
                      int32_t C, const float *uvw, const double *freqs,
                      const idg_baseline *baselines, int32_t nslots, const int32_t *aterm_offsets,
                      std::vector<idg_metadata> &items, PlanResult &res, std::string &err);

// Arguments of the fused gridder / degridder launches (device pointers).
struct KernelArgs {
    int32_t subgrid_size;        // N~
    int32_t grid_size;           // N
    float cell_l;                // L / N~   (direction-cosine step of a subgrid pixel)
    double inv_image_size;       // du = 1/L (wavelengths per grid cell)
    double w_offset;             // w0 (centre of the W-planes)
    int32_t nr_w_planes;         // >= 1
    double w_step;               // W-plane spacing (wavelengths)
    int32_t nr_stations, nr_baselines, nr_timesteps, nr_channels;
    int64_t nr_items;
    const idg_metadata *items;   // [nr_items]
    const int32_t *order;        // [nr_items] launch order (largest work first)
    const int32_t *baselines;    // [nbl][2]
    const double *frequencies;   // [C] Hz
    const float *uvw;            // [nbl][T][3]
    const float2 *aterms;        // [slots][S][N~][N~][4]
    const float *taper;          // [N~][N~]
    float2 *vis;                 // [nbl][T][C][4]  (const for gridding)
    float2 *grid;                // [4][N][N]       (const for degridding)
    float2 *subgrids;            // nullptr, or [nr_items][4][N~][N~] in launch order: the gridders store their
                                 // transformed subgrids here instead of adding them to `grid`, the
                                 // degridders read their split subgrids from here (host adder / splitter)
    float2 *const *bands;        // nullptr, or [nr_bands] pointers (banded grid, possibly peer memory of other
                                 // ranks): grid rows [r R, (r+1) R) of every [plane][pol] live in bands[r] as
                                 // [planes][4][R][N]; replaces `grid` (idg_grid_bands / idg_degrid_bands)
    int32_t band_rows;           // R
    int32_t max_channels_in_item;
    int32_t max_timesteps_in_item;
    float mean_timesteps_in_item; // mean T~ over the items (short-item kernel choice)
    int32_t channel_gcd;         // gcd of all items' channel counts
    int32_t channels_uniform;    // 1 if nu_c = nu_0 + c d for all c (to 1e-12 nu_0)
    float channel_step;          // (nu_{c+1} - nu_c) / c  [1/m], valid when channels_uniform
};

using Launcher = cudaError_t (*)(const KernelArgs &, cudaStream_t);
using SmemFn = size_t (*)(const KernelArgs &);
constexpr int kSimt = 0, kTensor = 1;
struct Variant {
    int ns;            // subgrid size
    int v;             // channels per thread (SIMT degridder) / channel multiple (tensor gridder); 0 = any
    int kind;          // kSimt | kTensor
    int needs_uniform; // 1: requires uniformly spaced channels (phasor rotation over channels)
    const char *name;
    Launcher fn;
    int max_channels = 0;  // > 0: every item has at most this many channels (unrolled channel groups)
    SmemFn smem = nullptr; // dynamic shared memory of a launch (the plan's items must fit the device)
    int max_mean_timesteps = 0;  // > 0: eligible only when the items' mean T~ is at most this (short items)
};
// Tensor-core variants (idg_kernels_tc.cu); the first eligible one is the default.
const Variant *tc_gridder_variants(int *n);     // split-f16 mma (idg_kernels_tc.cu)
const Variant *tc_degridder_variants(int *n);

cudaError_t launch_gridder(const KernelArgs &a, cudaStream_t s);
cudaError_t launch_degridder(const KernelArgs &a, cudaStream_t s);
const char *variant_names(int which);
// vis[r[2i] - base .. + r[2i+1]) = 0 for i < nr (the plan's dropped-visibility runs, R-12 / R-13)
cudaError_t launch_zero_ranges(float2 *vis, const int64_t *ranges, int64_t nr, int64_t base, cudaStream_t s);
const char *last_variant(int which);   // name of the variant the last launch used ("" before any)
cudaError_t launch_rho_benchmark(int rho, int iterations, float *d_out, cudaStream_t s,
                                 int *blocks, int *threads, int *units_per_thread, bool packed);

// Kernel-launch bookkeeping (profiling + launch counter), idg_api.cpp.
struct LaunchScope {
    LaunchScope(const char *name, cudaStream_t s);
    ~LaunchScope();
    const char *name;
    cudaStream_t stream;
    cudaEvent_t e0 = nullptr, e1 = nullptr;
};

}  // namespace idg
