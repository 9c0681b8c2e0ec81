/*
 * idg.h -- C ABI of the B200-native Image-Domain Gridding hot path (libidg_b200.so).
 *
 * Method: Veenboer, Petschow, Romein, "Image-Domain Gridding on Graphics Processors", IPDPS 2017.
 * "P:n" = line n of /root/reference/PAPER.md (the paper text); "R-k" = reading k of the paper in
 * DESIGN.md section 3.  Every call returns an idg_status; no C++ exception crosses this boundary.
 *
 * Conventions
 *   - Visibility V_pq(t,c) in C^{2x2} is stored as 4 complex64 = 8 float, pol order
 *     XX,XY,YX,YY = row-major 2x2 (Alg. 2 lines 10-11; R-17).
 *   - uvw in METRES, float32, per (baseline, timestep); u_lambda = u * nu / c.
 *   - Grid cell g <-> u = (g - N/2) du, du = 1/L wavelengths (L = image size in direction cosines).
 *   - Subgrid pixel (y,x) <-> l = (x - N~/2) L/N~, m = (y - N~/2) L/N~, n = 1 - sqrt(1-l^2-m^2)
 *     (R-3, R-4).  Grid/subgrid planes are [pol][row=v][col=u].
 *   - "d_" arguments are DEVICE pointers (cudaMalloc / torch CUDA tensors) on the current device;
 *     the caller owns them.  Host arrays are only read during the call.
 *   - Calls that take a cudaStream_t are asynchronous on that stream (0 = legacy default stream).
 *
 * Errors: arguments and shapes are validated before any launch (IDG_ERR_INVALID_ARG /
 * IDG_ERR_UNSUPPORTED).  CUDA failures return IDG_ERR_CUDA; idg_last_error() gives a
 * thread-local detail message for the last failing call on the calling thread.
 */
#ifndef IDG_B200_H
#define IDG_B200_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct CUstream_st *idg_stream; /* == cudaStream_t */

typedef enum {
    IDG_OK = 0,
    IDG_ERR_INVALID_ARG = 1,         /* NULL pointer, negative size, inconsistent shapes           */
    IDG_ERR_UNSUPPORTED = 2,         /* e.g. subgrid size not in {16, 24, 32}; no sm_100 device    */
    IDG_ERR_OUT_OF_MEMORY = 3,
    IDG_ERR_CUDA = 4,                /* a CUDA runtime call or kernel launch failed               */
    IDG_ERR_WORKSPACE_TOO_SMALL = 5
} idg_status;

typedef struct {
    int32_t station1, station2;      /* station1 < station2; A_p = A[station1], A_q = A[station2] (R-16) */
} idg_baseline;

/* Plan parameters. */
typedef struct {
    int32_t subgrid_size;              /* N~: 16, 24 or 32 ("as small as 24x24")              */
    int32_t grid_size;                 /* N: even, >= 2 N~ (2048)                            */
    double image_size;                 /* L in (0, sqrt 2) (direction cosines); cell du = 1/L       */
    int32_t kernel_size;               /* K: support reserved around the footprint (Fig. 5; R-8)    */
    int32_t max_timesteps_per_subgrid; /* T~max >= 1 (R-14)                                   */
    int32_t max_channels_per_subgrid;  /* C~: channel block size; 0 = all channels (R-9)     */
    double w_offset;                   /* w0 (wavelengths) subtracted in the w-term           */
    int32_t nr_w_planes;               /* W-stacking: number of W-planes; 0 or 1 = none */
    double w_step;                     /* W-plane spacing (wavelengths), > 0 when nr_w_planes > 1.   */
                                       /* Plane z has w0_z = w_offset + (z - (nz-1)/2) w_step; each  */
                                       /* item lies in the plane nearest to w at its block's middle  */
                                       /* channel (clamped) and never straddles a plane (R-21).       */
} idg_plan_params;

/* One work item = one subgrid and its visibilities.  Bit-exact with the oracle's plan. */
typedef struct {
    int32_t baseline;                  /* index into baselines[]                                   */
    int32_t time_offset;               /* t0                                                        */
    int32_t nr_timesteps;              /* T~ (1 .. T~max); items never straddle an A-term slot     */
    int32_t channel_begin;             /* c0                                                        */
    int32_t channel_end;               /* c1 (exclusive)                                            */
    int32_t aterm_index;               /* A-term slot of t0 (R-15)                                  */
    int32_t x, y;                      /* subgrid corner in grid cells; centre cell x+N~/2 (R-11)   */
    int32_t z;                         /* W-plane index (0 without W-stacking, R-21)               */
} idg_metadata;

typedef struct idg_plan idg_plan;

/*
 * idg_plan_create -- the execution plan (greedy rules R-8..R-16), built on the host.
 *   params           plan parameters (copied)
 *   nr_stations      S (A-term station dimension)
 *   nr_baselines     nbl;  nr_timesteps T;  nr_channels C
 *   uvw              HOST float32 [nbl][T][3], metres
 *   frequencies      HOST float64 [C], Hz
 *   baselines        HOST [nbl]; 0 <= station1 < station2 < S
 *   nr_aterm_slots   >= 1;  aterm_offsets HOST int32 [slots+1], 0 = off[0] < ... < off[slots] = T
 *   out              receives the plan; free with idg_plan_destroy.
 * Visibilities whose subgrid would fall off the grid (R-12) or whose single timestep does not fit
 * (R-13) are dropped and counted (idg_plan_stats).  The plan is immutable and may be shared by
 * threads and streams; its device copy is made on first use on a device (lazily, thread-safe), so
 * creating a plan needs no GPU.
 */
idg_status idg_plan_create(const idg_plan_params *params, int32_t nr_stations, int32_t nr_baselines,
                           int32_t nr_timesteps, int32_t nr_channels, const float *uvw,
                           const double *frequencies, const idg_baseline *baselines,
                           int32_t nr_aterm_slots, const int32_t *aterm_offsets, idg_plan **out);

idg_status idg_plan_destroy(idg_plan *plan);

/* Number of work items (subgrids). */
idg_status idg_plan_nr_subgrids(const idg_plan *plan, int64_t *n);

/* Copy min(n, nr_subgrids) work items into HOST dst, in plan order (baseline, channel block, time). */
idg_status idg_plan_metadata(const idg_plan *plan, idg_metadata *dst, int64_t n);

/* Visibilities in items, dropped visibilities, and (pixel, visibility) pairs = sum_j N~^2 T~_j C~_j. */
idg_status idg_plan_stats(const idg_plan *plan, int64_t *nr_vis_assigned, int64_t *nr_vis_dropped,
                          int64_t *nr_pairs);

/* Device workspace idg_grid / idg_degrid need, in bytes (0: the fused sm_100a kernels keep every
 * subgrid on chip).  The host-streamed calls need idg_host_workspace_size() instead. */
idg_status idg_workspace_size(const idg_plan *plan, size_t *bytes);

/*
 * idg_grid -- gridding (Fig. 4): gridder (Alg. 1) -> A-term/taper -> subgrid FFT -> adder,
 * fused into one sm_100a kernel per work item.
 *   d_vis      complex64 [nbl][T][C][4]
 *   d_uvw      float32 [nbl][T][3] metres (the same values the plan was built from)
 *   d_aterms   complex64 [slots][S][N~][N~][4] (Jones matrices per station and subgrid pixel)
 *   d_taper    float32 [N~][N~] (spheroidal)
 *   d_grid     complex64 [nz][4][N][N] (nz = W-planes, 1 without W-stacking), ACCUMULATED (+=);
 *              subgrid sums use fp32 atomics, so the order of
 *              additions (not the math) is unspecified (R-19)
 *   d_workspace, workspace_bytes   >= idg_workspace_size (may be NULL/0 when that is 0)
 * Only the visibilities in the plan's items are read.
 */
idg_status idg_grid(const idg_plan *plan, const void *d_vis, const float *d_uvw,
                    const void *d_aterms, const float *d_taper, void *d_grid, void *d_workspace,
                    size_t workspace_bytes, idg_stream stream);

/*
 * idg_degrid -- degridding: splitter -> subgrid inverse FFT -> taper/A-term (Alg. 2
 * lines 2-3) -> degridder (Alg. 2), fused into one sm_100a kernel per work item.
 *   d_grid     complex64 [nz][4][N][N] model grid (read only)
 *   d_vis      complex64 [nbl][T][C][4], OVERWRITTEN; dropped visibilities are set to 0
 *   other arguments as idg_grid.
 */
idg_status idg_degrid(const idg_plan *plan, const void *d_grid, const float *d_uvw,
                      const void *d_aterms, const float *d_taper, void *d_vis, void *d_workspace,
                      size_t workspace_bytes, idg_stream stream);

/*
 * Banded grid: the multi-GPU exchange fused into the kernels.  The work is split over devices by
 * baselines ("embarrassingly parallel"); what couples the devices is the adder, which sums
 * every subgrid into the one uv-grid, and, for prediction, every device reading the one model grid.
 * Here the grid is distributed by row bands: band r holds grid rows [r R, (r+1) R) of every [plane][pol]
 * as complex64 [nz][4][R][N] (R = band_rows), and the adder of every work item adds each subgrid row
 * straight into the band that owns it -- another rank's memory when d_bands holds CUDA-IPC mappings
 * (idg_ipc_open; NVLink / NVSwitch peer access) -- so the cross-rank reduction happens inside the gridder;
 * the degridder's splitter reads the owners' bands the same way (no broadcast).
 *   d_bands    DEVICE array of nr_bands device pointers (nr_bands * band_rows >= N); the pointers may be
 *              peer mappings; the caller keeps them valid for the call
 *   idg_grid_bands    the bands are ACCUMULATED (scalar fp32 atomics, order unspecified: R-19); they are
 *                     complete for readers once every rank's call has completed (synchronise, then a
 *                     cross-rank barrier)
 *   idg_degrid_bands  the bands are read only; d_vis OVERWRITTEN as idg_degrid
 * Other arguments as idg_grid / idg_degrid.  Errors: IDG_ERR_INVALID_ARG for NULL pointers or bands that
 * do not cover the grid; IDG_ERR_CUDA for launch failures (asynchronous faults surface at the next sync).
 */
idg_status idg_grid_bands(const idg_plan *plan, const void *d_vis, const float *d_uvw, const void *d_aterms,
                          const float *d_taper, void *const *d_bands, int32_t nr_bands, int32_t band_rows,
                          idg_stream stream);
idg_status idg_degrid_bands(const idg_plan *plan, const void *const *d_bands, int32_t nr_bands,
                            int32_t band_rows, const float *d_uvw, const void *d_aterms, const float *d_taper,
                            void *d_vis, idg_stream stream);

/*
 * CUDA IPC for the bands.  idg_ipc_handle: the 64-byte cudaIpcMemHandle_t of the allocation containing
 * d_ptr and d_ptr's byte offset in it (handles name whole allocations, e.g. a caching allocator's
 * segment).  idg_ipc_open: map another process's allocation (peer access enabled lazily) and return the
 * pointer at `offset`; not for the calling process's own allocations.  idg_ipc_close: unmap (same offset).
 * Errors: IDG_ERR_INVALID_ARG for NULL arguments, IDG_ERR_CUDA when the runtime refuses.
 */
idg_status idg_ipc_handle(const void *d_ptr, unsigned char handle[64], uint64_t *offset);
idg_status idg_ipc_open(const unsigned char handle[64], uint64_t offset, void **d_ptr);
idg_status idg_ipc_close(void *d_ptr, uint64_t offset);

/*
 * Host-streamed calls: the paper's asynchronous I/O (Fig. 7).  The visibilities live in
 * HOST memory (page-locked for overlap, e.g. cudaHostAlloc / torch pin_memory) and stream through
 * triple-buffered device staging buffers in work groups of contiguous baselines: uploads on an
 * internal copy stream, kernels on `stream`, downloads on another internal copy stream, ordered with
 * events, so transfers overlap the kernels.  Semantics are those of idg_grid / idg_degrid:
 *   idg_grid_host    h_vis (read) -> d_grid (ACCUMULATED)
 *   idg_degrid_host  d_grid -> h_vis (OVERWRITTEN, dropped visibilities = 0)
 * d_workspace must hold at least idg_host_workspace_size() bytes (three staging buffers per direction,
 * in separate halves so a grid call's uploads can overlap a preceding degrid call).  A larger workspace
 * gives more buffers per direction (workspace_bytes / (2 x work-group bytes), up to one per work group);
 * with one per work group the uploads of a grid call never wait for kernels, so the next step's
 * visibilities stream in while the current step degrids.  Both calls are asynchronous on `stream`;
 * h_vis must stay valid (and, for idg_grid_host, unmodified) until `stream` reaches the call's end.
 * Calls on the same plan are serialised internally (the pipeline streams and events belong to the
 * plan's device copy).
 */
idg_status idg_host_workspace_size(const idg_plan *plan, size_t *bytes);
idg_status idg_grid_host(const idg_plan *plan, const void *h_vis, const float *d_uvw,
                         const void *d_aterms, const float *d_taper, void *d_grid, void *d_workspace,
                         size_t workspace_bytes, idg_stream stream);
idg_status idg_degrid_host(const idg_plan *plan, const void *d_grid, const float *d_uvw,
                           const void *d_aterms, const float *d_taper, void *h_vis, void *d_workspace,
                           size_t workspace_bytes, idg_stream stream);

/*
 * Host adder / splitter: the grid lives in HOST memory (Section V-C-e, option 2: "copy the subgrids
 * into host memory and perform the operation on the CPU ... only required when dealing with large images
 * that no longer fit into GPU device memory").  Visibilities are in host memory as for idg_grid_host.
 * Per work group the kernels write (gridding) or read (degridding) the group's transformed subgrids in a
 * device buffer instead of the grid; the subgrids stream to / from page-locked host buffers (allocated by
 * the library per workspace, freed with the plan) and host threads (IDG_HOST_THREADS, default: the
 * hardware concurrency, at most 32) add them into / split them out of the host grid -- each thread owns
 * the grid rows r with r mod T == its index, so no atomics -- while the GPU processes the next groups.
 *   idg_grid_host_adder      h_vis (read) -> h_grid complex64 [nz][4][N][N] HOST, ACCUMULATED (+=).
 *                            Returns when h_grid holds the result (the host adds are done); later work
 *                            on `stream` may reuse the workspace.
 *   idg_degrid_host_splitter h_grid (read) -> h_vis OVERWRITTEN (dropped visibilities = 0).  Waits for
 *                            the caller's earlier work on `stream` before reading h_grid; asynchronous
 *                            afterwards: h_vis is complete when `stream` reaches the call's end.
 * d_workspace must hold idg_host_adder_workspace_size() bytes (3 staging buffers per direction, each
 * one work group's visibilities + subgrids); a larger workspace gives more buffers.  Errors as idg_grid.
 */
idg_status idg_host_adder_workspace_size(const idg_plan *plan, size_t *bytes);
idg_status idg_grid_host_adder(const idg_plan *plan, const void *h_vis, const float *d_uvw,
                               const void *d_aterms, const float *d_taper, void *h_grid, void *d_workspace,
                               size_t workspace_bytes, idg_stream stream);
idg_status idg_degrid_host_splitter(const idg_plan *plan, const void *h_grid, const float *d_uvw,
                                    const void *d_aterms, const float *d_taper, void *h_vis,
                                    void *d_workspace, size_t workspace_bytes, idg_stream stream);

/*
 * idg_rho_benchmark -- the paper's FMA:sincos throughput benchmark (Fig. 12) on the
 * current device: every sincos evaluation is followed by rho-1 FMAs plus the one FMA that forms its
 * argument (rho FMAs per sincos).  ops = 2 per FMA + 1 per sin + 1 per cos (op definition).
 *   rho in {0,1,2,3,4,6,8,12,16,17,20,24,32,48,64}; rho = 0 measures sincos alone (2 ops each: the
 *   XU/MUFU bound);  iterations >= 1 (work per thread);  ops_per_second receives the measured
 *   throughput (synchronous: the call waits for the kernel; timed with CUDA events on `stream`).
 * The FMAs of two units run as one packed f32x2 FFMA2 (the B200 FMA-pipe form);
 * idg_rho_benchmark_scalar issues them as scalar 3-register FFMA (the paper's form, which sm_100 issues
 * at half the FP32 lane rate).
 */
idg_status idg_rho_benchmark(int32_t rho, int32_t iterations, idg_stream stream,
                             double *ops_per_second, double *seconds);
idg_status idg_rho_benchmark_scalar(int32_t rho, int32_t iterations, idg_stream stream,
                                    double *ops_per_second, double *seconds);

/*
 * Kernel timing (measurement only).  When enabled, every kernel the library launches is bracketed
 * by CUDA events on its launch stream; idg_profiling_read synchronises those events and returns,
 * per kernel name, the number of launches and the summed device time in ms.
 */
typedef struct {
    char name[48];
    int64_t launches;
    double total_ms;
} idg_kernel_time;

idg_status idg_profiling_enable(int32_t enable);
idg_status idg_profiling_reset(void);
idg_status idg_profiling_read(idg_kernel_time *dst, int32_t capacity, int32_t *n);

/* Diagnostics: newline-separated names of the compiled launch-shape variants of the gridder
 * (which = 0) or degridder (which = 1).  Setting the environment variable IDG_GRIDDER_VARIANT /
 * IDG_DEGRIDDER_VARIANT to one of these names before a call overrides the default (tuning only);
 * a name prefix ending in '*' selects the first eligible match; the values "tc" (direct tensor-core
 * kernel) and "simt" (CUDA-core kernel, the paper's structure) select a kernel family.  The default
 * is the fastest eligible tensor-core variant. */
const char *idg_kernel_variants(int32_t which);

/* Diagnostics: name of the variant (one of idg_kernel_variants(which)) that the most recent gridder
 * (which = 0) or degridder (which = 1) launch in this process used, or "" before the first launch.
 * Static storage; safe to call from any thread (the name may be stale if calls race). */
const char *idg_last_variant(int32_t which);

/* Number of kernel launches issued by this library in the calling process so far. */
int64_t idg_launch_count(void);

const char *idg_status_string(idg_status status);
const char *idg_last_error(void);

#ifdef __cplusplus
}
#endif
#endif /* IDG_B200_H */
