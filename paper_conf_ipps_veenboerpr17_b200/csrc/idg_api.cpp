// idg_api.cpp -- the C ABI of include/idg.h: validation, plan object, lazy device copies, kernel
// launches, profiling.  No C++ exception crosses the ABI; errors map to idg_status and a
// thread-local message (idg_last_error).
#include <algorithm>
#include <atomic>
#include <cmath>
#include <complex>
#include <condition_variable>
#include <functional>
#include <thread>
#include <cstdio>
#include <cstring>
#include <cstdlib>
#include <map>
#include <memory>
#include <mutex>
#include <new>
#include <numeric>
#include <string>
#include <vector>

#include "idg_internal.h"

namespace {

thread_local std::string g_last_error;

idg_status fail(idg_status st, const std::string &msg) {
    g_last_error = msg;
    return st;
}

idg_status cuda_fail(cudaError_t e, const std::string &what) {
    return fail(IDG_ERR_CUDA, what + ": " + cudaGetErrorName(e) + " (" + cudaGetErrorString(e) + ")");
}

std::atomic<int64_t> g_launches{0};

struct ProfileRecord {
    std::string name;
    cudaEvent_t e0, e1;
};
std::mutex g_prof_mu;
std::atomic<bool> g_prof_enabled{false};
std::vector<ProfileRecord> g_prof_pending;
std::map<std::string, std::pair<int64_t, double>> g_prof_totals;

constexpr int kStagingBuffers = 3;                  // triple buffering (Fig. 7)
constexpr size_t kHostChunkBytes = size_t(128) << 20;  // visibilities per work group (host-streamed calls)

// Events of the host-streamed pipeline for one workspace (its staging buffers), grown on demand, and the
// page-locked host subgrid buffers of the host adder / splitter.
struct PipeEvents {
    cudaEvent_t entry = nullptr;                              // the caller's stream at call entry
    std::vector<cudaEvent_t> h2d, kernel_g, kernel_d, d2h;    // per staging buffer
    std::vector<void *> host_subgrids;                        // [buffer] pinned, host_subgrid_bytes each
    size_t host_subgrid_bytes = 0;
    ~PipeEvents() {
        if (entry) cudaEventDestroy(entry);
        for (auto *v : {&h2d, &kernel_g, &kernel_d, &d2h})
            for (cudaEvent_t ev : *v) cudaEventDestroy(ev);
        for (void *p : host_subgrids) cudaFreeHost(p);
    }
};

// A fixed pool of host threads for the host adder / splitter: run(f) calls f(thread, nthreads) on every
// thread and returns when all are done.
class HostPool {
  public:
    explicit HostPool(int n) : n_(std::max(1, n)) {
        for (int t = 1; t < n_; ++t) threads_.emplace_back([this, t] { loop(t); });
    }
    ~HostPool() {
        {
            std::lock_guard<std::mutex> l(mu_);
            stop_ = true;
            ++gen_;
        }
        cv_.notify_all();
        for (auto &th : threads_) th.join();
    }
    void run(const std::function<void(int, int)> &f) {
        {
            std::lock_guard<std::mutex> l(mu_);
            job_ = &f;
            pending_ = n_ - 1;
            ++gen_;
        }
        cv_.notify_all();
        f(0, n_);
        std::unique_lock<std::mutex> l(mu_);
        done_cv_.wait(l, [this] { return pending_ == 0; });
        job_ = nullptr;
    }
    int size() const { return n_; }

  private:
    void loop(int t) {
        uint64_t seen = 0;
        for (;;) {
            const std::function<void(int, int)> *job;
            {
                std::unique_lock<std::mutex> l(mu_);
                cv_.wait(l, [&] { return gen_ != seen; });
                seen = gen_;
                if (stop_) return;
                job = job_;
            }
            (*job)(t, n_);
            std::lock_guard<std::mutex> l(mu_);
            if (--pending_ == 0) done_cv_.notify_one();
        }
    }
    int n_;
    std::vector<std::thread> threads_;
    std::mutex mu_;
    std::condition_variable cv_, done_cv_;
    const std::function<void(int, int)> *job_ = nullptr;
    int pending_ = 0;
    uint64_t gen_ = 0;
    bool stop_ = false;
};

int host_threads() {
    if (const char *env = std::getenv("IDG_HOST_THREADS")) return std::max(1, std::atoi(env));
    return int(std::max(1u, std::min(32u, std::thread::hardware_concurrency())));
}

struct DeviceCopy {
    idg_metadata *items = nullptr;
    int32_t *order = nullptr;      // launch order of the device-resident calls (largest work first)
    int32_t *iota = nullptr;       // plan order (work groups of the host-streamed calls)
    int32_t *baselines = nullptr;
    double *frequencies = nullptr;
    int64_t *dropped = nullptr;    // [nr][2] (visibility offset, count) of the dropped visibilities
    // host-streamed pipeline: one copy stream per direction + events per workspace (keyed by its address,
    // so calls on different workspaces never wait on each other's buffers)
    cudaStream_t h2d = nullptr, d2h = nullptr;
    std::map<const void *, std::unique_ptr<PipeEvents>> *pipes = nullptr;
    std::mutex *pipeline_mu = nullptr;
};

// A work group of the host-streamed calls: baselines [b0, b1) (contiguous in host memory) and their
// items [i0, i1) in plan order ("grouping m <= n work items into a work group").
struct WorkGroup {
    int32_t b0, b1;
    int64_t i0, i1;
    int64_t r0, r1;   // its dropped-visibility ranges [r0, r1) (indices into idg_plan::dropped)
};

bool supported_subgrid(int32_t n) { return n == 16 || n == 24 || n == 32; }

}  // namespace

struct idg_plan {
    idg_plan_params params{};
    int32_t nr_stations = 0, nr_baselines = 0, nr_timesteps = 0, nr_channels = 0;
    int32_t nr_aterm_slots = 0;
    std::vector<int32_t> baselines;  // [nbl][2]
    std::vector<double> frequencies;
    std::vector<idg_metadata> items;
    std::vector<int32_t> order;      // launch order: largest T~ C~ first (tail balance)
    int64_t nr_vis_assigned = 0, nr_vis_dropped = 0, nr_pairs = 0;
    int32_t max_channels_in_item = 0;
    int32_t max_timesteps_in_item = 0;
    float mean_timesteps_in_item = 0.0f;
    std::vector<int64_t> dropped;    // [nr][2]: (offset, count) in visibilities of every dropped run,
                                     // split at baseline boundaries (R-12, R-13: predicted as 0)
    std::vector<WorkGroup> groups;   // host-streamed work groups
    size_t group_bytes = 0;          // largest work group's visibility bytes
    int64_t group_items = 0;         // most work items in a work group (host adder / splitter)
    int32_t channel_gcd = 1;
    int32_t channels_uniform = 0;
    float channel_step = 0.0f;
    mutable std::mutex mu;
    mutable std::map<int, DeviceCopy> device;

    ~idg_plan() {
        for (auto &kv : device) {
            int prev = -1;
            cudaGetDevice(&prev);
            cudaSetDevice(kv.first);
            cudaFree(kv.second.items);
            cudaFree(kv.second.order);
            cudaFree(kv.second.iota);
            cudaFree(kv.second.dropped);
            delete kv.second.pipes;
            if (kv.second.h2d) cudaStreamDestroy(kv.second.h2d);
            if (kv.second.d2h) cudaStreamDestroy(kv.second.d2h);
            delete kv.second.pipeline_mu;
            cudaFree(kv.second.baselines);
            cudaFree(kv.second.frequencies);
            if (prev >= 0) cudaSetDevice(prev);
        }
    }

    // Device copy of the plan on the current device, made on first use (thread-safe).
    idg_status device_copy(const DeviceCopy **out) const {
        int dev = -1;
        cudaError_t e = cudaGetDevice(&dev);
        if (e != cudaSuccess) return cuda_fail(e, "cudaGetDevice");
        std::lock_guard<std::mutex> lock(mu);
        auto it = device.find(dev);
        if (it != device.end()) {
            *out = &it->second;
            return IDG_OK;
        }
        cudaDeviceProp prop;
        e = cudaGetDeviceProperties(&prop, dev);
        if (e != cudaSuccess) return cuda_fail(e, "cudaGetDeviceProperties");
        if (prop.major != 10 || prop.minor != 0)
            return fail(IDG_ERR_UNSUPPORTED, std::string("libidg_b200 is built for sm_100a only; device ") +
                                                 prop.name + " is sm_" + std::to_string(prop.major) +
                                                 std::to_string(prop.minor));
        DeviceCopy dc;
        auto release = [&dc]() {  // undo a partial device copy
            cudaFree(dc.items); cudaFree(dc.order); cudaFree(dc.iota); cudaFree(dc.baselines);
            cudaFree(dc.frequencies); cudaFree(dc.dropped);
            if (dc.h2d) cudaStreamDestroy(dc.h2d);
            if (dc.d2h) cudaStreamDestroy(dc.d2h);
        };
        const size_t ni = std::max<size_t>(1, items.size());
        if ((e = cudaMalloc(&dc.items, ni * sizeof(idg_metadata))) != cudaSuccess ||
            (e = cudaMalloc(&dc.order, ni * sizeof(int32_t))) != cudaSuccess ||
            (e = cudaMalloc(&dc.iota, ni * sizeof(int32_t))) != cudaSuccess ||
            (e = cudaMalloc(&dc.baselines, std::max<size_t>(2, baselines.size()) * 4)) != cudaSuccess ||
            (e = cudaMalloc(&dc.frequencies, frequencies.size() * 8)) != cudaSuccess ||
            (!dropped.empty() && (e = cudaMalloc(&dc.dropped, dropped.size() * 8)) != cudaSuccess)) {
            release();
            return e == cudaErrorMemoryAllocation ? fail(IDG_ERR_OUT_OF_MEMORY, "plan device copy")
                                                  : cuda_fail(e, "cudaMalloc(plan)");
        }
        std::vector<int32_t> iota(items.size());
        std::iota(iota.begin(), iota.end(), 0);
        if ((!items.empty() &&
             ((e = cudaMemcpy(dc.items, items.data(), items.size() * sizeof(idg_metadata), cudaMemcpyHostToDevice)) != cudaSuccess ||
              (e = cudaMemcpy(dc.order, order.data(), order.size() * sizeof(int32_t), cudaMemcpyHostToDevice)) != cudaSuccess ||
              (e = cudaMemcpy(dc.iota, iota.data(), iota.size() * sizeof(int32_t), cudaMemcpyHostToDevice)) != cudaSuccess)) ||
            (!baselines.empty() &&
             (e = cudaMemcpy(dc.baselines, baselines.data(), baselines.size() * 4, cudaMemcpyHostToDevice)) != cudaSuccess) ||
            (e = cudaMemcpy(dc.frequencies, frequencies.data(), frequencies.size() * 8, cudaMemcpyHostToDevice)) != cudaSuccess ||
            (!dropped.empty() &&
             (e = cudaMemcpy(dc.dropped, dropped.data(), dropped.size() * 8, cudaMemcpyHostToDevice)) != cudaSuccess)) {
            release();
            return cuda_fail(e, "cudaMemcpy(plan)");
        }
        if ((e = cudaStreamCreateWithFlags(&dc.h2d, cudaStreamNonBlocking)) != cudaSuccess ||
            (e = cudaStreamCreateWithFlags(&dc.d2h, cudaStreamNonBlocking)) != cudaSuccess) {
            release();
            return cuda_fail(e, "cudaStreamCreate(pipeline)");
        }
        dc.pipes = new std::map<const void *, std::unique_ptr<PipeEvents>>();
        dc.pipeline_mu = new std::mutex();
        auto res = device.emplace(dev, dc);
        *out = &res.first->second;
        return IDG_OK;
    }
};

namespace idg {

LaunchScope::LaunchScope(const char *n, cudaStream_t s) : name(n), stream(s) {
    g_launches.fetch_add(1);
    if (g_prof_enabled.load()) {
        cudaEventCreate(&e0);
        cudaEventCreate(&e1);
        cudaEventRecord(e0, stream);
    }
}

LaunchScope::~LaunchScope() {
    if (e0) {
        cudaEventRecord(e1, stream);
        std::lock_guard<std::mutex> lock(g_prof_mu);
        g_prof_pending.push_back({name, e0, e1});
    }
}

}  // namespace idg

namespace {

idg_status validate_params(const idg_plan_params *p) {
    if (!p) return fail(IDG_ERR_INVALID_ARG, "params is NULL");
    if (!supported_subgrid(p->subgrid_size))
        return fail(IDG_ERR_UNSUPPORTED, "subgrid_size must be 16, 24 or 32 (got " +
                                             std::to_string(p->subgrid_size) + ")");
    if (p->grid_size < 2 * p->subgrid_size || p->grid_size % 2 != 0 || p->grid_size > (1 << 16))
        return fail(IDG_ERR_INVALID_ARG, "grid_size must be even, >= 2*subgrid_size and <= 65536");
    // every subgrid pixel must be a direction on the sky: l^2 + m^2 < 1 at the corner (-L/2, -L/2)
    if (!(p->image_size > 0.0) || !std::isfinite(p->image_size) || p->image_size >= 1.4142135)
        return fail(IDG_ERR_INVALID_ARG, "image_size must be in (0, sqrt(2))");
    if (p->kernel_size < 0 || p->kernel_size >= p->subgrid_size)
        return fail(IDG_ERR_INVALID_ARG, "kernel_size must be in [0, subgrid_size)");
    if (p->max_timesteps_per_subgrid < 1)
        return fail(IDG_ERR_INVALID_ARG, "max_timesteps_per_subgrid must be >= 1");
    if (p->max_channels_per_subgrid < 0)
        return fail(IDG_ERR_INVALID_ARG, "max_channels_per_subgrid must be >= 0");
    if (!std::isfinite(p->w_offset)) return fail(IDG_ERR_INVALID_ARG, "w_offset is not finite");
    if (p->nr_w_planes < 0 || p->nr_w_planes > 4096)
        return fail(IDG_ERR_INVALID_ARG, "nr_w_planes must be in [0, 4096]");
    if (p->nr_w_planes > 1 && !(p->w_step > 0.0 && std::isfinite(p->w_step)))
        return fail(IDG_ERR_INVALID_ARG, "w_step must be positive and finite when nr_w_planes > 1");
    return IDG_OK;
}

idg_status validate_call(const idg_plan *plan, const void *a, const void *b, const void *c,
                         const void *d, const void *e) {
    if (!plan) return fail(IDG_ERR_INVALID_ARG, "plan is NULL");
    if (plan->items.empty()) return IDG_OK;
    if (!a || !b || !c || !d || !e) return fail(IDG_ERR_INVALID_ARG, "NULL device pointer");
    return IDG_OK;
}

// number of staging buffers per direction a workspace provides (>= kStagingBuffers), and events for them
int staging_buffers(const idg_plan *plan, size_t workspace_bytes) {
    if (plan->group_bytes == 0) return kStagingBuffers;
    const size_t per_dir = workspace_bytes / (2 * plan->group_bytes);
    return int(std::max<size_t>(kStagingBuffers, std::min<size_t>(per_dir, plan->groups.size())));
}
// The pipeline events of workspace `ws` with at least n per-buffer events (pipeline_mu held).
cudaError_t pipe_events(const DeviceCopy *dc, const void *ws, int n, PipeEvents **out) {
    auto &slot = (*dc->pipes)[ws];
    if (!slot) slot.reset(new PipeEvents());
    PipeEvents *pe = slot.get();
    cudaError_t e = cudaSuccess;
    if (!pe->entry && (e = cudaEventCreateWithFlags(&pe->entry, cudaEventDisableTiming)) != cudaSuccess) return e;
    for (auto *v : {&pe->h2d, &pe->kernel_g, &pe->kernel_d, &pe->d2h})
        while (int(v->size()) < n) {
            cudaEvent_t ev;
            if ((e = cudaEventCreateWithFlags(&ev, cudaEventDisableTiming)) != cudaSuccess) return e;
            v->push_back(ev);
        }
    *out = pe;
    return cudaSuccess;
}

// Zero the dropped visibilities [r0, r1) of the plan's range list in `vis` (whose first element is
// visibility `base` of the full array) on stream s.
cudaError_t zero_dropped(const DeviceCopy *dc, void *vis, int64_t base, int64_t r0, int64_t r1, cudaStream_t s) {
    if (r1 <= r0) return cudaSuccess;
    return idg::launch_zero_ranges(static_cast<float2 *>(vis), dc->dropped + 2 * r0, r1 - r0, base, s);
}

// The runs of visibilities no item covers (R-12, R-13), per baseline, as (offset, count) pairs.
void dropped_ranges(const std::vector<idg_metadata> &items, int32_t nbl, int32_t T, int32_t C,
                    std::vector<int64_t> &out) {
    const int64_t per = int64_t(T) * C;
    std::vector<uint8_t> cov(size_t(per), 0);
    size_t it = 0;
    for (int32_t b = 0; b < nbl; ++b) {
        std::fill(cov.begin(), cov.end(), uint8_t(0));
        for (; it < items.size() && items[it].baseline == b; ++it) {
            const idg_metadata &m = items[it];
            for (int32_t t = m.time_offset; t < m.time_offset + m.nr_timesteps; ++t)
                std::fill(cov.begin() + int64_t(t) * C + m.channel_begin, cov.begin() + int64_t(t) * C + m.channel_end,
                          uint8_t(1));
        }
        for (int64_t i = 0; i < per;) {
            if (cov[size_t(i)]) { ++i; continue; }
            int64_t j = i;
            while (j < per && !cov[size_t(j)]) ++j;
            out.push_back(int64_t(b) * per + i);
            out.push_back(j - i);
            i = j;
        }
    }
}

idg::KernelArgs make_args(const idg_plan *plan, const DeviceCopy *dc, const float *d_uvw,
                          const void *d_aterms, const float *d_taper, void *d_vis, void *d_grid) {
    idg::KernelArgs a{};
    const auto &p = plan->params;
    a.subgrid_size = p.subgrid_size;
    a.grid_size = p.grid_size;
    a.cell_l = float(p.image_size / p.subgrid_size);
    a.inv_image_size = 1.0 / p.image_size;
    a.w_offset = p.w_offset;
    a.nr_w_planes = p.nr_w_planes > 1 ? p.nr_w_planes : 1;
    a.w_step = p.nr_w_planes > 1 ? p.w_step : 0.0;
    a.nr_stations = plan->nr_stations;
    a.nr_baselines = plan->nr_baselines;
    a.nr_timesteps = plan->nr_timesteps;
    a.nr_channels = plan->nr_channels;
    a.nr_items = int64_t(plan->items.size());
    a.items = dc->items;
    a.order = dc->order;
    a.baselines = dc->baselines;
    a.frequencies = dc->frequencies;
    a.uvw = d_uvw;
    a.aterms = static_cast<const float2 *>(d_aterms);
    a.taper = d_taper;
    a.vis = static_cast<float2 *>(d_vis);
    a.grid = static_cast<float2 *>(d_grid);
    a.max_channels_in_item = plan->max_channels_in_item;
    a.max_timesteps_in_item = plan->max_timesteps_in_item;
    a.mean_timesteps_in_item = plan->mean_timesteps_in_item;
    a.channel_gcd = plan->channel_gcd;
    a.channels_uniform = plan->channels_uniform;
    a.channel_step = plan->channel_step;
    return a;
}

}  // namespace

extern "C" {

const char *idg_status_string(idg_status s) {
    switch (s) {
        case IDG_OK: return "IDG_OK";
        case IDG_ERR_INVALID_ARG: return "IDG_ERR_INVALID_ARG";
        case IDG_ERR_UNSUPPORTED: return "IDG_ERR_UNSUPPORTED";
        case IDG_ERR_OUT_OF_MEMORY: return "IDG_ERR_OUT_OF_MEMORY";
        case IDG_ERR_CUDA: return "IDG_ERR_CUDA";
        case IDG_ERR_WORKSPACE_TOO_SMALL: return "IDG_ERR_WORKSPACE_TOO_SMALL";
    }
    return "IDG_ERR_UNKNOWN";
}

const char *idg_last_error(void) { return g_last_error.c_str(); }

int64_t idg_launch_count(void) { return g_launches.load(); }

const char *idg_kernel_variants(int32_t which) { return idg::variant_names(which == 0 ? 0 : 1); }

const char *idg_last_variant(int32_t which) { return idg::last_variant(which == 0 ? 0 : 1); }

idg_status idg_plan_create(const idg_plan_params *params, int32_t nr_stations, int32_t nr_baselines,
                           int32_t nr_timesteps, int32_t nr_channels, const float *uvw,
                           const double *frequencies, const idg_baseline *baselines,
                           int32_t nr_aterm_slots, const int32_t *aterm_offsets, idg_plan **out) {
    try {
        if (!out) return fail(IDG_ERR_INVALID_ARG, "out is NULL");
        *out = nullptr;
        idg_status st = validate_params(params);
        if (st != IDG_OK) return st;
        if (nr_stations < 2 || nr_baselines < 0 || nr_timesteps < 1 || nr_channels < 1 ||
            nr_aterm_slots < 1)
            return fail(IDG_ERR_INVALID_ARG, "need nr_stations >= 2, nr_baselines >= 0, "
                                             "nr_timesteps >= 1, nr_channels >= 1, nr_aterm_slots >= 1");
        if ((nr_baselines > 0 && (!uvw || !baselines)) || !frequencies || !aterm_offsets)
            return fail(IDG_ERR_INVALID_ARG, "NULL host array");
        for (int32_t c = 0; c < nr_channels; ++c)
            if (!(frequencies[c] > 0.0) || !std::isfinite(frequencies[c]))
                return fail(IDG_ERR_INVALID_ARG, "frequencies must be positive and finite");
        if (aterm_offsets[0] != 0 || aterm_offsets[nr_aterm_slots] != nr_timesteps)
            return fail(IDG_ERR_INVALID_ARG, "aterm_offsets must start at 0 and end at nr_timesteps");
        for (int32_t s = 0; s < nr_aterm_slots; ++s)
            if (aterm_offsets[s + 1] <= aterm_offsets[s])
                return fail(IDG_ERR_INVALID_ARG, "aterm_offsets must be strictly increasing");
        for (int32_t b = 0; b < nr_baselines; ++b)
            if (baselines[b].station1 < 0 || baselines[b].station1 >= baselines[b].station2 ||
                baselines[b].station2 >= nr_stations)
                return fail(IDG_ERR_INVALID_ARG, "baseline " + std::to_string(b) +
                                                     ": need 0 <= station1 < station2 < nr_stations");

        auto plan = std::make_unique<idg_plan>();
        plan->params = *params;
        plan->nr_stations = nr_stations;
        plan->nr_baselines = nr_baselines;
        plan->nr_timesteps = nr_timesteps;
        plan->nr_channels = nr_channels;
        plan->nr_aterm_slots = nr_aterm_slots;
        plan->frequencies.assign(frequencies, frequencies + nr_channels);
        plan->baselines.resize(size_t(nr_baselines) * 2);
        for (int32_t b = 0; b < nr_baselines; ++b) {
            plan->baselines[2 * b] = baselines[b].station1;
            plan->baselines[2 * b + 1] = baselines[b].station2;
        }
        idg::PlanResult res;
        std::string err;
        st = idg::build_plan(*params, nr_stations, nr_baselines, nr_timesteps, nr_channels, uvw,
                             frequencies, baselines, nr_aterm_slots, aterm_offsets, plan->items, res, err);
        if (st != IDG_OK) return fail(st, err);
        if (plan->items.size() > size_t(0x7fffffff))
            return fail(IDG_ERR_UNSUPPORTED, "more than 2^31-1 work items");
        plan->nr_vis_assigned = res.nr_vis_assigned;
        plan->nr_vis_dropped = res.nr_vis_dropped;
        const int64_t npix = int64_t(params->subgrid_size) * params->subgrid_size;
        int g = 0;
        double sum_t = 0.0;
        for (const auto &it : plan->items) {
            const int nc = it.channel_end - it.channel_begin;
            plan->nr_pairs += npix * it.nr_timesteps * nc;
            plan->max_channels_in_item = std::max(plan->max_channels_in_item, nc);
            plan->max_timesteps_in_item = std::max(plan->max_timesteps_in_item, it.nr_timesteps);
            sum_t += double(it.nr_timesteps);
            g = std::gcd(g, nc);
        }
        plan->channel_gcd = g == 0 ? 1 : g;
        plan->mean_timesteps_in_item = plan->items.empty() ? 0.0f : float(sum_t / double(plan->items.size()));
        // uniform channel spacing (enables the phasor recurrence over channels in the gridder)
        // (every nu_c within 1e-12 nu_0 of nu_0 + c d: the kernels that rotate phasors across channels
        // then see phase errors below 2 pi |u| 1e-12 nu_0 C / c * L/2 ~ 1e-6 rad at the configs)
        if (nr_channels >= 2) {
            const double d0 = (frequencies[nr_channels - 1] - frequencies[0]) / double(nr_channels - 1);
            bool uni = d0 != 0.0;
            for (int32_t c = 1; c < nr_channels && uni; ++c)
                uni = std::fabs(frequencies[c] - (frequencies[0] + double(c) * d0)) <= 1e-12 * std::fabs(frequencies[0]);
            plan->channels_uniform = uni ? 1 : 0;
            plan->channel_step = float(d0 / idg::kSpeedOfLight);
        }
        if (plan->nr_vis_dropped > 0)
            dropped_ranges(plan->items, nr_baselines, nr_timesteps, nr_channels, plan->dropped);
        // host-streamed work groups: contiguous baseline ranges of <= kHostChunkBytes visibilities
        {
            const size_t bl_bytes = size_t(nr_timesteps) * nr_channels * 32;
            size_t chunk = kHostChunkBytes;
            if (const char *env = std::getenv("IDG_HOST_CHUNK_BYTES")) chunk = std::max<size_t>(1, std::strtoull(env, nullptr, 10));
            const int32_t per = int32_t(std::max<size_t>(1, chunk / std::max<size_t>(1, bl_bytes)));
            int64_t it = 0, r = 0;
            const int64_t nr = int64_t(plan->dropped.size() / 2);
            const int64_t vis_per_bl = int64_t(nr_timesteps) * nr_channels;
            for (int32_t b0 = 0; b0 < nr_baselines; b0 += per) {
                const int32_t b1 = std::min(nr_baselines, b0 + per);
                const int64_t i0 = it, r0 = r;
                while (it < int64_t(plan->items.size()) && plan->items[it].baseline < b1) ++it;
                while (r < nr && plan->dropped[2 * r] < int64_t(b1) * vis_per_bl) ++r;
                plan->groups.push_back(WorkGroup{b0, b1, i0, it, r0, r});
                plan->group_bytes = std::max(plan->group_bytes, size_t(b1 - b0) * bl_bytes);
                plan->group_items = std::max(plan->group_items, it - i0);
            }
        }
        plan->order.resize(plan->items.size());
        std::iota(plan->order.begin(), plan->order.end(), 0);
        std::stable_sort(plan->order.begin(), plan->order.end(), [&](int32_t a, int32_t b) {
            const auto &ia = plan->items[a], &ib = plan->items[b];
            return int64_t(ia.nr_timesteps) * (ia.channel_end - ia.channel_begin) >
                   int64_t(ib.nr_timesteps) * (ib.channel_end - ib.channel_begin);
        });
        *out = plan.release();
        return IDG_OK;
    } catch (const std::bad_alloc &) {
        return fail(IDG_ERR_OUT_OF_MEMORY, "host allocation failed in idg_plan_create");
    } catch (const std::exception &e) {
        return fail(IDG_ERR_INVALID_ARG, e.what());
    }
}

idg_status idg_plan_destroy(idg_plan *plan) {
    delete plan;
    return IDG_OK;
}

idg_status idg_plan_nr_subgrids(const idg_plan *plan, int64_t *n) {
    if (!plan || !n) return fail(IDG_ERR_INVALID_ARG, "NULL argument");
    *n = int64_t(plan->items.size());
    return IDG_OK;
}

idg_status idg_plan_metadata(const idg_plan *plan, idg_metadata *dst, int64_t n) {
    if (!plan || (!dst && n > 0) || n < 0) return fail(IDG_ERR_INVALID_ARG, "bad argument");
    const int64_t k = std::min<int64_t>(n, int64_t(plan->items.size()));
    if (k > 0) std::memcpy(dst, plan->items.data(), size_t(k) * sizeof(idg_metadata));
    return IDG_OK;
}

idg_status idg_plan_stats(const idg_plan *plan, int64_t *assigned, int64_t *dropped, int64_t *pairs) {
    if (!plan) return fail(IDG_ERR_INVALID_ARG, "plan is NULL");
    if (assigned) *assigned = plan->nr_vis_assigned;
    if (dropped) *dropped = plan->nr_vis_dropped;
    if (pairs) *pairs = plan->nr_pairs;
    return IDG_OK;
}

idg_status idg_workspace_size(const idg_plan *plan, size_t *bytes) {
    if (!plan || !bytes) return fail(IDG_ERR_INVALID_ARG, "NULL argument");
    *bytes = 0;  // gridder/degridder are fused with FFT + adder/splitter: no subgrid round trip
    return IDG_OK;
}

idg_status idg_host_workspace_size(const idg_plan *plan, size_t *bytes) {
    if (!plan || !bytes) return fail(IDG_ERR_INVALID_ARG, "NULL argument");
    // kStagingBuffers staging buffers for gridding + as many for degridding (separate, so that the
    // uploads of a grid call overlap a preceding degrid call and its downloads)
    *bytes = size_t(2) * kStagingBuffers * plan->group_bytes;
    return IDG_OK;
}

idg_status idg_grid(const idg_plan *plan, const void *d_vis, const float *d_uvw, const void *d_aterms,
                    const float *d_taper, void *d_grid, void *d_workspace, size_t workspace_bytes,
                    idg_stream stream) {
    (void)d_workspace;
    (void)workspace_bytes;
    try {
        idg_status st = validate_call(plan, d_vis, d_uvw, d_aterms, d_taper, d_grid);
        if (st != IDG_OK || plan->items.empty()) return st;
        const DeviceCopy *dc = nullptr;
        if ((st = plan->device_copy(&dc)) != IDG_OK) return st;
        idg::KernelArgs a = make_args(plan, dc, d_uvw, d_aterms, d_taper, const_cast<void *>(d_vis), d_grid);
        cudaError_t e = idg::launch_gridder(a, reinterpret_cast<cudaStream_t>(stream));
        if (e != cudaSuccess) return cuda_fail(e, "gridder launch");
        return IDG_OK;
    } catch (const std::exception &ex) {
        return fail(IDG_ERR_INVALID_ARG, ex.what());
    }
}

idg_status idg_degrid(const idg_plan *plan, const void *d_grid, const float *d_uvw, const void *d_aterms,
                      const float *d_taper, void *d_vis, void *d_workspace, size_t workspace_bytes,
                      idg_stream stream) {
    (void)d_workspace;
    (void)workspace_bytes;
    try {
        if (!plan) return fail(IDG_ERR_INVALID_ARG, "plan is NULL");
        const cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
        if (plan->items.empty()) {
            // nothing to predict: every visibility is dropped and defined as 0 (R-12, R-13)
            const size_t bytes = size_t(plan->nr_baselines) * plan->nr_timesteps * plan->nr_channels * 32;
            if (bytes > 0 && !d_vis) return fail(IDG_ERR_INVALID_ARG, "d_vis is NULL");
            cudaError_t e = bytes > 0 ? cudaMemsetAsync(d_vis, 0, bytes, s) : cudaSuccess;
            return e == cudaSuccess ? IDG_OK : cuda_fail(e, "cudaMemsetAsync(vis)");
        }
        idg_status st = validate_call(plan, d_vis, d_uvw, d_aterms, d_taper, d_grid);
        if (st != IDG_OK) return st;
        const DeviceCopy *dc = nullptr;
        if ((st = plan->device_copy(&dc)) != IDG_OK) return st;
        // dropped visibilities are 0 (R-12, R-13): only their runs are written; the items overwrite the rest
        cudaError_t e = zero_dropped(dc, d_vis, 0, 0, int64_t(plan->dropped.size() / 2), s);
        if (e != cudaSuccess) return cuda_fail(e, "zero dropped visibilities");
        idg::KernelArgs a = make_args(plan, dc, d_uvw, d_aterms, d_taper, d_vis, const_cast<void *>(d_grid));
        e = idg::launch_degridder(a, s);
        if (e != cudaSuccess) return cuda_fail(e, "degridder launch");
        return IDG_OK;
    } catch (const std::exception &ex) {
        return fail(IDG_ERR_INVALID_ARG, ex.what());
    }
}

// ------------------------------------------------------------------------------------------------
// Banded grid (peer memory): the grid is distributed over the ranks by row bands and the adder / splitter
// of every work item goes straight to the owner's band -- the cross-rank sum of the gridded subgrids
// (the adder, independent work split over devices) and the model-grid broadcast of the
// degridding step are fused into the kernels instead of following them as collectives.
// ------------------------------------------------------------------------------------------------
static idg_status validate_bands(const idg_plan *plan, const void *bands, int32_t nr_bands, int32_t band_rows) {
    if (!bands) return fail(IDG_ERR_INVALID_ARG, "d_bands is NULL");
    if (nr_bands < 1 || band_rows < 1)
        return fail(IDG_ERR_INVALID_ARG, "nr_bands and band_rows must be >= 1");
    if (int64_t(nr_bands) * band_rows < plan->params.grid_size)
        return fail(IDG_ERR_INVALID_ARG, "nr_bands * band_rows must cover the grid_size rows");
    return IDG_OK;
}

idg_status idg_grid_bands(const idg_plan *plan, const void *d_vis, const float *d_uvw, const void *d_aterms,
                          const float *d_taper, void *const *d_bands, int32_t nr_bands, int32_t band_rows,
                          idg_stream stream) {
    try {
        idg_status st = validate_call(plan, d_vis, d_uvw, d_aterms, d_taper, d_bands);
        if (st != IDG_OK) return st;
        if ((st = validate_bands(plan, d_bands, nr_bands, band_rows)) != IDG_OK || plan->items.empty()) return st;
        const DeviceCopy *dc = nullptr;
        if ((st = plan->device_copy(&dc)) != IDG_OK) return st;
        idg::KernelArgs a = make_args(plan, dc, d_uvw, d_aterms, d_taper, const_cast<void *>(d_vis), nullptr);
        a.bands = reinterpret_cast<float2 *const *>(d_bands);
        a.band_rows = band_rows;
        cudaError_t e = idg::launch_gridder(a, reinterpret_cast<cudaStream_t>(stream));
        if (e != cudaSuccess) return cuda_fail(e, "gridder launch (banded)");
        return IDG_OK;
    } catch (const std::exception &ex) {
        return fail(IDG_ERR_INVALID_ARG, ex.what());
    }
}

idg_status idg_degrid_bands(const idg_plan *plan, const void *const *d_bands, int32_t nr_bands, int32_t band_rows,
                            const float *d_uvw, const void *d_aterms, const float *d_taper, void *d_vis,
                            idg_stream stream) {
    try {
        if (!plan) return fail(IDG_ERR_INVALID_ARG, "plan is NULL");
        const cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
        if (plan->items.empty()) {   // every visibility dropped: all 0 (R-12, R-13)
            const size_t bytes = size_t(plan->nr_baselines) * plan->nr_timesteps * plan->nr_channels * 32;
            if (bytes > 0 && !d_vis) return fail(IDG_ERR_INVALID_ARG, "d_vis is NULL");
            cudaError_t e = bytes > 0 ? cudaMemsetAsync(d_vis, 0, bytes, s) : cudaSuccess;
            return e == cudaSuccess ? IDG_OK : cuda_fail(e, "cudaMemsetAsync(vis)");
        }
        idg_status st = validate_call(plan, d_vis, d_uvw, d_aterms, d_taper, d_bands);
        if (st != IDG_OK) return st;
        if ((st = validate_bands(plan, d_bands, nr_bands, band_rows)) != IDG_OK) return st;
        const DeviceCopy *dc = nullptr;
        if ((st = plan->device_copy(&dc)) != IDG_OK) return st;
        cudaError_t e = zero_dropped(dc, d_vis, 0, 0, int64_t(plan->dropped.size() / 2), s);
        if (e != cudaSuccess) return cuda_fail(e, "zero dropped visibilities");
        idg::KernelArgs a = make_args(plan, dc, d_uvw, d_aterms, d_taper, d_vis, nullptr);
        a.bands = reinterpret_cast<float2 *const *>(const_cast<void *const *>(d_bands));
        a.band_rows = band_rows;
        e = idg::launch_degridder(a, s);
        if (e != cudaSuccess) return cuda_fail(e, "degridder launch (banded)");
        return IDG_OK;
    } catch (const std::exception &ex) {
        return fail(IDG_ERR_INVALID_ARG, ex.what());
    }
}

// CUDA IPC: a band allocated by one process, mapped into the others (peer access over NVLink / NVSwitch
// enabled lazily by the driver).  Handles name whole allocations, so the pointer's offset inside its
// allocation travels with the handle (cuMemGetAddressRange through the runtime's driver entry point: the
// library does not link libcuda).
using AddressRangeFn = int (*)(unsigned long long *, size_t *, unsigned long long);

static cudaError_t allocation_base(const void *p, const void **base) {
    static AddressRangeFn fn = nullptr;
    if (!fn) {
        void *f = nullptr;
        cudaDriverEntryPointQueryResult q{};
        cudaError_t e = cudaGetDriverEntryPoint("cuMemGetAddressRange", &f, cudaEnableDefault, &q);
        if (e != cudaSuccess) return e;
        if (!f || q != cudaDriverEntryPointSuccess) return cudaErrorNotSupported;
        fn = reinterpret_cast<AddressRangeFn>(f);
    }
    unsigned long long b = 0;
    size_t n = 0;
    if (fn(&b, &n, reinterpret_cast<unsigned long long>(p)) != 0) return cudaErrorInvalidValue;
    *base = reinterpret_cast<const void *>(b);
    return cudaSuccess;
}

idg_status idg_ipc_handle(const void *d_ptr, unsigned char handle[64], uint64_t *offset) {
    if (!d_ptr || !handle || !offset) return fail(IDG_ERR_INVALID_ARG, "NULL argument");
    static_assert(sizeof(cudaIpcMemHandle_t) == 64, "CUDA IPC handle size");
    const void *base = nullptr;
    cudaError_t e = allocation_base(d_ptr, &base);
    if (e != cudaSuccess) return cuda_fail(e, "allocation range of d_ptr");
    cudaIpcMemHandle_t h;
    if ((e = cudaIpcGetMemHandle(&h, const_cast<void *>(base))) != cudaSuccess) return cuda_fail(e, "cudaIpcGetMemHandle");
    std::memcpy(handle, &h, 64);
    *offset = uint64_t(static_cast<const char *>(d_ptr) - static_cast<const char *>(base));
    return IDG_OK;
}

idg_status idg_ipc_open(const unsigned char handle[64], uint64_t offset, void **d_ptr) {
    if (!handle || !d_ptr) return fail(IDG_ERR_INVALID_ARG, "NULL argument");
    cudaIpcMemHandle_t h;
    std::memcpy(&h, handle, 64);
    void *base = nullptr;
    cudaError_t e = cudaIpcOpenMemHandle(&base, h, cudaIpcMemLazyEnablePeerAccess);
    if (e != cudaSuccess) return cuda_fail(e, "cudaIpcOpenMemHandle");
    *d_ptr = static_cast<char *>(base) + offset;
    return IDG_OK;
}

idg_status idg_ipc_close(void *d_ptr, uint64_t offset) {
    if (!d_ptr) return fail(IDG_ERR_INVALID_ARG, "d_ptr is NULL");
    cudaError_t e = cudaIpcCloseMemHandle(static_cast<char *>(d_ptr) - offset);
    return e == cudaSuccess ? IDG_OK : cuda_fail(e, "cudaIpcCloseMemHandle");
}

// ------------------------------------------------------------------------------------------------
// Host-streamed calls: the paper's asynchronous I/O with triple buffering (Fig. 7).  Work
// groups (contiguous baseline ranges) stream through kStagingBuffers device buffers; uploads run on a
// copy stream, downloads on another, kernels on the caller's stream, ordered with events.
// ------------------------------------------------------------------------------------------------
// A failing event call inside the pipeline is reported like a failing copy or launch.
#define IDG_PIPE(call)                      \
    do {                                    \
        if ((e = (call)) != cudaSuccess) {  \
            what = #call;                   \
            goto pipe_error;                \
        }                                   \
    } while (0)

idg_status idg_grid_host(const idg_plan *plan, const void *h_vis, const float *d_uvw, const void *d_aterms,
                         const float *d_taper, void *d_grid, void *d_workspace, size_t workspace_bytes,
                         idg_stream stream) {
    try {
        idg_status st = validate_call(plan, h_vis, d_uvw, d_aterms, d_taper, d_grid);
        if (st != IDG_OK || plan->items.empty()) return st;
        const size_t need = size_t(2) * kStagingBuffers * plan->group_bytes;
        if (!d_workspace || workspace_bytes < need)
            return fail(IDG_ERR_WORKSPACE_TOO_SMALL, "host-streamed gridding needs idg_host_workspace_size() = " +
                                                         std::to_string(need) + " bytes");
        const DeviceCopy *dc = nullptr;
        if ((st = plan->device_copy(&dc)) != IDG_OK) return st;
        std::lock_guard<std::mutex> lock(*dc->pipeline_mu);
        const cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
        const size_t bl_bytes = size_t(plan->nr_timesteps) * plan->nr_channels * 32;
        const int64_t bl_f2 = int64_t(plan->nr_timesteps) * plan->nr_channels * 4;  // float2 per baseline
        const int nb = staging_buffers(plan, workspace_bytes);
        char *staging = static_cast<char *>(d_workspace);                        // grid half of the workspace
        const char *what = "";
        PipeEvents *pe = nullptr;
        cudaError_t e = pipe_events(dc, d_workspace, nb, &pe);
        if (e != cudaSuccess) return cuda_fail(e, "idg_grid_host: events");
        // the uploads read h_vis and overwrite the staging buffers: both may still be in use by work the
        // caller queued on `stream` before this call (a copy into h_vis, a kernel on a recycled workspace)
        IDG_PIPE(cudaEventRecord(pe->entry, s));
        IDG_PIPE(cudaStreamWaitEvent(dc->h2d, pe->entry, 0));
        for (size_t gi = 0; gi < plan->groups.size(); ++gi) {
            const WorkGroup &g = plan->groups[gi];
            const int b = int(gi % nb);
            char *buf = staging + size_t(b) * plan->group_bytes;
            // the buffer is free once the gridder that last read it has finished
            // (also across calls: an event never recorded is complete)
            IDG_PIPE(cudaStreamWaitEvent(dc->h2d, pe->kernel_g[b], 0));
            IDG_PIPE(cudaMemcpyAsync(buf, static_cast<const char *>(h_vis) + size_t(g.b0) * bl_bytes,
                                     size_t(g.b1 - g.b0) * bl_bytes, cudaMemcpyHostToDevice, dc->h2d));
            IDG_PIPE(cudaEventRecord(pe->h2d[b], dc->h2d));
            IDG_PIPE(cudaStreamWaitEvent(s, pe->h2d[b], 0));
            if (g.i1 > g.i0) {
                idg::KernelArgs a = make_args(plan, dc, d_uvw, d_aterms, d_taper,
                                              reinterpret_cast<float2 *>(buf) - int64_t(g.b0) * bl_f2, d_grid);
                a.order = dc->iota + g.i0;
                a.nr_items = g.i1 - g.i0;
                IDG_PIPE(idg::launch_gridder(a, s));
            }
            IDG_PIPE(cudaEventRecord(pe->kernel_g[b], s));
        }
        return IDG_OK;
    pipe_error:
        return cuda_fail(e, std::string("idg_grid_host: ") + what);
    } catch (const std::exception &ex) {
        return fail(IDG_ERR_INVALID_ARG, ex.what());
    }
}

idg_status idg_degrid_host(const idg_plan *plan, const void *d_grid, const float *d_uvw, const void *d_aterms,
                           const float *d_taper, void *h_vis, void *d_workspace, size_t workspace_bytes,
                           idg_stream stream) {
    try {
        idg_status st = validate_call(plan, h_vis, d_uvw, d_aterms, d_taper, d_grid);
        if (st != IDG_OK) return st;
        const size_t bl_bytes = size_t(plan->nr_timesteps) * plan->nr_channels * 32;
        const cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
        if (plan->items.empty()) {  // nothing to predict: every visibility is dropped -> 0
            const size_t bytes = size_t(plan->nr_baselines) * bl_bytes;
            if (bytes > 0 && !h_vis) return fail(IDG_ERR_INVALID_ARG, "h_vis is NULL");
            // ordered after the caller's work on `stream` (which may still read h_vis), like the downloads
            // (without a CUDA device there is no queued work to wait for)
            cudaError_t e = cudaStreamSynchronize(s);
            if (e == cudaErrorNoDevice || e == cudaErrorInsufficientDriver) e = cudaGetLastError(), e = cudaSuccess;
            if (e != cudaSuccess) return cuda_fail(e, "idg_degrid_host: cudaStreamSynchronize");
            if (bytes > 0) std::memset(h_vis, 0, bytes);
            return IDG_OK;
        }
        const size_t need = size_t(2) * kStagingBuffers * plan->group_bytes;
        if (!d_workspace || workspace_bytes < need)
            return fail(IDG_ERR_WORKSPACE_TOO_SMALL, "host-streamed degridding needs idg_host_workspace_size() = " +
                                                         std::to_string(need) + " bytes");
        const DeviceCopy *dc = nullptr;
        if ((st = plan->device_copy(&dc)) != IDG_OK) return st;
        std::lock_guard<std::mutex> lock(*dc->pipeline_mu);
        const int64_t bl_f2 = int64_t(plan->nr_timesteps) * plan->nr_channels * 4;
        const int64_t bl_vis = int64_t(plan->nr_timesteps) * plan->nr_channels;
        const int nb = staging_buffers(plan, workspace_bytes);
        char *staging = static_cast<char *>(d_workspace) + size_t(nb) * plan->group_bytes;
        const char *what = "";
        PipeEvents *pe = nullptr;
        cudaError_t e = pipe_events(dc, d_workspace, nb, &pe);
        if (e != cudaSuccess) return cuda_fail(e, "idg_degrid_host: events");
        size_t last = 0;
        for (size_t gi = 0; gi < plan->groups.size(); ++gi) {
            const WorkGroup &g = plan->groups[gi];
            const int b = int(gi % nb);
            char *buf = staging + size_t(b) * plan->group_bytes;
            const size_t bytes = size_t(g.b1 - g.b0) * bl_bytes;
            // the buffer is free once its previous download has finished
            IDG_PIPE(cudaStreamWaitEvent(s, pe->d2h[b], 0));
            // dropped visibilities are 0 (R-12, R-13): only their runs are written, the items overwrite the rest
            IDG_PIPE(zero_dropped(dc, buf, int64_t(g.b0) * bl_vis, g.r0, g.r1, s));
            if (g.i1 > g.i0) {
                idg::KernelArgs a = make_args(plan, dc, d_uvw, d_aterms, d_taper,
                                              reinterpret_cast<float2 *>(buf) - int64_t(g.b0) * bl_f2,
                                              const_cast<void *>(d_grid));
                a.order = dc->iota + g.i0;
                a.nr_items = g.i1 - g.i0;
                IDG_PIPE(idg::launch_degridder(a, s));
            }
            // (the downloads start after all of the caller's earlier work on `stream`, which may read h_vis)
            IDG_PIPE(cudaEventRecord(pe->kernel_d[b], s));
            IDG_PIPE(cudaStreamWaitEvent(dc->d2h, pe->kernel_d[b], 0));
            IDG_PIPE(cudaMemcpyAsync(static_cast<char *>(h_vis) + size_t(g.b0) * bl_bytes, buf, bytes,
                                     cudaMemcpyDeviceToHost, dc->d2h));
            IDG_PIPE(cudaEventRecord(pe->d2h[b], dc->d2h));
            last = gi;
        }
        // completion of the call is observable on the caller's stream
        for (int b = 0; b < nb && size_t(b) <= last; ++b) IDG_PIPE(cudaStreamWaitEvent(s, pe->d2h[b], 0));
        return IDG_OK;
    pipe_error:
        return cuda_fail(e, std::string("idg_degrid_host: ") + what);
    } catch (const std::exception &ex) {
        return fail(IDG_ERR_INVALID_ARG, ex.what());
    }
}
#undef IDG_PIPE

}  // extern "C"

// ------------------------------------------------------------------------------------------------
// Host adder / splitter (Section V-C-e, option 2): "copy the subgrids into host memory and perform
// the operation on the CPU ... required when dealing with large images that no longer fit into GPU device
// memory".  The grid lives in HOST memory; the kernels write (gridding) or read (degridding) the work
// group's transformed subgrids in a device buffer, which streams to / from page-locked host buffers; host
// threads add them into (or split them out of) the host grid while the GPU works on the next groups.
// ------------------------------------------------------------------------------------------------
namespace {

size_t subgrid_bytes(const idg_plan *plan) { return size_t(4) * plan->params.subgrid_size * plan->params.subgrid_size * 8; }
size_t adder_buffer_bytes(const idg_plan *plan) {   // one staging buffer: visibilities + subgrids of a work group
    return plan->group_bytes + size_t(plan->group_items) * subgrid_bytes(plan);
}

// page-locked host subgrid buffers (n of them) of a workspace's pipeline
cudaError_t host_subgrid_buffers(PipeEvents *pe, int n, size_t bytes) {
    if (pe->host_subgrid_bytes < bytes) {
        for (void *p : pe->host_subgrids) cudaFreeHost(p);
        pe->host_subgrids.clear();
        pe->host_subgrid_bytes = bytes;
    }
    while (int(pe->host_subgrids.size()) < n) {
        void *p = nullptr;
        cudaError_t e = cudaHostAlloc(&p, std::max<size_t>(1, bytes), cudaHostAllocDefault);
        if (e != cudaSuccess) return e;
        pe->host_subgrids.push_back(p);
    }
    return cudaSuccess;
}

// grid[z][pol][y + ky][x + kx] (+)= sub[j][pol][ky][kx] for the items [i0, i1); rows interleaved over threads
// (row r -> thread r mod T), so no two threads touch the same grid row and no atomics are needed.
void host_add_or_split(const idg_plan *plan, HostPool &pool, int64_t i0, int64_t i1, std::complex<float> *grid,
                       std::complex<float> *sub, bool add) {
    const int ns = plan->params.subgrid_size;
    const int64_t N = plan->params.grid_size;
    pool.run([&](int t, int T) {
        for (int64_t j = i0; j < i1; ++j) {
            const idg_metadata &m = plan->items[size_t(j)];
            std::complex<float> *s = sub + (j - i0) * 4 * ns * ns;
            int ky0 = int(((int64_t(t) - m.y) % T + T) % T);
            for (int ky = ky0; ky < ns; ky += T)
                for (int pol = 0; pol < 4; ++pol) {
                    std::complex<float> *g = grid + ((int64_t(m.z) * 4 + pol) * N + m.y + ky) * N + m.x;
                    std::complex<float> *r = s + (int64_t(pol) * ns + ky) * ns;
                    if (add)
                        for (int kx = 0; kx < ns; ++kx) g[kx] += r[kx];
                    else
                        std::memcpy(r, g, size_t(ns) * sizeof(std::complex<float>));
                }
        }
    });
}

}  // namespace

extern "C" {

idg_status idg_host_adder_workspace_size(const idg_plan *plan, size_t *bytes) {
    if (!plan || !bytes) return fail(IDG_ERR_INVALID_ARG, "NULL argument");
    *bytes = size_t(2) * kStagingBuffers * adder_buffer_bytes(plan);
    return IDG_OK;
}

#define IDG_PIPE(call)                      \
    do {                                    \
        if ((e = (call)) != cudaSuccess) {  \
            what = #call;                   \
            goto pipe_error;                \
        }                                   \
    } while (0)

idg_status idg_grid_host_adder(const idg_plan *plan, const void *h_vis, const float *d_uvw, const void *d_aterms,
                               const float *d_taper, void *h_grid, void *d_workspace, size_t workspace_bytes,
                               idg_stream stream) {
    try {
        idg_status st = validate_call(plan, h_vis, d_uvw, d_aterms, d_taper, h_grid);
        if (st != IDG_OK || plan->items.empty()) return st;
        const size_t per = adder_buffer_bytes(plan);
        if (!d_workspace || workspace_bytes < size_t(2) * kStagingBuffers * per)
            return fail(IDG_ERR_WORKSPACE_TOO_SMALL, "idg_grid_host_adder needs idg_host_adder_workspace_size() = " +
                                                         std::to_string(size_t(2) * kStagingBuffers * per) + " bytes");
        const DeviceCopy *dc = nullptr;
        if ((st = plan->device_copy(&dc)) != IDG_OK) return st;
        std::lock_guard<std::mutex> lock(*dc->pipeline_mu);
        const cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
        const size_t bl_bytes = size_t(plan->nr_timesteps) * plan->nr_channels * 32;
        const int64_t bl_f2 = int64_t(plan->nr_timesteps) * plan->nr_channels * 4;
        const size_t sgb = subgrid_bytes(plan);
        const int nb = int(std::max<size_t>(kStagingBuffers, std::min(workspace_bytes / (2 * per), plan->groups.size())));
        char *base = static_cast<char *>(d_workspace);        // grid half: [nb][vis | subgrids]
        const char *what = "";
        PipeEvents *pe = nullptr;
        cudaError_t e = pipe_events(dc, d_workspace, nb, &pe);
        if (e == cudaSuccess) e = host_subgrid_buffers(pe, 2 * nb, size_t(plan->group_items) * sgb);
        if (e != cudaSuccess) return cuda_fail(e, "idg_grid_host_adder: events / host buffers");
        HostPool pool(host_threads());
        auto *grid = static_cast<std::complex<float> *>(h_grid);
        auto drain = [&](size_t gj) -> cudaError_t {   // host-add work group gj once its subgrids have arrived
            const int b = int(gj % nb);
            cudaError_t err = cudaEventSynchronize(pe->d2h[b]);
            if (err != cudaSuccess) return err;
            host_add_or_split(plan, pool, plan->groups[gj].i0, plan->groups[gj].i1, grid,
                              static_cast<std::complex<float> *>(pe->host_subgrids[b]), true);
            return cudaSuccess;
        };
        IDG_PIPE(cudaEventRecord(pe->entry, s));
        IDG_PIPE(cudaStreamWaitEvent(dc->h2d, pe->entry, 0));
        for (size_t gi = 0; gi < plan->groups.size(); ++gi) {
            const WorkGroup &g = plan->groups[gi];
            const int b = int(gi % nb);
            char *vbuf = base + size_t(b) * per;
            auto *sbuf = reinterpret_cast<float2 *>(vbuf + plan->group_bytes);
            if (gi >= size_t(nb)) IDG_PIPE(drain(gi - nb));   // frees host buffer b (and overlaps the GPU)
            IDG_PIPE(cudaStreamWaitEvent(dc->h2d, pe->kernel_g[b], 0));
            IDG_PIPE(cudaMemcpyAsync(vbuf, static_cast<const char *>(h_vis) + size_t(g.b0) * bl_bytes,
                                     size_t(g.b1 - g.b0) * bl_bytes, cudaMemcpyHostToDevice, dc->h2d));
            IDG_PIPE(cudaEventRecord(pe->h2d[b], dc->h2d));
            IDG_PIPE(cudaStreamWaitEvent(s, pe->h2d[b], 0));
            IDG_PIPE(cudaStreamWaitEvent(s, pe->d2h[b], 0));  // the subgrid buffer's previous download
            if (g.i1 > g.i0) {
                idg::KernelArgs a = make_args(plan, dc, d_uvw, d_aterms, d_taper,
                                              reinterpret_cast<float2 *>(vbuf) - int64_t(g.b0) * bl_f2, nullptr);
                a.subgrids = sbuf;
                a.order = dc->iota + g.i0;
                a.nr_items = g.i1 - g.i0;
                IDG_PIPE(idg::launch_gridder(a, s));
            }
            IDG_PIPE(cudaEventRecord(pe->kernel_g[b], s));
            IDG_PIPE(cudaStreamWaitEvent(dc->d2h, pe->kernel_g[b], 0));
            if (g.i1 > g.i0)
                IDG_PIPE(cudaMemcpyAsync(pe->host_subgrids[b], sbuf, size_t(g.i1 - g.i0) * sgb,
                                         cudaMemcpyDeviceToHost, dc->d2h));
            IDG_PIPE(cudaEventRecord(pe->d2h[b], dc->d2h));
        }
        for (size_t gi = plan->groups.size() > size_t(nb) ? plan->groups.size() - nb : 0; gi < plan->groups.size(); ++gi)
            IDG_PIPE(drain(gi));
        return IDG_OK;
    pipe_error:
        return cuda_fail(e, std::string("idg_grid_host_adder: ") + what);
    } catch (const std::exception &ex) {
        return fail(IDG_ERR_INVALID_ARG, ex.what());
    }
}

idg_status idg_degrid_host_splitter(const idg_plan *plan, const void *h_grid, const float *d_uvw,
                                    const void *d_aterms, const float *d_taper, void *h_vis, void *d_workspace,
                                    size_t workspace_bytes, idg_stream stream) {
    try {
        idg_status st = validate_call(plan, h_vis, d_uvw, d_aterms, d_taper, h_grid);
        if (st != IDG_OK) return st;
        if (plan->items.empty())   // everything dropped: the host-streamed degridder defines it as 0
            return idg_degrid_host(plan, h_grid, d_uvw, d_aterms, d_taper, h_vis, d_workspace, workspace_bytes, stream);
        const size_t per = adder_buffer_bytes(plan);
        if (!d_workspace || workspace_bytes < size_t(2) * kStagingBuffers * per)
            return fail(IDG_ERR_WORKSPACE_TOO_SMALL, "idg_degrid_host_splitter needs idg_host_adder_workspace_size() = " +
                                                         std::to_string(size_t(2) * kStagingBuffers * per) + " bytes");
        const DeviceCopy *dc = nullptr;
        if ((st = plan->device_copy(&dc)) != IDG_OK) return st;
        std::lock_guard<std::mutex> lock(*dc->pipeline_mu);
        const cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
        const size_t bl_bytes = size_t(plan->nr_timesteps) * plan->nr_channels * 32;
        const int64_t bl_f2 = int64_t(plan->nr_timesteps) * plan->nr_channels * 4;
        const int64_t bl_vis = int64_t(plan->nr_timesteps) * plan->nr_channels;
        const size_t sgb = subgrid_bytes(plan);
        const int nb = int(std::max<size_t>(kStagingBuffers, std::min(workspace_bytes / (2 * per), plan->groups.size())));
        char *base = static_cast<char *>(d_workspace) + size_t(nb) * per;   // degrid half
        const char *what = "";
        PipeEvents *pe = nullptr;
        cudaError_t e = pipe_events(dc, d_workspace, nb, &pe);
        if (e == cudaSuccess) e = host_subgrid_buffers(pe, 2 * nb, size_t(plan->group_items) * sgb);
        if (e != cudaSuccess) return cuda_fail(e, "idg_degrid_host_splitter: events / host buffers");
        HostPool pool(host_threads());
        auto *grid = const_cast<std::complex<float> *>(static_cast<const std::complex<float> *>(h_grid));
        size_t last = 0;
        // the host reads h_grid while the caller's earlier work on `stream` may still write it
        IDG_PIPE(cudaStreamSynchronize(s));
        for (size_t gi = 0; gi < plan->groups.size(); ++gi) {
            const WorkGroup &g = plan->groups[gi];
            const int b = int(gi % nb);
            char *vbuf = base + size_t(b) * per;
            auto *sbuf = reinterpret_cast<float2 *>(vbuf + plan->group_bytes);
            void *hsub = pe->host_subgrids[nb + b];
            const size_t bytes = size_t(g.b1 - g.b0) * bl_bytes;
            if (g.i1 > g.i0) {
                // host splitter: the previous upload from this host buffer must have finished
                IDG_PIPE(cudaEventSynchronize(pe->h2d[b]));
                host_add_or_split(plan, pool, g.i0, g.i1, grid, static_cast<std::complex<float> *>(hsub), false);
                IDG_PIPE(cudaStreamWaitEvent(dc->h2d, pe->kernel_d[b], 0));   // the kernel that last read sbuf
                IDG_PIPE(cudaMemcpyAsync(sbuf, hsub, size_t(g.i1 - g.i0) * sgb, cudaMemcpyHostToDevice, dc->h2d));
                IDG_PIPE(cudaEventRecord(pe->h2d[b], dc->h2d));
                IDG_PIPE(cudaStreamWaitEvent(s, pe->h2d[b], 0));
            }
            IDG_PIPE(cudaStreamWaitEvent(s, pe->d2h[b], 0));   // the visibility buffer's previous download
            IDG_PIPE(zero_dropped(dc, vbuf, int64_t(g.b0) * bl_vis, g.r0, g.r1, s));
            if (g.i1 > g.i0) {
                idg::KernelArgs a = make_args(plan, dc, d_uvw, d_aterms, d_taper,
                                              reinterpret_cast<float2 *>(vbuf) - int64_t(g.b0) * bl_f2, nullptr);
                a.subgrids = sbuf;
                a.order = dc->iota + g.i0;
                a.nr_items = g.i1 - g.i0;
                IDG_PIPE(idg::launch_degridder(a, s));
            }
            IDG_PIPE(cudaEventRecord(pe->kernel_d[b], s));
            IDG_PIPE(cudaStreamWaitEvent(dc->d2h, pe->kernel_d[b], 0));
            IDG_PIPE(cudaMemcpyAsync(static_cast<char *>(h_vis) + size_t(g.b0) * bl_bytes, vbuf, bytes,
                                     cudaMemcpyDeviceToHost, dc->d2h));
            IDG_PIPE(cudaEventRecord(pe->d2h[b], dc->d2h));
            last = gi;
        }
        for (int b = 0; b < nb && size_t(b) <= last; ++b) IDG_PIPE(cudaStreamWaitEvent(s, pe->d2h[b], 0));
        return IDG_OK;
    pipe_error:
        return cuda_fail(e, std::string("idg_degrid_host_splitter: ") + what);
    } catch (const std::exception &ex) {
        return fail(IDG_ERR_INVALID_ARG, ex.what());
    }
}
#undef IDG_PIPE

}  // extern "C"

extern "C" {

static idg_status rho_benchmark(int32_t rho, int32_t iterations, idg_stream stream, double *ops_per_second,
                                double *seconds, bool packed) {
    static const int kSupported[] = {0, 1, 2, 3, 4, 6, 8, 12, 16, 17, 20, 24, 32, 48, 64};
    if (std::find(std::begin(kSupported), std::end(kSupported), rho) == std::end(kSupported) ||
        iterations < 1 || !ops_per_second)
        return fail(IDG_ERR_INVALID_ARG,
                    "rho in {0,1,2,3,4,6,8,12,16,17,20,24,32,48,64}, iterations >= 1, ops_per_second != NULL");
    const cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
    float *d_out = nullptr;
    cudaError_t e = cudaMalloc(&d_out, sizeof(float) * 148 * 64 * 256);
    if (e != cudaSuccess) return cuda_fail(e, "cudaMalloc(rho)");
    cudaEvent_t e0 = nullptr, e1 = nullptr;
    int blocks = 0, threads = 0, units = 0;
    if ((e = cudaEventCreate(&e0)) == cudaSuccess && (e = cudaEventCreate(&e1)) == cudaSuccess) {
        // warm-up launch, then the timed one
        e = idg::launch_rho_benchmark(rho, std::max(1, iterations / 8), d_out, s, &blocks, &threads, &units, packed);
        if (e == cudaSuccess) e = cudaEventRecord(e0, s);
        if (e == cudaSuccess) e = idg::launch_rho_benchmark(rho, iterations, d_out, s, &blocks, &threads, &units, packed);
        if (e == cudaSuccess) e = cudaEventRecord(e1, s);
    }
    if (e == cudaSuccess) e = cudaEventSynchronize(e1);
    float ms = 0.0f;
    if (e == cudaSuccess) e = cudaEventElapsedTime(&ms, e0, e1);
    if (e0) cudaEventDestroy(e0);
    if (e1) cudaEventDestroy(e1);
    cudaFree(d_out);
    if (e != cudaSuccess) return cuda_fail(e, "rho benchmark");
    const double sincos = double(blocks) * threads * units * double(iterations);
    const double ops = sincos * (2.0 * rho + 2.0);  // rho FMAs (2 ops each) + sin + cos
    *ops_per_second = ops / (double(ms) * 1e-3);
    if (seconds) *seconds = double(ms) * 1e-3;
    return IDG_OK;
}

idg_status idg_rho_benchmark(int32_t rho, int32_t iterations, idg_stream stream, double *ops_per_second,
                             double *seconds) {
    return rho_benchmark(rho, iterations, stream, ops_per_second, seconds, true);
}

idg_status idg_rho_benchmark_scalar(int32_t rho, int32_t iterations, idg_stream stream, double *ops_per_second,
                                    double *seconds) {
    return rho_benchmark(rho, iterations, stream, ops_per_second, seconds, false);
}

idg_status idg_profiling_enable(int32_t enable) {
    g_prof_enabled.store(enable != 0);
    return IDG_OK;
}

static void drain_profiling_locked() {
    for (auto &r : g_prof_pending) {
        cudaEventSynchronize(r.e1);
        float ms = 0.0f;
        cudaEventElapsedTime(&ms, r.e0, r.e1);
        auto &t = g_prof_totals[r.name];
        t.first += 1;
        t.second += ms;
        cudaEventDestroy(r.e0);
        cudaEventDestroy(r.e1);
    }
    g_prof_pending.clear();
}

idg_status idg_profiling_reset(void) {
    std::lock_guard<std::mutex> lock(g_prof_mu);
    drain_profiling_locked();
    g_prof_totals.clear();
    return IDG_OK;
}

idg_status idg_profiling_read(idg_kernel_time *dst, int32_t capacity, int32_t *n) {
    if (!n || (capacity > 0 && !dst)) return fail(IDG_ERR_INVALID_ARG, "bad argument");
    std::lock_guard<std::mutex> lock(g_prof_mu);
    drain_profiling_locked();
    int32_t k = 0;
    for (auto &kv : g_prof_totals) {
        if (k < capacity) {
            std::memset(dst[k].name, 0, sizeof(dst[k].name));
            std::strncpy(dst[k].name, kv.first.c_str(), sizeof(dst[k].name) - 1);
            dst[k].launches = kv.second.first;
            dst[k].total_ms = kv.second.second;
        }
        ++k;
    }
    *n = k;
    return IDG_OK;
}

}  // extern "C"
