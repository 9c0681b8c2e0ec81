#!/usr/bin/env python
"""IDG gridding + degridding throughput on B200 (BASELINE.json metric), one JSON line on rank 0.

A step = one pass of the hot path over the SKA-low-shaped data set on an 8192^2 grid (BASELINE.json
configs[3], the north star's 8-GPU target; --config lofar / lofar_dde / predict / tiny for the others):
    grid(visibilities) -> [N>1: NCCL reduce of the uv-grid to rank 0 -> broadcast] -> degrid(grid)
(predict, configs[4]: broadcast of the model grid -> degrid only).  The plan (host, built once per
observation, "before any execution") is built before the timed region and reported as plan_s.
value = visibilities per step / step time (MVis/s), whole job; with N GPUs the baselines are split into
N contiguous shards (strong scaling).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config ska] [--impl ours|reference]

--impl reference times the fp64 CPU oracle (oracle/, the correctness reference) on the host cores, on a
bounded sample of the same workload per step; under torchrun only rank 0 runs it.
"""
from __future__ import annotations

import argparse
import json
import math
import os
import re
import statistics
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import idgsynth  # noqa: E402

BASELINE = json.load(open(os.path.join(ROOT, "BASELINE.json")))
METRIC = BASELINE["metric"]
OPS_PER_PAIR = 36        # 17 FMA (2 ops) + sin + cos per (pixel, visibility) pair
CONFIG_NAMES = {"tiny": 0, "lofar": 1, "lofar_dde": 2, "ska": 3, "predict": 4, "lofar_short": 1}


def log(*a):
    print(*a, file=sys.stderr, flush=True)


# ------------------------------------------------------------------------------------------------
# clocks during the timed region (NVML = what nvidia-smi reads)
# ------------------------------------------------------------------------------------------------
class ClockSampler:
    REASONS = {0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap",
               0x8: "hw_slowdown", 0x10: "sync_boost", 0x20: "sw_thermal_slowdown",
               0x40: "hw_thermal_slowdown", 0x80: "hw_power_brake_slowdown", 0x100: "display_clock_setting"}

    def __init__(self, torch_device: int, period_s: float = 0.1):
        self.period = period_s
        self.samples, self.reasons = [], set()
        self.max_mhz = None
        self._stop = threading.Event()
        self._h = None
        try:
            import pynvml
            pynvml.nvmlInit()
            import torch
            p = torch.cuda.get_device_properties(torch_device)
            bus = f"{p.pci_domain_id:08x}:{p.pci_bus_id:02x}:{p.pci_device_id:02x}.0"
            self._h = pynvml.nvmlDeviceGetHandleByPciBusId(bus.encode())
            self._nvml = pynvml
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self._h, pynvml.NVML_CLOCK_SM)
        except Exception as e:  # pragma: no cover
            log(f"[bench] NVML unavailable: {e}")

    def _run(self):
        n = self._nvml
        while not self._stop.is_set():
            try:
                self.samples.append(n.nvmlDeviceGetClockInfo(self._h, n.NVML_CLOCK_SM))
                mask = n.nvmlDeviceGetCurrentClocksEventReasons(self._h)
                for bit, name in self.REASONS.items():
                    if mask & bit and bit != 0x1:
                        self.reasons.add(name)
            except Exception:
                pass
            self._stop.wait(self.period)

    def __enter__(self):
        if self._h is not None:
            self._t = threading.Thread(target=self._run, daemon=True)
            self._t.start()
        return self

    def __exit__(self, *exc):
        self._stop.set()
        if self._h is not None:
            self._t.join()

    def energy_mj(self):
        """Board energy counter (mJ since driver load; NVML), None if unavailable."""
        try:
            return self._nvml.nvmlDeviceGetTotalEnergyConsumption(self._h)
        except Exception:
            return None

    def summary(self):
        return {"sm_mhz": statistics.median(self.samples) if self.samples else None,
                "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons), "samples": len(self.samples)}


# ------------------------------------------------------------------------------------------------
# distributed plumbing
# ------------------------------------------------------------------------------------------------
def dist_env():
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return rank, world, local


def workload_description(name):
    obs_cfg = idgsynth.CONFIGS[name]
    short = (" [short-item variant: dt=8 s over 18 h, N=8192 -- not a BASELINE config]" if name == "lofar_short"
             else "")
    return (f"{BASELINE['configs'][CONFIG_NAMES[name]]}{short} | synthetic: {obs_cfg['nr_stations']} stations, "
            f"T={obs_cfg['T']}, C={obs_cfg['C']}, N~={obs_cfg['Ns']}, N={obs_cfg['N']}, K={obs_cfg['K']}, "
            f"T~max={obs_cfg['Tmax']}, A-terms={obs_cfg['aterms']} (slots of {obs_cfg['slot']})")


# ------------------------------------------------------------------------------------------------
# CPU oracle (cpu_baseline / --impl reference)
# ------------------------------------------------------------------------------------------------
def oracle_sample(obs, target_s: float, kind="grid+degrid"):
    """Choose a deterministic sample (first baselines x all timesteps) worth ~target_s of oracle time."""
    probe = obs.subset(nr_baselines=1, nr_timesteps=min(obs.nr_timesteps, 16 * obs.max_timesteps_per_subgrid))
    t = time_oracle_step(probe, kind)[0]
    per_vis = t / max(1, probe.nr_visibilities)
    want_vis = target_s / max(per_vis, 1e-12)
    nt = obs.nr_timesteps
    nb = max(1, min(obs.nr_baselines, int(want_vis // (nt * obs.nr_channels))))
    if nb == 1 and want_vis < nt * obs.nr_channels:
        nt = max(obs.max_timesteps_per_subgrid, int(want_vis // obs.nr_channels))
        nt = min(nt, obs.nr_timesteps)
    return obs.subset(nr_baselines=nb, nr_timesteps=nt)


def time_oracle_step(sample, kind="grid+degrid"):
    import oracle
    vis = idgsynth.make_visibilities(sample)
    aterms = idgsynth.make_aterms(sample)
    taper = idgsynth.make_taper(sample.subgrid_size)
    items, _ = oracle.plan(sample)
    t0 = time.perf_counter()
    if kind == "grid+degrid":
        g = oracle.grid(sample, items, vis, aterms, taper).astype(np.complex64)
    else:   # degrid only (predict): a model grid over the sample's covered window
        g = np.zeros(oracle.grid_shape(sample), dtype=np.complex64)
        g[..., items["y"].min():items["y"].max() + sample.subgrid_size,
          items["x"].min():items["x"].max() + sample.subgrid_size] = 1.0
    t1 = time.perf_counter()
    oracle.degrid(sample, items, g, aterms, taper)
    t2 = time.perf_counter()
    nvis = int(np.sum(items["nr_timesteps"].astype(np.int64) * (items["channel_end"] - items["channel_begin"])))
    return t2 - t0, nvis, t1 - t0, t2 - t1


def cpu_baseline(obs, target_s=15.0, kind="grid+degrid"):
    import oracle
    sample = oracle_sample(obs, target_s, kind)
    dt, nvis, tg, td = time_oracle_step(sample, kind)
    return {"value": nvis / dt / 1e6, "unit": "MVis/s", "cores": oracle.max_threads(), "kind": "oracle",
            "sample": f"{sample.nr_baselines} baselines x {sample.nr_timesteps} timesteps x "
                      f"{sample.nr_channels} channels of '{obs.name}' ({nvis} visibilities), step {kind}: grid "
                      f"{tg:.2f} s + degrid {td:.2f} s, fp64 C + OpenMP"}


def run_reference(args):
    rank, world, _ = dist_env()
    if rank != 0:
        return 0
    import oracle
    obs = idgsynth.make_observation(args.config)
    kind = STEP_KIND[args.config]
    sample = oracle_sample(obs, args.reference_step_s, kind)
    for _ in range(args.warmup):
        time_oracle_step(sample, kind)
    times, nvis = [], 0
    for _ in range(args.steps):
        dt, nvis, _, _ = time_oracle_step(sample, kind)
        times.append(dt)
    total = sum(times)
    value = nvis * args.steps / total / 1e6
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": "MVis/s", "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * total / args.steps,
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic",
            "config": {"workload": workload_description(args.config), "step": kind,
                       "sample_baselines": sample.nr_baselines,
                       "sample_timesteps": sample.nr_timesteps, "parallelism": "host OpenMP"},
            "cpu_baseline": {"value": value, "unit": "MVis/s", "cores": oracle.max_threads(), "kind": "oracle",
                             "sample": f"{sample.nr_baselines} baselines x {sample.nr_timesteps} timesteps x "
                                       f"{sample.nr_channels} channels ({nvis} visibilities) per step"},
            "e2e": {"value": value, "unit": "MVis/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


# ------------------------------------------------------------------------------------------------
# our arm
# ------------------------------------------------------------------------------------------------
# A step per config: SKA-, LOFAR-shaped and tiny sets grid then degrid (the imaging cycle's two kernels,
# P:45-47); the predict sweep (configs[4]) degrids only, from a model grid broadcast by rank 0.
STEP_KIND = {"tiny": "grid+degrid", "lofar": "grid+degrid", "lofar_dde": "grid+degrid", "ska": "grid+degrid",
             "predict": "degrid", "lofar_short": "grid+degrid"}
# e2e: the SKA-shaped set streams from the host as time chunks ("8 time chunks of 1024")
E2E_TIME_CHUNK = {"ska": 1024}
TENSOR_FLOPS_PER_PAIR = 96   # split-f16 contraction: 3 products x 16 real MACs x 2 flops per pair


def tensor_ops_per_pair(variant: str):
    """Tensor-core operations executed per (pixel, visibility) pair by a kernel variant: the f16 forms run
    3 products x 16 real MACs (96 flops); the integer degridders (`degridder_rot16i`) 3 weight classes of
    m16n8k32 u8 x s8 with 2 limbs per operand value along K (3 x 32 MACs: 192 int8 ops); likewise the
    integer 8- / 4-row units (`rot8i`, `roti`) and the integer direct kernel (`degridder_tci`)."""
    if re.match(r"degridder_(rot\d*(s2)?|tc)i<", variant or ""):
        return 192, "3 u8 x s8 weight classes, 2 limbs per value along K"
    return TENSOR_FLOPS_PER_PAIR, "3 split-f16 products"



def sincos_per_pair(variant: str, nc_item: int) -> float:
    """sincos evaluations per (pixel, visibility) pair of a kernel variant (the paper's kernels and the
    direct tensor-core kernels: 1).  gridder_rot2: per (pixel, timestep) the 8 group-0 slot phasors for
    8 J pairs (J = channel groups of 8; E_t is derived from them); degridder_rot / rot8 / rot16: per
    (visibility row 0, pixel) one phasor and one rotation E for 4 / 8 / 16 channel rows (rot16s2: plus the
    phasor of row 8, which starts the second rotation chain)."""
    j = max(1, nc_item // 8)
    if variant.startswith("gridder_rot2"):
        return 1.0 / j
    if variant.startswith("gridder_rot"):
        return (8.0 + (4.0 if j > 1 else 0.0)) / (8.0 * j)
    if variant.startswith("degridder_rot16s2"):
        return 3.0 / 16      # row 0, E and row 8 (the second rotation chain's start)
    if variant.startswith("degridder_rot16"):
        return 2.0 / 16
    if variant.startswith("degridder_rot8"):
        return 2.0 / 8
    if variant.startswith("degridder_rot"):
        return 0.5
    return 1.0


def sincos_fma_roofline(sm_mhz: float) -> float:
    """The paper's sincos+FMA roofline of its formulation (17 FMA + 1 sincos per pair) from the
    B200 unit counts: per SM and clock 128 FP32 FMA lanes (/17 per pair) and 16 MUFU lanes (/2 per sincos),
    148 SMs, 36 paper-ops per pair; TOps/s at `sm_mhz`."""
    return 148 * min(128.0 / 17.0, 16.0 / 2.0) * OPS_PER_PAIR * sm_mhz * 1e6 / 1e12


def register_host(t):
    """Page-lock an existing host tensor in place (cudaHostRegister: no power-of-two rounding of the
    caching host allocator, which would turn a 94 GB buffer into 128 GB).  Returns True on success."""
    import torch
    try:
        return int(torch._C._cudart.cudaHostRegister(t.data_ptr(), t.numel() * t.element_size(), 0)) == 0
    except Exception:
        return False


def unregister_host(t):
    import torch
    try:
        torch._C._cudart.cudaHostUnregister(t.data_ptr())
    except Exception:
        pass


def host_buffer(shape, dtype):
    """A page-locked host tensor (registered in place, else torch's pinned allocator)."""
    import torch
    t = torch.empty(shape, dtype=dtype)
    if register_host(t):
        return t, True
    return torch.empty(shape, dtype=dtype, pin_memory=True), False


def vdot_chunked(a, b, dev, chunk=1 << 27):
    """sum conj(a) b in complex128 on the device, streaming host tensors through in chunks."""
    import torch
    a, b = a.reshape(-1), b.reshape(-1)
    acc = torch.zeros((), dtype=torch.complex128, device=dev)
    for i in range(0, a.numel(), chunk):
        x = a[i:i + chunk].to(dev, non_blocking=True).to(torch.complex128)
        y = b[i:i + chunk].to(dev, non_blocking=True).to(torch.complex128)
        acc += torch.vdot(x, y)
    return complex(acc.item())


def run_ours(args):
    import torch
    import torch.distributed as dist

    import paper_conf_ipps_veenboerpr17_b200 as idg
    from paper_conf_ipps_veenboerpr17_b200 import _build, parallel
    if not os.path.exists(_build.LIB):
        _build.build()

    rank, world, local = dist_env()
    # IDG_BENCH_SHARED_GPU=1 (testing only): every rank on cuda:0 over gloo, to exercise the multi-rank
    # path (sharding, collectives, max-over-ranks timing) on a one-GPU box; NCCL refuses duplicate GPUs.
    shared_gpu = os.environ.get("IDG_BENCH_SHARED_GPU") == "1"
    if shared_gpu:
        local = 0
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        if shared_gpu:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=dev)
    kind = STEP_KIND[args.config]

    over = {"T": args.timesteps} if args.timesteps else {}
    full = idgsynth.make_observation(args.config, **over)
    b0, b1 = parallel.shard_range(full.nr_baselines, rank, world)
    obs = full.subset(nr_baselines=b1 - b0, baseline_begin=b0)
    t0 = time.perf_counter()
    plan = idg.Plan.from_observation(obs)
    plan_s = time.perf_counter() - t0
    st = plan.stats()
    pairs = st["nr_pairs"]
    nvis_rank = st["nr_vis_assigned"]
    vis_shape = (obs.nr_baselines, obs.nr_timesteps, obs.nr_channels, 4)
    vis_bytes = obs.nr_visibilities * 32

    aterms = idgsynth.make_aterms(obs)
    taper = idgsynth.make_taper(obs.subgrid_size)
    uvw_d = torch.from_numpy(obs.uvw).to(dev)
    at_d = torch.from_numpy(aterms).to(dev)
    tp_d = torch.from_numpy(taper).to(dev)
    N = obs.grid_size
    stream = torch.cuda.current_stream(dev)
    sharded = parallel.ShardedIDG(plan)
    if kind == "grid+degrid":
        vis_d = idgsynth.torch_visibilities(obs, dev, seed_offset=11 + b0)
        free, _ = torch.cuda.mem_get_info(dev)
        # the SKA-shaped set (94 GB) does not fit twice: degrid into the input buffer then (timing is
        # value-independent; the next step grids the previous predictions)
        inplace = free < vis_bytes + (16 << 30)
        out_d = vis_d if inplace else torch.empty_like(vis_d)
        grid_d = torch.zeros((4, N, N), dtype=torch.complex64, device=dev)
    else:
        # predict: degrid only; rank 0 holds the model grid (synthetic: values do not affect run time)
        vis_d, inplace = None, False
        out_d = torch.empty(vis_shape, dtype=torch.complex64, device=dev)
        grid_d = idgsynth.torch_grid(obs, dev) if rank == 0 else torch.zeros((4, N, N), dtype=torch.complex64,
                                                                             device=dev)

    # --exchange peer (N > 1): the banded grid -- every rank's gridder adds into the owners' row bands through
    # CUDA-IPC peer memory and every degridder reads them, so no reduce / broadcast runs (parallel.BandedGrid)
    banded = parallel.BandedGrid(plan, dev) if (world > 1 and args.exchange == "peer") else None
    if banded is not None and kind != "grid+degrid":
        banded.load(grid_d if rank == 0 else idgsynth.torch_grid(obs, dev))   # every rank its band of the model

    def step():
        if banded is not None:
            if kind == "grid+degrid":
                banded.sync()                                            # no peer still reads the bands
                banded.band.zero_()
                banded.sync()                                            # every band zeroed before any add
                banded.grid(vis_d, uvw_d, at_d, tp_d)                    # adder into the owners' bands
                banded.sync()                                            # every rank's adds have landed
            banded.degrid(uvw_d, at_d, tp_d, out_d)                      # splitter reads the owners' bands
            return
        if kind == "grid+degrid":
            grid_d.zero_()
            sharded.grid(vis_d, uvw_d, at_d, tp_d, grid_d, dst=0)        # + NCCL reduce of the uv-grids
        sharded.degrid(grid_d, uvw_d, at_d, tp_d, out_d, src=0)          # NCCL broadcast of the model grid

    def barrier():
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize(dev)

    for _ in range(args.warmup):
        step()
    barrier()

    # ---- timed region: device-resident inputs -------------------------------------------------
    idg.profiling_reset()
    idg.profiling_enable(True)
    launches0 = idg.launch_count()
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with ClockSampler(local) as clocks:
        barrier()
        mj0 = clocks.energy_mj()
        ev0.record(stream)
        for _ in range(args.steps):
            step()
        ev1.record(stream)
        barrier()
        mj1 = clocks.energy_mj()
    idg.profiling_enable(False)
    gpu_launches = idg.launch_count() - launches0
    kern = idg.profiling_read()
    if banded is not None:
        banded.sync()                 # no rank still reads a peer's band
        banded.close()
    ms = ev0.elapsed_time(ev1)
    t = torch.tensor([ms], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    ms_max = float(t.item())
    nvis_t = torch.tensor([nvis_rank], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(nvis_t)
    nvis_total = float(nvis_t.item())
    value = nvis_total * args.steps / (ms_max * 1e-3) / 1e6
    md = plan.metadata()
    nc_item = int((md["channel_end"] - md["channel_begin"]).max()) if len(md) else 1
    kernels_in_step = ["gridder", "degridder"] if kind == "grid+degrid" else ["degridder"]
    energy = None
    if mj0 is not None and mj1 is not None and mj1 > mj0:
        joules = (mj1 - mj0) / 1e3
        ops = len(kernels_in_step) * OPS_PER_PAIR * float(pairs) * args.steps
        energy = {"J_per_step": joules / args.steps, "avg_W": joules / (ms * 1e-3),
                  "GOps_per_J": ops / joules / 1e9, "source": "NVML total energy counter, this GPU, timed region"}

    # ---- roofline denominators, measured right after the timed region on an idle GPU (before the host-
    # streamed legs: measured after them, the rho = 17 kernel ran 15-40% slow in some runs, r02y) ----------
    def best(rho, iters, scalar=False):
        return max(idg.rho_benchmark(rho, iters, scalar=scalar)[0] for _ in range(5))
    barrier()
    with ClockSampler(local) as rclocks:
        sincos_per_s = best(0, 4 * args.rho_iterations) / 2.0
        rho17 = best(17, args.rho_iterations) / 1e12
        rho17_scalar = best(17, args.rho_iterations, scalar=True) / 1e12
        rho_sweep = {}
        if not args.no_rho_sweep:
            for r in (0, 1, 2, 4, 8, 12, 16, 17, 24, 32, 64):
                rho_sweep[str(r)] = best(r, args.rho_iterations) / 1e12

    # ---- energy per kernel (Fig. 15: GFlops/W of the gridder and the degridder) -----------
    # separate timed loops of one kernel each, NVML board energy over the loop
    if energy is not None and not args.no_kernel_energy:
        per = {}
        n_e = max(3, min(args.steps, args.energy_launches))
        loops = {"gridder": lambda: idg.grid(plan, vis_d, uvw_d, at_d, tp_d, grid_d),
                 "degridder": lambda: idg.degrid(plan, grid_d, uvw_d, at_d, tp_d, out_d)}
        for name in kernels_in_step:
            barrier()
            if name == "gridder":
                grid_d.zero_()
            e_a, e_b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            barrier()
            mja = clocks.energy_mj()
            e_a.record(stream)
            for _ in range(n_e):
                loops[name]()
            e_b.record(stream)
            barrier()
            mjb = clocks.energy_mj()
            if mja is None or mjb is None or mjb <= mja:
                continue
            J = (mjb - mja) / 1e3 / n_e
            sec = e_a.elapsed_time(e_b) * 1e-3 / n_e
            variant = idg.last_variant(name)
            spp = sincos_per_pair(variant, nc_item)
            tops, tdesc = tensor_ops_per_pair(variant)
            per[name] = {"launches": n_e, "J_per_launch": J, "s_per_launch": sec, "avg_W": J / sec,
                         "variant": variant,
                         "paper_GOps_per_J": OPS_PER_PAIR * pairs / J / 1e9,
                         "executed_tensor_GOps_per_J": tops * pairs / J / 1e9,
                         "executed_sincos_G_per_J": spp * pairs / J / 1e9,
                         "executed": f"per pair: {tops} tensor-core ops ({tdesc}), "
                                     f"{spp:g} sincos (MUFU), phasor rotation + operand split on the ALUs"}
        energy["per_kernel"] = per
        energy["paper_context"] = "GTX 1080: 32 / 23 GFlops/W gridder / degridder (P:306; paper-ops: 17 FMA + sincos)"

    # ---- one full imaging cycle, timed per stage (Fig. 9: "runtime is dominated by the gridder and
    # degridder kernels (more than 93%)"); grid+degrid configs, one GPU
    cycle = None
    if kind == "grid+degrid" and world == 1 and not args.no_imaging_cycle:
        from paper_conf_ipps_veenboerpr17_b200 import imaging
        N = obs.grid_size
        tap_img = torch.ones((N, N), dtype=torch.float32, device=dev)   # the taper function on the image grid
        for _ in range(2):   # warm-up (cuFFT plans), then the timed cycle
            stages = imaging.imaging_cycle(plan, vis_d, uvw_d, at_d, tp_d, tap_img, out_d, stream=stream)
        tot = stages["total_ms"]
        cycle = {"ms": stages, "share": {k: v / tot for k, v in stages.items() if k != "total_ms"},
                 "kernels_share": (stages["grid"] + stages["degrid"]) / tot,
                 "note": "grid / degrid are the fused kernels (subgrid FFT, adder / splitter, A-term and taper "
                         "inside); ifft / fft are cuFFT on the 4 x N^2 complex64 grid; the dirty image stands in "
                         "for the deconvolved model" + ("; residual skipped (predictions written in place)"
                                                        if inplace else ""),
                 "paper_context": "P:258: gridder + degridder > 93% of the cycle on Haswell / Fiji / Pascal"}
        del tap_img

    # ---- the host adder / splitter: grid in host memory ----------------------------------------
    host_adder = None
    if args.host_adder and kind == "grid+degrid" and world == 1:
        host_adder = run_host_adder(args, idg, obs, plan, vis_d, uvw_d, at_d, tp_d, dev, nvis_rank)

    # ---- e2e: host buffers through the public API ------------------------------------------------
    bufs = {"vis": vis_d, "out": out_d}
    del vis_d, out_d
    e2e = None if args.no_e2e else run_e2e(args, idg, parallel, obs, plan, kind, aterms, taper, dev, stream,
                                           world, rank, nvis_total, bufs, grid_d, sharded, barrier, inplace)
    bufs.clear()

    xu_peak = sincos_per_s * OPS_PER_PAIR / 1e12
    per_kernel = {}
    for name in ("gridder", "degridder"):
        k = kern.get(name)
        if not k:
            continue
        avg_ms = k["total_ms"] / k["launches"]
        achieved = OPS_PER_PAIR * pairs / (avg_ms * 1e-3) / 1e12
        variant = idg.last_variant(name)
        spp = sincos_per_pair(variant, nc_item)
        per_kernel[name] = {"launches": k["launches"], "avg_ms": avg_ms, "TOps_s": achieved,
                            "mvis_s": nvis_rank / (avg_ms * 1e-3) / 1e6,
                            "frac_rho17": achieved / rho17, "share_of_step": k["total_ms"] / ms, "variant": variant,
                            "sincos_per_pair": spp, "peak_own_xu_TOps_s": xu_peak / spp,
                            "frac_own_xu_bound": achieved * spp / xu_peak}
    dominant = max(per_kernel, key=lambda n: per_kernel[n]["avg_ms"]) if per_kernel else None
    sm_mhz = clocks.summary()["sm_mhz"] or 1965
    hw = None
    prof_json = os.path.join(ROOT, "profiles", "ncu_summary.json")
    if dominant and os.path.exists(prof_json):
        try:
            hw = json.load(open(prof_json)).get(args.config, {}).get(dominant)
        except Exception:
            hw = None
    peak = sincos_fma_roofline(sm_mhz)
    for k in per_kernel.values():
        k["frac_sincos_fma_roofline"] = k["TOps_s"] / peak
    roofline = None
    if dominant:
        traffic = (hw or {}).get("dram_bytes")
        if traffic and (hw or {}).get("capture_timesteps"):
            # the capture ran the same kernels at a shorter T: DRAM bytes scale with the visibilities
            traffic = traffic * obs.nr_timesteps / hw["capture_timesteps"]
        roofline = {"bound": "alu", "kernel": dominant, "achieved": per_kernel[dominant]["TOps_s"],
                    "peak": peak, "unit": "TOps/s", "frac": per_kernel[dominant]["TOps_s"] / peak,
                    "traffic": traffic,
                    "traffic_source": "dram__bytes_read.sum + dram__bytes_write.sum of the dominant kernel, one ncu "
                                      "--set full capture (profiles/ncu_summary.json), scaled to this T when the "
                                      "capture ran a shorter T",
                    "peak_source": "the paper's sincos+FMA roofline (P:276-290) from B200 unit counts at the timed "
                                   "region's SM clock: 148 SMs x min(128 FMA lanes / 17, 16 MUFU lanes / 2) pairs/clk "
                                   "x 36 paper-ops per pair (P:258); a ceiling for the paper's formulation (17 FMA + "
                                   "1 sincos per pair), which the B200 kernels leave (tensor-core MACs, sincos by "
                                   "rotation): their hardware bound is roofline.hw",
                    "variant": per_kernel[dominant]["variant"],
                    "peak_measured_rho17": rho17, "frac_measured_rho17": per_kernel[dominant]["TOps_s"] / rho17,
                    "peak_measured_rho17_source": "paper's FMA:sincos benchmark at rho=17 (P:276-290), FMAs as packed "
                                                  "FFMA2, measured in this process (best of 3)",
                    "rho17_scalar_ffma": rho17_scalar,
                    "peak_measured_xu": xu_peak,
                    "ops_per_pair": OPS_PER_PAIR, "pairs_per_launch": pairs,
                    "hw": hw, "clocks_during_peak": rclocks.summary()}

    if rank != 0:
        if world > 1:
            dist.destroy_process_group()
        return 0
    cpu = None
    if world == 1 and not args.no_cpu_baseline:
        cpu = cpu_baseline(full, args.cpu_baseline_s, kind)
    line = {
        "metric": METRIC, "value": value, "unit": "MVis/s", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms_max / args.steps, "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
        "config": {"workload": workload_description(args.config) + (f" [T reduced to {args.timesteps}]" if args.timesteps else ""),
                   "step": kind + (" (model grid broadcast from rank 0)" if kind == "degrid" else ""),
                   "visibilities": int(nvis_total),
                   "arithmetic": "fp32 phases + MUFU sincos; pixel x visibility products and the subgrid "
                                 "DFTs on tensor cores as split-f16 (hi*hi + hi*lo + lo*hi) mma with fp32 "
                                 "accumulation; sincos of one channel group / row per pixel, the other channels by "
                                 "exact rotation (uniform channels)",
                   "subgrids_rank0": st["nr_subgrids"], "pairs_rank0": pairs,
                   "items_timesteps": {"mean": float(md["nr_timesteps"].mean()) if len(md) else 0.0,
                                       "median": float(np.median(md["nr_timesteps"])) if len(md) else 0.0,
                                       "hist_bins_of_16": (np.bincount(np.minimum(md["nr_timesteps"], 128) // 16,
                                                                       minlength=9) / max(1, len(md))).round(4).tolist()},
                   "parallelism": f"baseline shards x{world}" + (
                       "" if world == 1 else " + banded grid, adder / splitter into the owners' bands over peer "
                       "memory (no collective; e2e: NCCL)" if banded is not None else " + NCCL reduce/broadcast"),
                   "l2": f"inputs larger than L2 (visibilities {vis_bytes / 1e9:.1f} GB/step)",
                   "degrid_in_place": inplace},
        "grid_mvis_s": per_kernel.get("gridder", {}).get("mvis_s"),
        "degrid_mvis_s": per_kernel.get("degridder", {}).get("mvis_s"),
        "plan_s": plan_s, "clocks": clocks.summary(), "energy": energy, "e2e": e2e, "gpu_launches": gpu_launches,
        "imaging_cycle": cycle, "host_adder": host_adder,
        "roofline": roofline, "kernels": per_kernel, "rho_sweep_TOps_s": rho_sweep or None,
        "cpu_baseline": cpu,
    }
    print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()
    return 0


def run_host_adder(args, idg, obs, plan, vis_d, uvw_d, at_d, tp_d, dev, nvis):
    """grid + degrid with the grid in HOST memory (idg_grid_host_adder / idg_degrid_host_splitter):
    visibilities from page-locked host memory, subgrids streamed to / from the host and added / split by
    host threads.  Wall-clock per step (the host adds are part of the call), MVis/s."""
    import torch
    try:
        import psutil
        avail = psutil.virtual_memory().available
    except Exception:
        avail = None
    vis_bytes = vis_d.numel() * 8
    grid_bytes = 4 * obs.grid_size * obs.grid_size * 8
    if avail is not None and 2 * vis_bytes + grid_bytes > 0.6 * avail:
        return {"value": None, "skipped": "host memory"}
    vis_h, r1 = host_buffer(tuple(vis_d.shape), torch.complex64)
    out_h, r2 = host_buffer(tuple(vis_d.shape), torch.complex64)
    vis_h.copy_(vis_d)
    grid_h = torch.zeros((4, obs.grid_size, obs.grid_size), dtype=torch.complex64)
    ws = idg.adder_workspace(plan, dev, buffers=8)
    times = []
    for k in range(1 + max(1, args.host_adder_steps)):
        torch.cuda.synchronize(dev)
        t0 = time.perf_counter()
        grid_h.zero_()
        idg.grid_host_adder(plan, vis_h, uvw_d, at_d, tp_d, grid_h, ws)
        idg.degrid_host_splitter(plan, grid_h, uvw_d, at_d, tp_d, out_h, ws)
        torch.cuda.synchronize(dev)
        if k > 0:
            times.append(time.perf_counter() - t0)
    res = {"value": nvis / statistics.median(times) / 1e6, "unit": "MVis/s", "steps": len(times),
           "s_per_step": statistics.median(times), "host_threads": int(os.environ.get("IDG_HOST_THREADS", "0")) or
           min(32, os.cpu_count() or 1),
           "subgrid_bytes_per_step": int(2 * plan.nr_subgrids * 4 * obs.subgrid_size ** 2 * 8),
           "api": "idg_grid_host_adder + idg_degrid_host_splitter (grid in host memory; wall clock per step)"}
    for t, r in ((vis_h, r1), (out_h, r2)):
        if r:
            unregister_host(t)
    del vis_h, out_h, grid_h, ws
    torch.cuda.empty_cache()
    return res


def run_e2e(args, idg, parallel, obs, plan, kind, aterms, taper, dev, stream, world, rank, nvis_total, bufs,
            grid_d, sharded, barrier, inplace):
    """The metric end to end through the public host-streamed calls (idg_grid_host / idg_degrid_host, the
    paper's triple-buffered work groups): every step uploads its inputs (visibilities, uvw,
    A-terms; the model grid for predict) from page-locked host memory and downloads the predictions.
    The SKA-shaped set streams as time chunks of 1024 (one plan per chunk)."""
    import torch
    import torch.distributed as dist
    vis_d, out_d = bufs["vis"], bufs["out"]
    try:
        import psutil
        host_avail = psutil.virtual_memory().available
    except Exception:
        host_avail = None
    T = obs.nr_timesteps
    chunk_T = min(T, E2E_TIME_CHUNK.get(args.config, T))
    nchunks = (T + chunk_T - 1) // chunk_T
    nbl, C = obs.nr_baselines, obs.nr_channels
    chunk_bytes = nbl * chunk_T * C * 32
    vis_bytes = nbl * T * C * 32
    n_in = 1 if kind == "grid+degrid" else 0
    local_world = int(os.environ.get("LOCAL_WORLD_SIZE", world))
    # host memory of ALL local ranks: inputs + outputs (full arrays; the two in-flight steps download into
    # the same host arrays), else 2 rotating chunk buffers per direction
    need_full = local_world * (n_in + 1) * vis_bytes
    need_rot = local_world * (n_in + 1) * 2 * chunk_bytes
    # 0: full host arrays, 1: rotating chunk buffers, 2: skip -- agreed over the ranks (the most conservative
    # choice), since the collectives below must be entered by every rank alike
    mode = 0
    if host_avail is not None and need_full > 0.7 * host_avail:
        mode = 2 if (nchunks == 1 or need_rot > 0.7 * host_avail) else 1
    if world > 1:
        tm = torch.tensor([mode], dtype=torch.int64, device=dev)
        dist.all_reduce(tm, op=dist.ReduceOp.MAX)
        mode = int(tm.item())
    if mode == 2:
        return {"value": None, "unit": "MVis/s", "skipped": f"page-locked host buffers ({need_full / 1e9:.0f} GB for "
                f"{local_world} local ranks) do not fit the host "
                f"({(host_avail or 0) / 1e9:.0f} GB available on this rank)"}
    rotating = mode == 1
    t_plan = time.perf_counter()
    if nchunks == 1:
        cobs, cplans = [obs], [plan]
    else:
        cobs = [obs.select(np.arange(nbl), chunk_T, k * chunk_T) for k in range(nchunks)]
        cplans = [idg.Plan.from_observation(o) for o in cobs]
    plan_s = time.perf_counter() - t_plan
    # A-term slots of every chunk (slot boundaries are cut to the chunk window)
    first_slot = [int(np.searchsorted(obs.aterm_offsets, k * chunk_T, side="right")) - 1 for k in range(nchunks)]
    # union of the covered grid rows of all chunk plans (the band the collectives move)
    rows = None
    if world > 1:
        ys = np.concatenate([p.metadata()["y"] for p in cplans])
        rows = parallel.union_rows(parallel.coverage_rows(ys, obs.subgrid_size, obs.grid_size), device=dev)

    # host buffers: [chunk][nbl][chunk_T][C][4] (chunk-major), or 2 rotating chunk buffers per direction
    nbuf = 2 if rotating else nchunks
    regs = []
    def alloc(n):
        t, reg = host_buffer((n, nbl, chunk_T, C, 4), torch.complex64)
        if reg:
            regs.append(t)
        return t
    in_h = alloc(nbuf) if n_in else None
    out_h = alloc(nbuf)
    uvw_h, reg = host_buffer((nchunks, nbl, chunk_T, 3), torch.float32)
    if reg:
        regs.append(uvw_h)
    for k in range(nchunks):
        uvw_h[k].copy_(torch.from_numpy(cobs[k].uvw))
    at_h = torch.from_numpy(aterms).pin_memory()
    model_h = grid_d.cpu().pin_memory() if kind == "degrid" else None
    chk_ref = None
    if kind == "grid+degrid":
        for k in range(nbuf):
            in_h[k].copy_(vis_d[:, k * chunk_T:(k + 1) * chunk_T])
    elif nchunks == 1:
        chk_ref = None   # compared after the loop against the device path's predictions (same plan)
    if kind == "degrid" and nchunks == 1:
        nb_chk = min(64, nbl)
        chk_ref = out_d[:nb_chk].cpu()
    del vis_d, out_d
    bufs.clear()                 # the device-resident arrays are freed here (the caller holds no reference)
    torch.cuda.empty_cache()
    # one workspace, grid, uvw and A-term buffer per stream: a workspace serves one in-flight call.  Steps
    # rotate over NS streams: a host-streamed call starts its uploads after the work queued before it on its
    # stream (the caller's ordering), so with NS streams step k+1's uploads wait only for step k+1-NS.
    NS = 3
    wss = [idg.workspace(cplans[0], dev, max_buffers=32) for _ in range(NS)]
    streams = [stream] + [torch.cuda.Stream(dev) for _ in range(NS - 1)]
    grids = [grid_d] + [torch.zeros_like(grid_d) for _ in range(NS - 1)]
    uvws = [torch.empty((nchunks, nbl, chunk_T, 3), dtype=torch.float32, device=dev) for _ in range(NS)]
    ats = [torch.empty_like(torch.from_numpy(aterms), device=dev) for _ in range(NS)]
    tp_d = torch.from_numpy(taper).to(dev)

    def e2e_step(k):
        j = k % NS
        s_k, g_k, u_k, a_k, w_k, o_k = streams[j], grids[j], uvws[j], ats[j], wss[j], out_h
        with torch.cuda.stream(s_k):
            u_k.copy_(uvw_h, non_blocking=True)
            a_k.copy_(at_h, non_blocking=True)
            if kind == "grid+degrid":
                g_k.zero_()
                for c in range(nchunks):
                    sl = slice(first_slot[c], first_slot[c] + cobs[c].nr_aterm_slots)
                    idg.grid_host(cplans[c], in_h[c % nbuf], u_k[c], a_k[sl], tp_d, g_k, w_k, stream=s_k)
                parallel.reduce_grid(g_k, dst=0, rows=rows)
            elif rank == 0:
                g_k.copy_(model_h, non_blocking=True)
            parallel.broadcast_grid(g_k, src=0, rows=rows)
            for c in range(nchunks):
                sl = slice(first_slot[c], first_slot[c] + cobs[c].nr_aterm_slots)
                idg.degrid_host(cplans[c], g_k, u_k[c], a_k[sl], tp_d, o_k[c % nbuf], w_k, stream=s_k)

    for k in range(NS):
        e2e_step(k)
    barrier()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ksteps = max(1, min(args.steps, args.e2e_steps))
    e0.record(stream)
    for s_ in streams[1:]:
        s_.wait_event(e0)
    for k in range(ksteps):
        e2e_step(k)
    for s_ in streams[1:]:
        last = torch.cuda.Event()
        last.record(s_)
        stream.wait_event(last)
    e1.record(stream)
    barrier()
    te = torch.tensor([e0.elapsed_time(e1)], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(te, op=dist.ReduceOp.MAX)
    check = None
    out_last = out_h
    if kind == "grid+degrid" and not rotating:
        # whole-data check: degrid = grid^H, so <vis, degrid(grid(vis))> = ||grid(vis)||^2 (adjoint identity;
        # with N ranks the left side sums over the shards and the grid is the reduced + broadcast one)
        lhs = vdot_chunked(in_h, out_last, dev)
        if world > 1:
            t2 = torch.tensor([lhs.real, lhs.imag], dtype=torch.float64, device=dev)
            dist.all_reduce(t2)
            lhs = complex(float(t2[0]), float(t2[1]))
        g = grids[(ksteps - 1) % NS]
        rhs = float(torch.linalg.vector_norm(g.view(torch.float32).to(torch.float64)) ** 2)
        check = {"adjoint_identity_rel_err": abs(lhs - rhs) / abs(rhs)}
    elif chk_ref is not None:
        got = out_last[0, :chk_ref.shape[0]]
        check = {"rel_rms_vs_device_path": float(torch.linalg.vector_norm(got - chk_ref) /
                                                 torch.linalg.vector_norm(chk_ref))}
    h2d = (n_in * nbl * T * C * 32 + uvw_h.numel() * 4 + at_h.numel() * 8 +
           (model_h.numel() * 8 if model_h is not None and rank == 0 else 0))
    res = {"value": nvis_total * ksteps / (float(te.item()) * 1e-3) / 1e6, "unit": "MVis/s",
           "h2d_bytes_per_step": int(h2d), "d2h_bytes_per_step": int(nbl * T * C * 32), "steps": ksteps,
           "time_chunks": nchunks, "chunk_timesteps": chunk_T, "chunk_plans_s": plan_s,
           "host_buffers": ("2 rotating chunk buffers per direction (host memory); every chunk still crosses "
                            "PCIe each step") if rotating else "full page-locked host arrays",
           "check": check,
           "api": "idg_grid_host + idg_degrid_host (host-streamed work groups through <= 32 staging buffers "
                  "per direction; independent steps rotate over 3 streams so the uploads of step k+1 overlap the "
                  "degridding and downloads of step k)"}
    for t in regs:
        unregister_host(t)
    return res


def main():
    ap = argparse.ArgumentParser(description=__doc__, formatter_class=argparse.RawDescriptionHelpFormatter)
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="ska", choices=sorted(CONFIG_NAMES),
                    help="default: the SKA-low-shaped set on an 8192^2 grid (configs[3], the north star's target)")
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--e2e-steps", type=int, default=10)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-baseline-s", type=float, default=15.0)
    ap.add_argument("--reference-step-s", type=float, default=5.0)
    ap.add_argument("--rho-iterations", type=int, default=16384)
    ap.add_argument("--no-rho-sweep", action="store_true")
    ap.add_argument("--no-kernel-energy", action="store_true")
    ap.add_argument("--no-imaging-cycle", action="store_true")
    ap.add_argument("--exchange", default="nccl", choices=["nccl", "peer"],
                    help="N > 1: NCCL reduce / broadcast of the covered grid band (default), or the banded grid "
                         "with the exchange fused into the kernels (peer memory)")
    ap.add_argument("--host-adder", action="store_true",
                    help="also time grid + degrid with the grid in host memory (host adder / splitter, P:226)")
    ap.add_argument("--host-adder-steps", type=int, default=3)
    ap.add_argument("--energy-launches", type=int, default=5)
    ap.add_argument("--timesteps", type=int, default=0,
                    help="tuning only: override the config's T (the line then names the reduced workload)")
    args = ap.parse_args()
    if args.warmup < 3:
        log("[bench] warmup < 3 violates the timing rules; using 3")
        args.warmup = 3
    return run_reference(args) if args.impl == "reference" else run_ours(args)


if __name__ == "__main__":
    sys.exit(main())
