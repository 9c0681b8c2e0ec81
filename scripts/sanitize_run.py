#!/usr/bin/env python
"""One small grid + degrid (device-resident, host-streamed and host adder / splitter) of a config through
one kernel family, for compute-sanitizer (memcheck / racecheck / synccheck):

  compute-sanitizer --tool racecheck python scripts/sanitize_run.py small_dde default
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import idgsynth  # noqa: E402

FAMILIES = {"default": (None, None), "tc": ("tc", "tc"), "simt": ("simt", "simt"),
            "umma": ("gridder_umma_rot<*", "")}


def main():
    name, fam = sys.argv[1], sys.argv[2]
    kw = {}
    if name == "ska_small":
        name, kw = "ska", dict(T=128, nr_stations=3)
    if name == "predict_small":       # 16-channel items at N~ = 32 (the KPT 2 rotation / tcgen05 gridders)
        name, kw = "predict", dict(T=128, nr_stations=3)
    if name == "lofar_small":
        name, kw = "lofar", dict(T=256, nr_stations=4)
    if name == "small_dde8":          # 8 channels: the N~ = 16 rotation gridder (KPT 1) and 8-row degridder
        name, kw = "small_dde", dict(C=8)
    select = None
    if name == "short_items":         # long baselines of lofar_short: the short-item (mean T~ <= 64) degridder
        name, select = "lofar_short", (3, 256, 2048)
    g, d = FAMILIES[fam]
    if g:
        os.environ["IDG_GRIDDER_VARIANT"], os.environ["IDG_DEGRIDDER_VARIANT"] = g, d
    os.environ["IDG_HOST_CHUNK_BYTES"] = "60000"
    import torch
    import paper_conf_ipps_veenboerpr17_b200 as idg
    obs = idgsynth.make_observation(name, **kw)
    if select:
        obs = obs.select(obs.longest_baselines(select[0]), nr_timesteps=select[1], time_begin=select[2])
    vis = idgsynth.make_visibilities(obs)
    aterms = idgsynth.make_aterms(obs, "random")
    taper = idgsynth.make_taper(obs.subgrid_size, "asymmetric")
    plan = idg.Plan.from_observation(obs)
    dev = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
    uvw, at, tp = dev(obs.uvw), dev(aterms), dev(taper)
    shape = (4, obs.grid_size, obs.grid_size) if obs.nr_w_planes == 1 else (obs.nr_w_planes, 4, obs.grid_size, obs.grid_size)
    G = torch.zeros(shape, dtype=torch.complex64, device="cuda")
    idg.grid(plan, dev(vis), uvw, at, tp, G)
    V = torch.empty(vis.shape, dtype=torch.complex64, device="cuda")
    idg.degrid(plan, G, uvw, at, tp, V)
    ws = idg.workspace(plan)
    vh = torch.from_numpy(vis).pin_memory()
    idg.grid_host(plan, vh, uvw, at, tp, G, ws)
    out = torch.empty_like(vh).pin_memory()
    idg.degrid_host(plan, G, uvw, at, tp, out, ws)
    wa = idg.adder_workspace(plan)
    gh = torch.zeros(shape, dtype=torch.complex64)
    idg.grid_host_adder(plan, vh, uvw, at, tp, gh, wa)
    idg.degrid_host_splitter(plan, gh, uvw, at, tp, out, wa)
    # the banded grid (3 bands in separate allocations): adder into / splitter from the owners' bands
    from paper_conf_ipps_veenboerpr17_b200 import parallel
    R = parallel.band_rows(obs.grid_size, 3)
    bands = [torch.zeros(shape[:-2] + (R, obs.grid_size), dtype=torch.complex64, device="cuda") for _ in range(3)]
    ptrs = torch.tensor([b.data_ptr() for b in bands], dtype=torch.int64, device="cuda")
    idg.grid_bands(plan, dev(vis), uvw, at, tp, ptrs, R)
    idg.degrid_bands(plan, ptrs, R, uvw, at, tp, V)
    torch.cuda.synchronize()
    print(f"sanitize_run {name} {fam}: {plan.nr_subgrids} items, gridder {idg.last_variant('gridder')}, "
          f"degridder {idg.last_variant('degridder')}, launches {idg.launch_count()}")


if __name__ == "__main__":
    main()
