#!/usr/bin/env python
"""Time kernel variants in one process (IDG_GRIDDER_VARIANT / IDG_DEGRIDDER_VARIANT are read per launch).

  python scripts/variant_sweep.py --config ska --timesteps 1024 --which degridder \
      --variants 'degridder_rot16<32,W8,minB2,U2,C32>' 'degridder_rot16s2<32,W8,minB2,U2,C32>' ...

Prints one JSON line per variant: ms per launch (median of --reps after --warmup), MVis/s, and the
relative RMS difference of its output against the first variant's (a quick consistency check; parity
proper is tests/test_gpu_parity.py).
"""
import argparse
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import idgsynth  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="ska")
    ap.add_argument("--timesteps", type=int, default=1024)
    ap.add_argument("--which", choices=["gridder", "degridder"], default="degridder")
    ap.add_argument("--variants", nargs="+", required=True)
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=2)
    ap.add_argument("--obs", nargs="*", default=[], help="extra make_observation keywords, e.g. C=8")
    args = ap.parse_args()
    import torch
    import paper_conf_ipps_veenboerpr17_b200 as idg
    extra = {k: int(v) for k, v in (kv.split("=") for kv in args.obs)}
    obs = idgsynth.make_observation(args.config, T=args.timesteps, **extra)
    plan = idg.Plan.from_observation(obs)
    st = plan.stats()
    dev = torch.device("cuda", 0)
    uvw = torch.from_numpy(obs.uvw).to(dev)
    at = torch.from_numpy(idgsynth.make_aterms(obs)).to(dev)
    tp = torch.from_numpy(idgsynth.make_taper(obs.subgrid_size)).to(dev)
    vis = idgsynth.torch_visibilities(obs, dev)
    grid = idgsynth.torch_grid(obs, dev) if args.which == "degridder" else torch.zeros(
        (4, obs.grid_size, obs.grid_size), dtype=torch.complex64, device=dev)
    env = "IDG_DEGRIDDER_VARIANT" if args.which == "degridder" else "IDG_GRIDDER_VARIANT"
    ref = None
    for v in args.variants:
        os.environ[env] = v
        times = []
        for i in range(args.warmup + args.reps):
            if args.which == "gridder":
                grid.zero_()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            if args.which == "degridder":
                idg.degrid(plan, grid, uvw, at, tp, vis)
            else:
                idg.grid(plan, vis, uvw, at, tp, grid)
            e1.record()
            torch.cuda.synchronize()
            if i >= args.warmup:
                times.append(e0.elapsed_time(e1))
        used = idg.last_variant(args.which)
        out = (vis if args.which == "degridder" else grid)
        sample = out.reshape(-1)[: 1 << 24].clone()
        diff = None
        if ref is None:
            ref = sample
        else:
            diff = float(torch.linalg.vector_norm(sample - ref) / torch.linalg.vector_norm(ref))
        ms = statistics.median(times)
        print(json.dumps({"variant": v, "used": used, "ms": ms, "mvis_s": st["nr_vis_assigned"] / ms / 1e3,
                          "rel_diff_vs_first": diff, "config": args.config, "T": args.timesteps}), flush=True)


if __name__ == "__main__":
    main()
