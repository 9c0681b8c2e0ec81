#!/usr/bin/env python
"""Time every compiled launch-shape variant of the gridder and degridder on a config (GPU only).

  python scripts/tune.py [--config lofar] [--reps 3] [--T 8192] [--stations 44]

Prints one JSON line per variant: {"kernel", "variant", "ms", "mvis_s", "TOps_s"}.  The variant is
selected through IDG_GRIDDER_VARIANT / IDG_DEGRIDDER_VARIANT (see include/idg.h).
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import idgsynth  # noqa: E402
import paper_conf_ipps_veenboerpr17_b200 as idg  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="lofar")
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--T", type=int, default=None)
    ap.add_argument("--stations", type=int, default=None)
    ap.add_argument("--only", default=None, help="substring filter on variant names")
    args = ap.parse_args()
    kw = {}
    if args.T:
        kw["T"] = args.T
    if args.stations:
        kw["nr_stations"] = args.stations
    obs = idgsynth.make_observation(args.config, **kw)
    plan = idg.Plan.from_observation(obs)
    st = plan.stats()
    dev = torch.device("cuda")
    uvw = torch.from_numpy(obs.uvw).to(dev)
    at = torch.from_numpy(idgsynth.make_aterms(obs)).to(dev)
    tp = torch.from_numpy(idgsynth.make_taper(obs.subgrid_size)).to(dev)
    vis = idgsynth.torch_visibilities(obs, dev)
    out = torch.empty_like(vis)
    g = torch.zeros((4, obs.grid_size, obs.grid_size), dtype=torch.complex64, device=dev)
    ns = obs.subgrid_size
    print(json.dumps({"config": args.config, **kw, "stats": st}), flush=True)
    for kernel, env in (("gridder", "IDG_GRIDDER_VARIANT"), ("degridder", "IDG_DEGRIDDER_VARIANT")):
        for name in idg.idg.kernel_variants(kernel):
            if f"<{ns}," not in name:
                continue
            if args.only and args.only not in name:
                continue
            os.environ[env] = name
            fn = (lambda: idg.grid(plan, vis, uvw, at, tp, g)) if kernel == "gridder" else \
                (lambda: idg.degrid(plan, g, uvw, at, tp, out))
            try:
                fn()
                torch.cuda.synchronize()
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record()
                for _ in range(args.reps):
                    fn()
                e1.record()
                torch.cuda.synchronize()
                ms = e0.elapsed_time(e1) / args.reps
                rec = {"kernel": kernel, "variant": name, "ms": ms,
                       "mvis_s": st["nr_vis_assigned"] / ms / 1e3, "TOps_s": 36 * st["nr_pairs"] / ms / 1e9}
            except Exception as e:  # a variant that cannot launch (e.g. V does not divide the channels)
                rec = {"kernel": kernel, "variant": name, "error": str(e)[:200]}
            print(json.dumps(rec), flush=True)
        os.environ.pop(env, None)
    for r in (1, 2, 4, 8, 16, 17, 24, 32, 64):
        ops, sec = idg.rho_benchmark(r, 2048)
        print(json.dumps({"rho": r, "TOps_s": ops / 1e12, "s": sec}), flush=True)


if __name__ == "__main__":
    main()
