"""Diagnose the host-streamed e2e pipeline on the LOFAR config: per-phase throughput (GPU only)."""
import sys, os, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import idgsynth
import paper_conf_ipps_veenboerpr17_b200 as idg

obs = idgsynth.make_observation("lofar")
plan = idg.Plan.from_observation(obs)
dev = torch.device("cuda")
uvw = torch.from_numpy(obs.uvw).to(dev)
at = torch.from_numpy(idgsynth.make_aterms(obs)).to(dev)
tp = torch.from_numpy(idgsynth.make_taper(obs.subgrid_size)).to(dev)
vd = idgsynth.torch_visibilities(obs, dev)
vh = torch.empty(vd.shape, dtype=vd.dtype, pin_memory=True); vh.copy_(vd)
oh = torch.empty_like(vh, pin_memory=True)
del vd
g = torch.zeros((4, obs.grid_size, obs.grid_size), dtype=torch.complex64, device=dev)
for full in (False, True):
    ws = idg.workspace(plan, dev, full=full)
    def run(f, n=8):
        f(); torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(n): f()
        e1.record(); torch.cuda.synchronize()
        return e0.elapsed_time(e1) / n
    tg = run(lambda: idg.grid_host(plan, vh, uvw, at, tp, g, ws))
    td = run(lambda: idg.degrid_host(plan, g, uvw, at, tp, oh, ws))
    tb = run(lambda: (idg.grid_host(plan, vh, uvw, at, tp, g, ws), idg.degrid_host(plan, g, uvw, at, tp, oh, ws)))
    print(f"workspace {'full' if full else 'min '} {ws.numel()/1e9:.2f} GB: grid_host {tg:.1f} ms, degrid_host {td:.1f} ms, "
          f"both {tb:.1f} ms/step -> {obs.nr_visibilities/tb/1e3:.0f} MVis/s", flush=True)
    del ws
