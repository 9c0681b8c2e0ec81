"""Banded grid: the multi-GPU exchange fused into the kernels (include/idg.h, idg_grid_bands /
idg_degrid_bands; paper_conf_ipps_veenboerpr17_b200.parallel.BandedGrid).

* One process, several bands in separate allocations: every kernel family's adder writes each subgrid
  row into the band that owns it, and the splitter reads it back -- against the fp64 oracle, the
  device-resident call (degridding bit-identical: same kernels, same values read).
* Two processes on one GPU (the gpurun box has one): each grids its baseline shard into BOTH processes'
  bands through CUDA-IPC mappings, the exact code path of N GPUs over NVLink peer memory (only the
  physical link differs), then predicts its shard from the banded model grid.
"""
import os
import socket

import numpy as np
import pytest
import torch

import idgsynth
import oracle
import paper_conf_ipps_veenboerpr17_b200 as idg
from paper_conf_ipps_veenboerpr17_b200 import parallel

TOL = 1e-4
FAMILIES = {"default": (None, None), "tc": ("tc", "tc"), "simt": ("simt", "simt"),
            "umma": ("gridder_umma_rot<*", "")}


def rel_rms(a, b):
    return float(np.linalg.norm(a - b) / max(np.linalg.norm(b), 1e-300))


def _dev(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


@pytest.mark.gpu
@pytest.mark.parametrize("family", list(FAMILIES))
@pytest.mark.parametrize("name,kw,nb", [("small_dde", dict(w_planes=3), 3), ("lofar", dict(T=256, nr_stations=5), 2),
                                        ("ska", dict(T=128, nr_stations=4), 5)])
def test_bands_match_oracle_and_device_grid(name, kw, nb, family, monkeypatch):
    g, d = FAMILIES[family]
    if g:
        monkeypatch.setenv("IDG_GRIDDER_VARIANT", g)
        monkeypatch.setenv("IDG_DEGRIDDER_VARIANT", d)
    obs = idgsynth.make_observation(name, **kw)
    vis = idgsynth.make_visibilities(obs)
    aterms = idgsynth.make_aterms(obs, "random")
    taper = idgsynth.make_taper(obs.subgrid_size, "asymmetric")
    items, _ = oracle.plan(obs)
    plan = idg.Plan.from_observation(obs)
    N, R = obs.grid_size, parallel.band_rows(obs.grid_size, nb)
    shape = oracle.grid_shape(obs)
    nz = 1 if len(shape) == 3 else shape[0]
    bands = [torch.zeros((nz, 4, R, N), dtype=torch.complex64, device="cuda") for _ in range(nb)]
    ptrs = torch.tensor([b.data_ptr() for b in bands], dtype=torch.int64, device="cuda")
    v_d, uvw, at, tp = _dev(vis), _dev(obs.uvw), _dev(aterms), _dev(taper)
    idg.grid_bands(plan, v_d, uvw, at, tp, ptrs, R)
    idg.grid_bands(plan, v_d, uvw, at, tp, ptrs, R)          # accumulates
    torch.cuda.synchronize()
    got = parallel.join_bands([b.cpu() for b in bands], N).reshape(shape).numpy()
    ref = 2 * oracle.grid(obs, items, vis, aterms, taper)
    err = rel_rms(got, ref)
    print(f"grid_bands[{family}] {name} {kw} x{nb}: rel rms {err:.3e} ({idg.last_variant('gridder')})")
    assert err <= TOL, err
    G = idgsynth.make_grid(obs)
    mb = parallel.split_bands(torch.from_numpy(G).reshape(nz, 4, N, N), nb)
    mb = [b.cuda().contiguous() for b in mb]
    mptrs = torch.tensor([b.data_ptr() for b in mb], dtype=torch.int64, device="cuda")
    out_b = torch.full(vis.shape, complex(7, 7), dtype=torch.complex64, device="cuda")
    idg.degrid_bands(plan, mptrs, R, uvw, at, tp, out_b)
    out_d = torch.empty_like(out_b)
    idg.degrid(plan, _dev(G), uvw, at, tp, out_d)
    torch.cuda.synchronize()
    assert torch.equal(out_b, out_d)                         # the same values read through the bands
    refv = oracle.scatter_visibilities(obs, items, oracle.degrid(obs, items, G, aterms, taper))
    assert rel_rms(out_b.cpu().numpy(), refv) <= TOL


@pytest.mark.gpu
def test_bands_argument_checks():
    obs = idgsynth.make_observation("small_dde")
    plan = idg.Plan.from_observation(obs)
    vis = _dev(idgsynth.make_visibilities(obs))
    uvw, at = _dev(obs.uvw), _dev(idgsynth.make_aterms(obs))
    tp = _dev(idgsynth.make_taper(obs.subgrid_size))
    b = torch.zeros((1, 4, 8, obs.grid_size), dtype=torch.complex64, device="cuda")
    ptrs = torch.tensor([b.data_ptr()], dtype=torch.int64, device="cuda")
    with pytest.raises(ValueError):                          # 1 band of 8 rows cannot cover N rows
        idg.grid_bands(plan, vis, uvw, at, tp, ptrs, 8)
    with pytest.raises(TypeError):
        idg.grid_bands(plan, vis, uvw, at, tp, ptrs.cpu(), obs.grid_size)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, out_dir, name, kw):
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    obs = idgsynth.make_observation(name, **kw)
    vis = idgsynth.make_visibilities(obs)
    aterms = idgsynth.make_aterms(obs, "random")
    taper = idgsynth.make_taper(obs.subgrid_size, "asymmetric")
    b0, b1 = parallel.shard_range(obs.nr_baselines, rank, world)
    sub = obs.subset(nr_baselines=b1 - b0, baseline_begin=b0)
    plan = idg.Plan.from_observation(sub)
    dev = torch.device("cuda", 0)
    bg = parallel.BandedGrid(plan, dev)
    v_d, uvw, at, tp = _dev(vis[b0:b1]), _dev(sub.uvw), _dev(aterms), _dev(taper)
    bg.sync()                                                # every band zeroed before anyone adds
    bg.grid(v_d, uvw, at, tp)
    bg.sync()                                                # every rank's adds have landed
    full = bg.gather(dst=0)
    if rank == 0:
        np.save(os.path.join(out_dir, "grid.npy"), full.cpu().numpy())
    bg.load(torch.from_numpy(idgsynth.make_grid(obs)).to(dev))
    bg.sync()
    out = torch.empty((sub.nr_baselines, sub.nr_timesteps, sub.nr_channels, 4), dtype=torch.complex64, device=dev)
    bg.degrid(uvw, at, tp, out)
    bg.sync()                                                # no band is released while a peer reads it
    np.save(os.path.join(out_dir, f"vis{rank}.npy"), out.cpu().numpy())
    bg.close()
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.gpu
@pytest.mark.parametrize("name,kw,world", [("lofar", dict(T=256, nr_stations=6), 2),
                                           ("small_dde", dict(w_planes=3), 3)])
def test_two_processes_share_the_banded_grid_through_ipc(name, kw, world, tmp_path):
    import torch.multiprocessing as mp
    mp.spawn(_worker, args=(world, _free_port(), str(tmp_path), name, kw), nprocs=world, join=True)
    obs = idgsynth.make_observation(name, **kw)
    vis = idgsynth.make_visibilities(obs)
    aterms = idgsynth.make_aterms(obs, "random")
    taper = idgsynth.make_taper(obs.subgrid_size, "asymmetric")
    items, _ = oracle.plan(obs)
    ref = oracle.grid(obs, items, vis, aterms, taper)
    got = np.load(tmp_path / "grid.npy").reshape(ref.shape)
    err = rel_rms(got, ref)
    print(f"banded grid over {world} processes {name}: rel rms {err:.3e}")
    assert err <= TOL, err
    refv = oracle.scatter_visibilities(obs, items, oracle.degrid(obs, items, idgsynth.make_grid(obs), aterms, taper))
    gotv = np.concatenate([np.load(tmp_path / f"vis{r}.npy") for r in range(world)], axis=0)
    assert rel_rms(gotv, refv) <= TOL
