"""Multi-rank path on CPU (gloo, world size 2): sharding and the two collectives compose to the
single-process result.  On CPU the per-rank gridding/degridding is the fp64 oracle standing in for the
GPU kernels (test infrastructure); the sharding, the per-rank plans and the reduce/broadcast are the
product's (paper_conf_ipps_veenboerpr17_b200.parallel)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import idgsynth
import oracle
import paper_conf_ipps_veenboerpr17_b200 as idg
from paper_conf_ipps_veenboerpr17_b200 import parallel


@pytest.mark.parametrize("world", [2, 3, 4])
def test_rank_plans_are_slices_of_the_global_plan(world):
    obs = idgsynth.make_observation("lofar", T=1024, nr_stations=10)
    glob = idg.Plan.from_observation(obs).metadata()
    parts = []
    for r in range(world):
        b0, b1 = parallel.shard_range(obs.nr_baselines, r, world)
        sub = obs.subset(nr_baselines=b1 - b0, baseline_begin=b0)
        md = idg.Plan.from_observation(sub).metadata()
        md["baseline"] += b0
        parts.append(md)
    np.testing.assert_array_equal(np.concatenate(parts), glob)


def test_weighted_shards_cover_everything():
    w = np.arange(1, 101, dtype=float)
    ranges = [parallel.shard_range(100, r, 4, w) for r in range(4)]
    assert ranges[0][0] == 0 and ranges[-1][1] == 100
    assert all(ranges[i][1] == ranges[i + 1][0] for i in range(3))
    loads = [w[a:b].sum() for a, b in ranges]
    assert max(loads) / min(loads) < 1.3


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, result_dir):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    obs = idgsynth.make_observation("small_dde")
    vis = idgsynth.make_visibilities(obs)
    aterms = idgsynth.make_aterms(obs)
    taper = idgsynth.make_taper(obs.subgrid_size)
    b0, b1 = parallel.shard_range(obs.nr_baselines, rank, world)
    sub = obs.subset(nr_baselines=b1 - b0, baseline_begin=b0)
    items, _ = oracle.plan(sub)
    # gridding: per-rank grid, then the product's reduce (full grid, and the covered row band only)
    g = torch.from_numpy(oracle.grid(sub, items, vis[b0:b1], aterms, taper).astype(np.complex64))
    g_band = g.clone()
    rows = parallel.union_rows(parallel.coverage_rows(items["y"], obs.subgrid_size, obs.grid_size))
    parallel.reduce_grid(g, dst=0)
    parallel.reduce_grid(g_band, dst=0, rows=rows)
    # degridding: the model grid exists on rank 0 only, the product's broadcast ships it
    model = torch.from_numpy(idgsynth.make_grid(obs)) if rank == 0 else torch.zeros(
        (4, obs.grid_size, obs.grid_size), dtype=torch.complex64)
    model_band = model.clone() if rank == 0 else torch.full_like(model, float("nan"))
    parallel.broadcast_grid(model, src=0)
    parallel.broadcast_grid(model_band, src=0, rows=rows)   # rows outside the band stay NaN off rank 0
    v = oracle.scatter_visibilities(sub, items, oracle.degrid(sub, items, model.numpy(), aterms, taper))
    v_band = oracle.scatter_visibilities(sub, items, oracle.degrid(sub, items, model_band.numpy(), aterms, taper))
    np.save(os.path.join(result_dir, f"vis{rank}.npy"), v)
    np.save(os.path.join(result_dir, f"vis_band{rank}.npy"), v_band)
    if rank == 0:
        np.save(os.path.join(result_dir, "grid.npy"), g.numpy())
        np.save(os.path.join(result_dir, "grid_band.npy"), g_band.numpy())
        np.save(os.path.join(result_dir, "rows.npy"), np.array(rows))
    dist.destroy_process_group()


def test_gloo_two_ranks_compose_to_single_process(tmp_path):
    world = 2
    mp.spawn(_worker, args=(world, _free_port(), str(tmp_path)), nprocs=world, join=True)
    obs = idgsynth.make_observation("small_dde")
    vis = idgsynth.make_visibilities(obs)
    aterms = idgsynth.make_aterms(obs)
    taper = idgsynth.make_taper(obs.subgrid_size)
    items, _ = oracle.plan(obs)
    ref = oracle.grid(obs, items, vis, aterms, taper)
    got = np.load(tmp_path / "grid.npy")
    assert np.linalg.norm(got - ref) / np.linalg.norm(ref) < 1e-6        # fp32 storage of partial grids
    ref_v = oracle.scatter_visibilities(obs, items, oracle.degrid(obs, items, idgsynth.make_grid(obs), aterms, taper))
    got_v = np.concatenate([np.load(tmp_path / f"vis{r}.npy") for r in range(world)], axis=0)
    np.testing.assert_allclose(got_v, ref_v, rtol=0, atol=1e-9 * np.abs(ref_v).max())
    # the row-band collectives give the identical result with a strictly smaller message
    y0, y1 = np.load(tmp_path / "rows.npy")
    assert 0 <= y0 < y1 <= obs.grid_size and (y1 - y0) < obs.grid_size
    np.testing.assert_array_equal(np.load(tmp_path / "grid_band.npy"), got)
    for r in range(world):
        np.testing.assert_array_equal(np.load(tmp_path / f"vis_band{r}.npy"), np.load(tmp_path / f"vis{r}.npy"))


def test_coverage_rows():
    assert parallel.coverage_rows(np.array([5, 40, 17]), 24, 128) == (5, 64)
    assert parallel.coverage_rows(np.array([], dtype=np.int32), 24, 128) == (128, 0)
    assert parallel.union_rows((5, 64)) == (5, 64)            # single process: identity
    g = torch.arange(2 * 4 * 6 * 6, dtype=torch.float32).reshape(2, 4, 6, 6).to(torch.complex64)
    slabs = parallel._slabs(g, (1, 3))
    assert len(slabs) == 8 and all(s.is_contiguous() and s.shape == (2, 6, 2) for s in slabs)
    assert parallel._slabs(g, (3, 3)) == []


@pytest.mark.parametrize("N,world", [(128, 2), (128, 3), (100, 7), (8, 8)])
def test_band_helpers(N, world):
    R = parallel.band_rows(N, world)
    assert R * world >= N and (R - 1) * world < N
    ranges = [parallel.band_range(N, world, r) for r in range(world)]
    assert ranges[0][0] == 0 and ranges[-1][1] == N
    assert all(ranges[r][1] == ranges[r + 1][0] for r in range(world - 1))
    g = np.random.default_rng(N + world).standard_normal((2, 4, N, N)).astype(np.float32)
    bands = parallel.split_bands(g, world)
    assert all(b.shape == (2, 4, R, N) for b in bands)
    np.testing.assert_array_equal(parallel.join_bands(bands, N), g)
    # torch tensors take the same path
    gt = torch.from_numpy(g)
    assert torch.equal(parallel.join_bands(parallel.split_bands(gt, world), N), gt)


@pytest.mark.parametrize("world", [2, 3])
def test_banded_adder_composes_to_the_global_grid(world):
    """The fused cross-rank adder (idg_grid_bands): every rank adds each row of its subgrids into the band
    that owns the row.  Emulated with the oracle's per-shard grids: band r = sum over ranks of rows
    [r R, (r+1) R) of their grids; joined, the bands are the grid of the whole observation."""
    obs = idgsynth.make_observation("small_dde")
    vis = idgsynth.make_visibilities(obs)
    aterms = idgsynth.make_aterms(obs)
    taper = idgsynth.make_taper(obs.subgrid_size)
    N = obs.grid_size
    bands = None
    for r in range(world):
        b0, b1 = parallel.shard_range(obs.nr_baselines, r, world)
        sub = obs.subset(nr_baselines=b1 - b0, baseline_begin=b0)
        items, _ = oracle.plan(sub)
        parts = parallel.split_bands(oracle.grid(sub, items, vis[b0:b1], aterms, taper), world)
        bands = parts if bands is None else [a + b for a, b in zip(bands, parts)]
    items, _ = oracle.plan(obs)
    ref = oracle.grid(obs, items, vis, aterms, taper)
    got = parallel.join_bands(bands, N)
    assert np.linalg.norm(got - ref) <= 1e-12 * np.linalg.norm(ref)
