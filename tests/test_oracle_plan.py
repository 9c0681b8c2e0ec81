"""The oracle's execution plan satisfies the plan properties of P:137-145 (no GPU)."""
import dataclasses

import numpy as np
import pytest

import idgsynth
import oracle
from plan_checks import check_plan


@pytest.mark.parametrize("name,kw", [("tiny", {}), ("small_dde", {}),
                                     ("lofar", dict(T=1024, nr_stations=12)),
                                     ("ska", dict(T=512, nr_stations=10, N=2048, Ns=24, K=7))])
def test_oracle_plan_properties(name, kw):
    obs = idgsynth.make_observation(name, **kw)
    items, dropped = oracle.plan(obs)
    check_plan(obs, items, dropped)
    assert dropped == 0            # L is chosen so that nothing falls off the grid (DESIGN.md recipe)


def test_plan_channel_blocks():
    obs = idgsynth.make_observation("small_dde", C=7, C_block=3)
    items, dropped = oracle.plan(obs)
    check_plan(obs, items, dropped)
    blocks = sorted(set(zip(items["channel_begin"].tolist(), items["channel_end"].tolist())))
    assert blocks == [(0, 3), (3, 6), (6, 7)]


def test_plan_drops_are_counted():
    obs = idgsynth.make_observation("small_dde")
    # image size x6: long baselines fall off the grid (R-12) and fast tracks no longer fit (R-13)
    big = dataclasses.replace(obs, image_size=obs.image_size * 6)
    items, dropped = oracle.plan(big)
    check_plan(big, items, dropped)
    assert dropped > 0 and len(items) > 0
    # a single timestep whose channel spread alone exceeds N~ - K is dropped (R-13)
    wide = dataclasses.replace(obs, frequencies=np.linspace(100e6, 200e6, 4))
    items, dropped = oracle.plan(wide)
    check_plan(wide, items, dropped)
    assert dropped > 0


def test_plan_respects_tmax_and_slots():
    obs = idgsynth.make_observation("lofar", T=700, nr_stations=6)
    items, dropped = oracle.plan(obs)
    check_plan(obs, items, dropped)
    assert items["nr_timesteps"].max() == obs.max_timesteps_per_subgrid
    # slot boundaries every 256 steps: items split there even when they would fit
    assert set(items["time_offset"].tolist()) >= {0, 256, 512}


@pytest.mark.parametrize("nz", [2, 5])
def test_plan_w_planes(nz):
    obs = idgsynth.make_observation("small_dde", w_planes=nz)
    items, dropped = oracle.plan(obs)
    check_plan(obs, items, dropped)
    assert len(set(items["z"].tolist())) >= 2


def test_plan_checks_reject_unforced_drops():
    """Mutation test of the checker: dropping one gridable item (and counting its visibilities as
    dropped) must be caught, as must shortening an item (breaks maximality)."""
    obs = idgsynth.make_observation("small_dde")
    items, dropped = oracle.plan(obs)
    victim = items[len(items) // 2]
    nvis = int(victim["nr_timesteps"]) * int(victim["channel_end"] - victim["channel_begin"])
    fewer = np.delete(items, len(items) // 2)
    with pytest.raises(AssertionError, match="dropped but fits"):
        check_plan(obs, fewer, dropped + nvis)
    shorter = items.copy()
    k = int(np.argmax(items["nr_timesteps"]))
    shorter[k]["nr_timesteps"] -= 1
    nc = int(items[k]["channel_end"] - items[k]["channel_begin"])
    with pytest.raises(AssertionError):
        check_plan(obs, shorter, dropped + nc)
