"""C-ABI library (no GPU): it loads, exports every function include/idg.h declares, validates its
arguments, and its host plan builder is bit-exact with the oracle's plan (R-8..R-16)."""
import ctypes
import dataclasses
import os
import re

import numpy as np
import pytest

import idgsynth
import oracle
from plan_checks import check_plan

import paper_conf_ipps_veenboerpr17_b200 as idg
from paper_conf_ipps_veenboerpr17_b200 import idg as binding

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared_functions():
    src = open(os.path.join(ROOT, "include", "idg.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(idg_[a-z0-9_]+)\s*\(", src)))


def test_library_exports_every_declared_symbol():
    lib = idg.lib()
    declared = _declared_functions()
    assert len(declared) >= 15, declared
    for name in declared:
        assert hasattr(lib, name), f"{name} declared in idg.h but not exported"
    assert set(declared) == set(binding.EXPORTED)


def test_library_is_sm100a_only():
    import subprocess
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", binding._LIB_PATH],
                         capture_output=True, text=True).stdout
    assert "sm_100a" in out and "sm_90" not in out and "sm_80" not in out, out


def _plans_equal(obs):
    items_o, dropped_o = oracle.plan(obs)
    plan = idg.Plan.from_observation(obs)
    items_l = plan.metadata()
    st = plan.stats()
    assert st["nr_vis_dropped"] == dropped_o
    assert len(items_l) == len(items_o)
    for f in oracle.ITEM_DTYPE.names:                      # bit-exact integer metadata
        np.testing.assert_array_equal(items_l[f], items_o[f], err_msg=f)
    n2 = obs.subgrid_size ** 2
    nv = items_o["nr_timesteps"].astype(np.int64) * (items_o["channel_end"] - items_o["channel_begin"])
    assert st["nr_vis_assigned"] == int(nv.sum())
    assert st["nr_pairs"] == int(nv.sum()) * n2
    return items_l, st


@pytest.mark.parametrize("name,kw", [("tiny", {}), ("small_dde", {}), ("small_dde", dict(C=7, C_block=3)),
                                     ("lofar", dict(T=2048, nr_stations=16)),
                                     ("ska", dict(T=768, nr_stations=12)),
                                     ("predict", dict(T=256, nr_stations=14)),
                                     ("small_dde", dict(w_planes=4)),
                                     ("lofar_dde", dict(T=1024, nr_stations=12, w_planes=8))])
def test_plan_bit_exact_with_oracle(name, kw):
    obs = idgsynth.make_observation(name, **kw)
    items, st = _plans_equal(obs)
    check_plan(obs, items, st["nr_vis_dropped"])


def test_plan_bit_exact_with_drops():
    obs = idgsynth.make_observation("small_dde")
    big = dataclasses.replace(obs, image_size=obs.image_size * 6)
    items, st = _plans_equal(big)
    assert st["nr_vis_dropped"] > 0
    wide = dataclasses.replace(obs, frequencies=np.linspace(100e6, 200e6, 4))
    _, st = _plans_equal(wide)
    assert st["nr_vis_dropped"] > 0


def test_plan_full_lofar_bit_exact():
    obs = idgsynth.make_observation("lofar")
    items, st = _plans_equal(obs)
    assert st["nr_vis_dropped"] == 0 and st["nr_subgrids"] == 60544


def test_plan_argument_validation():
    obs = idgsynth.make_observation("tiny")
    kw = dict(**obs.plan_params(), nr_stations=obs.nr_stations, uvw=obs.uvw, frequencies=obs.frequencies,
              baselines=obs.baselines, aterm_offsets=obs.aterm_offsets)
    bad = [dict(subgrid_size=20), dict(grid_size=16), dict(image_size=-1.0), dict(kernel_size=16),
           dict(max_timesteps_per_subgrid=0), dict(aterm_offsets=np.array([0, 10], dtype=np.int32)),
           dict(frequencies=-obs.frequencies), dict(baselines=obs.baselines[:, ::-1].copy()),
           dict(nr_w_planes=4, w_step=0.0), dict(nr_w_planes=-1)]
    for b in bad:
        with pytest.raises(idg.IDGError) as e:
            idg.Plan(**{**kw, **b})
        assert e.value.status in (1, 2), b
    assert idg.Plan(**kw).workspace_size() == 0


def test_empty_plan():
    obs = idgsynth.make_observation("tiny")
    obs0 = obs.subset(nr_baselines=0)
    plan = idg.Plan.from_observation(obs0)
    assert plan.nr_subgrids == 0 and plan.stats()["nr_pairs"] == 0


def test_calls_on_a_plan_without_items_need_no_gpu():
    """A plan whose visibilities are all dropped launches nothing: degridding defines them as 0 (R-12,
    R-13) on the host path too, and a NULL host buffer is an argument error, not a crash."""
    obs = idgsynth.make_observation("small_dde")
    plan = idg.Plan.from_observation(dataclasses.replace(obs, image_size=1.4))  # every subgrid falls off
    assert plan.nr_subgrids == 0 and plan.stats()["nr_vis_dropped"] == obs.nr_baselines * obs.nr_timesteps * obs.nr_channels
    lib = idg.lib()
    h = plan._h
    assert lib.idg_degrid_host(h, None, None, None, None, None, None, 0, None) == 1   # IDG_ERR_INVALID_ARG
    vis = np.full((obs.nr_baselines, obs.nr_timesteps, obs.nr_channels, 4), 1 + 1j, dtype=np.complex64)
    assert lib.idg_degrid_host(h, None, None, None, None, vis.ctypes.data, None, 0, None) == 0
    assert not vis.any()
    assert lib.idg_grid_host(h, None, None, None, None, None, None, 0, None) == 0      # nothing to add
    assert lib.idg_grid(h, None, None, None, None, None, None, 0, None) == 0


def test_banded_and_ipc_calls_validate_arguments_without_a_gpu():
    """The banded-grid and IPC entry points reject bad arguments before touching the device."""
    obs = idgsynth.make_observation("small_dde")
    plan = idg.Plan.from_observation(obs)
    lib = idg.lib()
    h = plan._h
    fake = ctypes.c_void_p(0x1000)   # never dereferenced: validation fails first
    # NULL bands / bands that do not cover the grid rows
    assert lib.idg_grid_bands(h, fake, fake, fake, fake, None, 1, obs.grid_size, None) == 1
    assert "NULL" in lib.idg_last_error().decode()
    assert lib.idg_grid_bands(h, fake, fake, fake, fake, fake, 2, obs.grid_size // 2 - 1, None) == 1
    assert "cover" in lib.idg_last_error().decode()
    assert lib.idg_grid_bands(h, fake, fake, fake, fake, fake, 0, obs.grid_size, None) == 1
    assert lib.idg_degrid_bands(h, None, 1, obs.grid_size, fake, fake, fake, fake, None) == 1
    assert lib.idg_degrid_bands(h, fake, 3, 1, fake, fake, fake, fake, None) == 1
    assert lib.idg_grid_bands(None, fake, fake, fake, fake, fake, 1, obs.grid_size, None) == 1
    # IPC: NULL arguments
    off = ctypes.c_uint64()
    assert lib.idg_ipc_handle(None, (ctypes.c_ubyte * 64)(), ctypes.byref(off)) == 1
    assert lib.idg_ipc_open(None, 0, ctypes.byref(ctypes.c_void_p())) == 1
    assert lib.idg_ipc_close(None, 0) == 1
