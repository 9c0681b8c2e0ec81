"""ctypes front-end of the fp64 CPU oracle (oracle/idg_oracle.c).

TEST INFRASTRUCTURE ONLY: only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
``--impl reference`` leg may import this.  It never imports the product package
(paper_conf_ipps_veenboerpr17_b200) and the product never imports it.

Every function mirrors one step of the paper (P:n = /root/reference/PAPER.md line n):
  plan()            execution plan, P:93-145 (Fig. 5)
  gridder_item()    Alg. 1 + A-term/taper + subgrid FFT for one work item
  grid()            gridder -> subgrid FFT -> adder
  degridder_item()  subgrid iFFT + Alg. 2 for one work item
  degrid()          splitter -> subgrid iFFT -> degridder
  centred_dft()     the subgrid transform (direct O(N~^4) DFT)
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "idg_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

ITEM_DTYPE = np.dtype([("baseline", "<i4"), ("time_offset", "<i4"), ("nr_timesteps", "<i4"),
                       ("channel_begin", "<i4"), ("channel_end", "<i4"), ("aterm_index", "<i4"),
                       ("x", "<i4"), ("y", "<i4"), ("z", "<i4")])


class _Params(ctypes.Structure):
    _fields_ = [("subgrid_size", ctypes.c_int32), ("grid_size", ctypes.c_int32),
                ("image_size", ctypes.c_double), ("kernel_size", ctypes.c_int32),
                ("max_timesteps_per_subgrid", ctypes.c_int32),
                ("max_channels_per_subgrid", ctypes.c_int32), ("w_offset", ctypes.c_double),
                ("nr_w_planes", ctypes.c_int32), ("w_step", ctypes.c_double)]


def build(force: bool = False) -> str:
    """Compile liboracle.so with gcc (fp64, OpenMP, no FP contraction so the plan is reproducible)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-D_GNU_SOURCE", "-fopenmp", "-ffp-contract=off",
                               "-fno-fast-math", "-fPIC", "-shared", "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def lib():
    """The compiled oracle.  IDG_ORACLE_LIB (test infrastructure: tests/test_oracle_mutants.py) loads a
    mutated build of idg_oracle.c instead, to show that the pins reject it."""
    global _lib
    if _lib is None:
        _lib = ctypes.CDLL(os.environ.get("IDG_ORACLE_LIB") or build())
        P = ctypes.c_void_p
        i32, i64 = ctypes.c_int32, ctypes.c_int64
        _lib.oracle_plan.restype = i64
        _lib.oracle_plan.argtypes = [P, i32, i32, i32, i32, P, P, P, i32, P, ctypes.POINTER(P),
                                     ctypes.POINTER(i64)]
        _lib.oracle_free.argtypes = [P]
        _lib.oracle_centred_dft.argtypes = [i32, i32, P, P]
        _lib.oracle_gridder_item.argtypes = [P, i32, i32, i32, P, P, P, P, P, P, P, P]
        _lib.oracle_degridder_item.argtypes = [P, i32, i32, P, P, P, P, P, P, P, P]
        _lib.oracle_grid.argtypes = [P, i32, i32, i32, P, P, P, P, i64, P, P, P, P, i32]
        _lib.oracle_degrid.argtypes = [P, i32, i32, P, P, P, P, i64, P, i32, P, P, P, i32]
        _lib.oracle_max_threads.restype = i32
    return _lib


def max_threads() -> int:
    return int(lib().oracle_max_threads())


def _ptr(a: np.ndarray):
    return ctypes.c_void_p(a.ctypes.data)


def _params(p: dict) -> _Params:
    return _Params(int(p["subgrid_size"]), int(p["grid_size"]), float(p["image_size"]),
                   int(p["kernel_size"]), int(p["max_timesteps_per_subgrid"]),
                   int(p["max_channels_per_subgrid"]), float(p["w_offset"]),
                   int(p.get("nr_w_planes", 1)), float(p.get("w_step", 0.0)))


def _c(a, dtype):
    return np.ascontiguousarray(a, dtype=dtype)


def plan(obs, params: dict | None = None):
    """Execution plan of `obs` (an idgsynth.Observation). Returns (items[ITEM_DTYPE], nr_dropped)."""
    p = _params(obs.plan_params() if params is None else params)
    uvw = _c(obs.uvw, np.float32)
    fr = _c(obs.frequencies, np.float64)
    bl = _c(obs.baselines, np.int32)
    off = _c(obs.aterm_offsets, np.int32)
    out = ctypes.c_void_p()
    dropped = ctypes.c_int64()
    n = lib().oracle_plan(ctypes.byref(p), obs.nr_stations, obs.nr_baselines, obs.nr_timesteps,
                          obs.nr_channels, _ptr(uvw), _ptr(fr), _ptr(bl), obs.nr_aterm_slots, _ptr(off),
                          ctypes.byref(out), ctypes.byref(dropped))
    items = np.empty(n, dtype=ITEM_DTYPE)
    if n:
        ctypes.memmove(items.ctypes.data, out.value, n * ITEM_DTYPE.itemsize)
    lib().oracle_free(out)
    return items, int(dropped.value)


def centred_dft(plane: np.ndarray, sign: int) -> np.ndarray:
    """Centred 2-D DFT of one N~xN~ plane (sign -1: forward / gridding; +1: adjoint / degridding)."""
    a = _c(plane, np.complex128)
    out = np.empty_like(a)
    lib().oracle_centred_dft(a.shape[0], int(sign), _ptr(a), _ptr(out))
    return out


def gridder_item(obs, item, vis, aterms, taper) -> np.ndarray:
    """Transformed subgrid [4][N~][N~] (complex128) of one work item."""
    p = _params(obs.plan_params())
    n = obs.subgrid_size
    out = np.zeros((4, n, n), dtype=np.complex128)
    it = np.asarray(item, dtype=ITEM_DTYPE).reshape(1)
    args = [_c(obs.uvw, np.float32), _c(obs.frequencies, np.float64), _c(obs.baselines, np.int32)]
    v, a, t = _c(vis, np.complex64), _c(aterms, np.complex64), _c(taper, np.float32)
    lib().oracle_gridder_item(ctypes.byref(p), obs.nr_stations, obs.nr_timesteps, obs.nr_channels,
                              _ptr(args[0]), _ptr(args[1]), _ptr(args[2]), _ptr(it), _ptr(v), _ptr(a),
                              _ptr(t), _ptr(out))
    return out


def degridder_item(obs, item, subgrid, aterms, taper) -> np.ndarray:
    """Visibilities [T~][C~][4] (complex128) of one work item from a split subgrid [4][N~][N~]."""
    p = _params(obs.plan_params())
    it = np.asarray(item, dtype=ITEM_DTYPE).reshape(1)
    nt, nc = int(it["nr_timesteps"][0]), int(it["channel_end"][0] - it["channel_begin"][0])
    out = np.zeros((nt, nc, 4), dtype=np.complex128)
    uvw, fr, bl = _c(obs.uvw, np.float32), _c(obs.frequencies, np.float64), _c(obs.baselines, np.int32)
    s, a, t = _c(subgrid, np.complex128), _c(aterms, np.complex64), _c(taper, np.float32)
    lib().oracle_degridder_item(ctypes.byref(p), obs.nr_stations, obs.nr_timesteps, _ptr(uvw), _ptr(fr),
                                _ptr(bl), _ptr(it), _ptr(s), _ptr(a), _ptr(t), _ptr(out))
    return out


def grid_shape(obs):
    """[4][N][N], or [nz][4][N][N] with W-stacking (R-21)."""
    nz = int(obs.plan_params().get("nr_w_planes", 1))
    N = obs.grid_size
    return (4, N, N) if nz <= 1 else (nz, 4, N, N)


def grid(obs, items, vis, aterms, taper, grid_out: np.ndarray | None = None, nthreads: int = 0):
    """Accumulate the gridded visibilities of `items` into a complex128 grid_shape(obs) grid."""
    p = _params(obs.plan_params())
    g = np.zeros(grid_shape(obs), dtype=np.complex128) if grid_out is None else grid_out
    assert g.dtype == np.complex128 and g.flags.c_contiguous
    it = _c(items, ITEM_DTYPE)
    uvw, fr, bl = _c(obs.uvw, np.float32), _c(obs.frequencies, np.float64), _c(obs.baselines, np.int32)
    v, a, t = _c(vis, np.complex64), _c(aterms, np.complex64), _c(taper, np.float32)
    lib().oracle_grid(ctypes.byref(p), obs.nr_stations, obs.nr_timesteps, obs.nr_channels, _ptr(uvw),
                      _ptr(fr), _ptr(bl), _ptr(it), len(it), _ptr(v), _ptr(a), _ptr(t), _ptr(g), nthreads)
    return g


def degrid(obs, items, grid_in, aterms, taper, nthreads: int = 0) -> np.ndarray:
    """Predicted visibilities of `items`, concatenated item blocks [T~][C~][4] (complex128, flat).
    `grid_in` is complex64 (the product's grid format) or complex128 (exact models for the pins)."""
    p = _params(obs.plan_params())
    it = _c(items, ITEM_DTYPE)
    total = int(np.sum(it["nr_timesteps"].astype(np.int64) * (it["channel_end"] - it["channel_begin"]))) * 4
    out = np.zeros(total, dtype=np.complex128)
    uvw, fr, bl = _c(obs.uvw, np.float32), _c(obs.frequencies, np.float64), _c(obs.baselines, np.int32)
    f64 = np.asarray(grid_in).dtype == np.complex128
    g = _c(grid_in, np.complex128 if f64 else np.complex64)
    a, t = _c(aterms, np.complex64), _c(taper, np.float32)
    lib().oracle_degrid(ctypes.byref(p), obs.nr_stations, obs.nr_timesteps, _ptr(uvw), _ptr(fr), _ptr(bl),
                        _ptr(it), len(it), _ptr(g), int(f64), _ptr(a), _ptr(t), _ptr(out), nthreads)
    return out


def scatter_visibilities(obs, items, flat: np.ndarray) -> np.ndarray:
    """Place degrid() output into a full [nbl][T][C][4] array (visibilities not in any item stay 0)."""
    full = np.zeros((obs.nr_baselines, obs.nr_timesteps, obs.nr_channels, 4), dtype=flat.dtype)
    pos = 0
    for it in items:
        nt, c0, c1 = int(it["nr_timesteps"]), int(it["channel_begin"]), int(it["channel_end"])
        t0, b = int(it["time_offset"]), int(it["baseline"])
        k = nt * (c1 - c0) * 4
        full[b, t0:t0 + nt, c0:c1, :] = flat[pos:pos + k].reshape(nt, c1 - c0, 4)
        pos += k
    return full


def gather_visibilities(obs, items, full: np.ndarray) -> np.ndarray:
    """Inverse of scatter_visibilities: the visibilities of `items`, concatenated in item order."""
    parts = []
    for it in items:
        nt, c0, c1 = int(it["nr_timesteps"]), int(it["channel_begin"]), int(it["channel_end"])
        t0, b = int(it["time_offset"]), int(it["baseline"])
        parts.append(np.asarray(full[b, t0:t0 + nt, c0:c1, :]).reshape(-1))
    return np.concatenate(parts) if parts else np.zeros(0, dtype=full.dtype)
