"""Thin ctypes binding of libidg_b200.so (include/idg.h).  Argument marshalling only: every step of the
hot path (plan builder, gridder, degridder, subgrid FFTs, adder, splitter) runs in the C/C++/CUDA library.

PyTorch supplies device memory and streams.  There is no CPU fallback: if the library is missing or
the device is not sm_100a the calls raise.
"""
from __future__ import annotations

import ctypes
import os
from typing import Optional

import numpy as np

from . import _build

_LIB_PATH = _build.LIB

METADATA_DTYPE = np.dtype([("baseline", "<i4"), ("time_offset", "<i4"), ("nr_timesteps", "<i4"),
                           ("channel_begin", "<i4"), ("channel_end", "<i4"), ("aterm_index", "<i4"),
                           ("x", "<i4"), ("y", "<i4"), ("z", "<i4")])

IDG_OK = 0


class IDGError(RuntimeError):
    def __init__(self, status: int, what: str, detail: str):
        super().__init__(f"{what}: {_status_name(status)}: {detail}")
        self.status = status


class PlanParams(ctypes.Structure):
    _fields_ = [("subgrid_size", ctypes.c_int32), ("grid_size", ctypes.c_int32),
                ("image_size", ctypes.c_double), ("kernel_size", ctypes.c_int32),
                ("max_timesteps_per_subgrid", ctypes.c_int32),
                ("max_channels_per_subgrid", ctypes.c_int32), ("w_offset", ctypes.c_double),
                ("nr_w_planes", ctypes.c_int32), ("w_step", ctypes.c_double)]


class KernelTime(ctypes.Structure):
    _fields_ = [("name", ctypes.c_char * 48), ("launches", ctypes.c_int64), ("total_ms", ctypes.c_double)]


_lib = None

EXPORTED = ["idg_plan_create", "idg_plan_destroy", "idg_plan_nr_subgrids", "idg_plan_metadata",
            "idg_plan_stats", "idg_workspace_size", "idg_grid", "idg_degrid", "idg_rho_benchmark",
            "idg_rho_benchmark_scalar",
            "idg_profiling_enable", "idg_profiling_reset", "idg_profiling_read", "idg_launch_count",
            "idg_kernel_variants", "idg_host_workspace_size", "idg_grid_host", "idg_degrid_host",
            "idg_host_adder_workspace_size", "idg_grid_host_adder", "idg_degrid_host_splitter",
            "idg_grid_bands", "idg_degrid_bands", "idg_ipc_handle", "idg_ipc_open", "idg_ipc_close",
            "idg_status_string", "idg_last_error", "idg_last_variant"]


def lib() -> ctypes.CDLL:
    """Load libidg_b200.so (built in-tree by __graft_entry__.build() / _build.py)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(_LIB_PATH):
        raise ImportError(f"{_LIB_PATH} is not built; run `python -m paper_conf_ipps_veenboerpr17_b200._build`"
                          " (or __graft_entry__.build()). There is no fallback implementation.")
    L = ctypes.CDLL(_LIB_PATH)
    P, i32, i64, sz = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64, ctypes.c_size_t
    L.idg_plan_create.argtypes = [ctypes.POINTER(PlanParams), i32, i32, i32, i32, P, P, P, i32, P,
                                  ctypes.POINTER(P)]
    L.idg_plan_destroy.argtypes = [P]
    L.idg_plan_nr_subgrids.argtypes = [P, ctypes.POINTER(i64)]
    L.idg_plan_metadata.argtypes = [P, P, i64]
    L.idg_plan_stats.argtypes = [P, ctypes.POINTER(i64), ctypes.POINTER(i64), ctypes.POINTER(i64)]
    L.idg_workspace_size.argtypes = [P, ctypes.POINTER(sz)]
    L.idg_grid.argtypes = [P, P, P, P, P, P, P, sz, P]
    L.idg_degrid.argtypes = [P, P, P, P, P, P, P, sz, P]
    L.idg_host_workspace_size.argtypes = [P, ctypes.POINTER(sz)]
    L.idg_grid_host.argtypes = [P, P, P, P, P, P, P, sz, P]
    L.idg_degrid_host.argtypes = [P, P, P, P, P, P, P, sz, P]
    L.idg_host_adder_workspace_size.argtypes = [P, ctypes.POINTER(sz)]
    L.idg_grid_host_adder.argtypes = [P, P, P, P, P, P, P, sz, P]
    L.idg_degrid_host_splitter.argtypes = [P, P, P, P, P, P, P, sz, P]
    L.idg_grid_bands.argtypes = [P, P, P, P, P, P, i32, i32, P]
    L.idg_degrid_bands.argtypes = [P, P, i32, i32, P, P, P, P, P]
    L.idg_ipc_handle.argtypes = [P, P, ctypes.POINTER(ctypes.c_uint64)]
    L.idg_ipc_open.argtypes = [P, ctypes.c_uint64, ctypes.POINTER(P)]
    L.idg_ipc_close.argtypes = [P, ctypes.c_uint64]
    for f in ("idg_rho_benchmark", "idg_rho_benchmark_scalar"):
        getattr(L, f).argtypes = [i32, i32, P, ctypes.POINTER(ctypes.c_double), ctypes.POINTER(ctypes.c_double)]
    L.idg_profiling_enable.argtypes = [i32]
    L.idg_profiling_read.argtypes = [ctypes.POINTER(KernelTime), i32, ctypes.POINTER(i32)]
    L.idg_launch_count.restype = i64
    L.idg_kernel_variants.restype = ctypes.c_char_p
    L.idg_kernel_variants.argtypes = [i32]
    L.idg_last_variant.restype = ctypes.c_char_p
    L.idg_last_variant.argtypes = [i32]
    L.idg_status_string.restype = ctypes.c_char_p
    L.idg_status_string.argtypes = [i32]
    L.idg_last_error.restype = ctypes.c_char_p
    for f in EXPORTED:
        if f not in ("idg_launch_count", "idg_status_string", "idg_last_error", "idg_kernel_variants",
                     "idg_last_variant"):
            getattr(L, f).restype = i32
    _lib = L
    return L


def _status_name(st: int) -> str:
    try:
        return lib().idg_status_string(st).decode()
    except Exception:  # pragma: no cover
        return str(st)


def _check(st: int, what: str):
    if st != IDG_OK:
        raise IDGError(st, what, lib().idg_last_error().decode(errors="replace"))


def _np(a, dtype):
    return np.ascontiguousarray(a, dtype=dtype)


class Plan:
    """idg_plan_create: host plan of visibility -> subgrid work items."""

    def __init__(self, *, subgrid_size: int, grid_size: int, image_size: float, kernel_size: int,
                 max_timesteps_per_subgrid: int, max_channels_per_subgrid: int = 0, w_offset: float = 0.0,
                 nr_w_planes: int = 1, w_step: float = 0.0,
                 nr_stations: int, uvw: np.ndarray, frequencies: np.ndarray, baselines: np.ndarray,
                 aterm_offsets: np.ndarray):
        self.params = PlanParams(subgrid_size, grid_size, image_size, kernel_size, max_timesteps_per_subgrid,
                                 max_channels_per_subgrid, w_offset, nr_w_planes, w_step)
        self.nr_w_planes = max(1, int(nr_w_planes))
        uvw = _np(uvw, np.float32)
        freqs = _np(frequencies, np.float64)
        bl = _np(baselines, np.int32)
        offs = _np(aterm_offsets, np.int32)
        if uvw.ndim != 3 or uvw.shape[2] != 3 or bl.shape != (uvw.shape[0], 2):
            raise ValueError("uvw must be [nbl][T][3] and baselines [nbl][2]")
        self.nr_stations = int(nr_stations)
        self.nr_baselines, self.nr_timesteps = int(uvw.shape[0]), int(uvw.shape[1])
        self.nr_channels = int(freqs.shape[0])
        self.nr_aterm_slots = int(offs.shape[0] - 1)
        self.subgrid_size, self.grid_size = int(subgrid_size), int(grid_size)
        h = ctypes.c_void_p()
        _check(lib().idg_plan_create(ctypes.byref(self.params), self.nr_stations, self.nr_baselines,
                                     self.nr_timesteps, self.nr_channels, uvw.ctypes.data, freqs.ctypes.data,
                                     bl.ctypes.data, self.nr_aterm_slots, offs.ctypes.data, ctypes.byref(h)),
               "idg_plan_create")
        self._h = h

    @classmethod
    def from_observation(cls, obs) -> "Plan":
        return cls(**obs.plan_params(), nr_stations=obs.nr_stations, uvw=obs.uvw, frequencies=obs.frequencies,
                   baselines=obs.baselines, aterm_offsets=obs.aterm_offsets)

    @property
    def handle(self):
        return self._h

    def __del__(self):
        h = getattr(self, "_h", None)
        if h is not None and h.value and _lib is not None:
            _lib.idg_plan_destroy(h)
            self._h = None

    @property
    def nr_subgrids(self) -> int:
        n = ctypes.c_int64()
        _check(lib().idg_plan_nr_subgrids(self._h, ctypes.byref(n)), "idg_plan_nr_subgrids")
        return int(n.value)

    def metadata(self) -> np.ndarray:
        n = self.nr_subgrids
        out = np.zeros(n, dtype=METADATA_DTYPE)
        _check(lib().idg_plan_metadata(self._h, out.ctypes.data, n), "idg_plan_metadata")
        return out

    def stats(self) -> dict:
        a, d, p = ctypes.c_int64(), ctypes.c_int64(), ctypes.c_int64()
        _check(lib().idg_plan_stats(self._h, ctypes.byref(a), ctypes.byref(d), ctypes.byref(p)), "idg_plan_stats")
        return {"nr_vis_assigned": a.value, "nr_vis_dropped": d.value, "nr_pairs": p.value,
                "nr_subgrids": self.nr_subgrids}

    def workspace_size(self) -> int:
        b = ctypes.c_size_t()
        _check(lib().idg_workspace_size(self._h, ctypes.byref(b)), "idg_workspace_size")
        return int(b.value)

    def host_adder_workspace_size(self) -> int:
        b = ctypes.c_size_t()
        _check(lib().idg_host_adder_workspace_size(self._h, ctypes.byref(b)), "idg_host_adder_workspace_size")
        return int(b.value)

    def host_workspace_size(self) -> int:
        b = ctypes.c_size_t()
        _check(lib().idg_host_workspace_size(self._h, ctypes.byref(b)), "idg_host_workspace_size")
        return int(b.value)


# ------------------------------------------------------------------------------------------------
# device calls (torch tensors are used only as device buffers)
# ------------------------------------------------------------------------------------------------

def _dev(t, dtype, shape, name):
    import torch
    if not isinstance(t, torch.Tensor) or not t.is_cuda:
        raise TypeError(f"{name} must be a CUDA torch tensor")
    if t.dtype != dtype:
        raise TypeError(f"{name} must be {dtype}, got {t.dtype}")
    if tuple(t.shape) != tuple(shape):
        raise ValueError(f"{name} must have shape {tuple(shape)}, got {tuple(t.shape)}")
    if not t.is_contiguous():
        raise ValueError(f"{name} must be contiguous")
    return ctypes.c_void_p(t.data_ptr())


def _stream(stream):
    import torch
    s = torch.cuda.current_stream() if stream is None else stream
    return ctypes.c_void_p(s.cuda_stream)


def _one_device(*tensors):
    """The single CUDA device of the call's device tensors (made current for the call: the plan's device
    copy and the default stream are per device)."""
    import torch
    devs = {t.device for t in tensors if isinstance(t, torch.Tensor) and t.is_cuda}
    if len(devs) != 1:
        raise ValueError(f"all device tensors of a call must be on one CUDA device, got {sorted(map(str, devs))}")
    return torch.cuda.device(devs.pop())


def _shapes(plan: Plan):
    import torch
    n = plan.subgrid_size
    return dict(vis=(torch.complex64, (plan.nr_baselines, plan.nr_timesteps, plan.nr_channels, 4)),
                uvw=(torch.float32, (plan.nr_baselines, plan.nr_timesteps, 3)),
                aterms=(torch.complex64, (plan.nr_aterm_slots, plan.nr_stations, n, n, 4)),
                taper=(torch.float32, (n, n)),
                grid=(torch.complex64, (4, plan.grid_size, plan.grid_size) if plan.nr_w_planes == 1
                      else (plan.nr_w_planes, 4, plan.grid_size, plan.grid_size)))


def grid(plan: Plan, vis, uvw, aterms, taper, grid_out, stream=None):
    """idg_grid: grid_out += gridded visibilities.  Asynchronous on `stream` (default: current)."""
    sh = _shapes(plan)
    args = [_dev(vis, *sh["vis"], "vis"), _dev(uvw, *sh["uvw"], "uvw"), _dev(aterms, *sh["aterms"], "aterms"),
            _dev(taper, *sh["taper"], "taper"), _dev(grid_out, *sh["grid"], "grid")]
    with _one_device(vis, uvw, aterms, taper, grid_out):
        _check(lib().idg_grid(plan.handle, *args, None, 0, _stream(stream)), "idg_grid")
    return grid_out


def degrid(plan: Plan, grid_in, uvw, aterms, taper, vis_out, stream=None):
    """idg_degrid: vis_out = predicted visibilities; dropped visibilities are 0."""
    sh = _shapes(plan)
    args = [_dev(grid_in, *sh["grid"], "grid"), _dev(uvw, *sh["uvw"], "uvw"),
            _dev(aterms, *sh["aterms"], "aterms"), _dev(taper, *sh["taper"], "taper"),
            _dev(vis_out, *sh["vis"], "vis")]
    with _one_device(grid_in, uvw, aterms, taper, vis_out):
        _check(lib().idg_degrid(plan.handle, *args, None, 0, _stream(stream)), "idg_degrid")
    return vis_out


def _bands_args(plan: Plan, bands_ptrs, band_rows: int):
    """(device pointer array, count) of a banded grid: bands_ptrs is an int64 CUDA tensor of band pointers."""
    import torch
    if not (isinstance(bands_ptrs, torch.Tensor) and bands_ptrs.is_cuda and bands_ptrs.dtype == torch.int64
            and bands_ptrs.dim() == 1 and bands_ptrs.is_contiguous()):
        raise TypeError("bands_ptrs must be a contiguous 1-D int64 CUDA tensor of band pointers")
    if band_rows < 1 or bands_ptrs.numel() * band_rows < plan.grid_size:
        raise ValueError("the bands must cover the grid rows (nr_bands * band_rows >= grid_size)")
    return ctypes.c_void_p(bands_ptrs.data_ptr()), int(bands_ptrs.numel())


def grid_bands(plan: Plan, vis, uvw, aterms, taper, bands_ptrs, band_rows: int, stream=None):
    """idg_grid_bands: every band += its rows of the gridded visibilities (the adder into the owners' bands,
    possibly other ranks' memory: the cross-rank reduction fused into the gridder)."""
    sh = _shapes(plan)
    args = [_dev(vis, *sh["vis"], "vis"), _dev(uvw, *sh["uvw"], "uvw"), _dev(aterms, *sh["aterms"], "aterms"),
            _dev(taper, *sh["taper"], "taper")]
    bp, nb = _bands_args(plan, bands_ptrs, band_rows)
    with _one_device(vis, uvw, aterms, taper, bands_ptrs):
        _check(lib().idg_grid_bands(plan.handle, *args, bp, nb, int(band_rows), _stream(stream)), "idg_grid_bands")


def degrid_bands(plan: Plan, bands_ptrs, band_rows: int, uvw, aterms, taper, vis_out, stream=None):
    """idg_degrid_bands: vis_out = predictions from the banded model grid (the splitter reads the owners'
    bands: no broadcast)."""
    sh = _shapes(plan)
    bp, nb = _bands_args(plan, bands_ptrs, band_rows)
    args = [_dev(uvw, *sh["uvw"], "uvw"), _dev(aterms, *sh["aterms"], "aterms"), _dev(taper, *sh["taper"], "taper"),
            _dev(vis_out, *sh["vis"], "vis")]
    with _one_device(uvw, aterms, taper, vis_out, bands_ptrs):
        _check(lib().idg_degrid_bands(plan.handle, bp, nb, int(band_rows), *args, _stream(stream)),
               "idg_degrid_bands")
    return vis_out


def ipc_handle(t) -> tuple[bytes, int]:
    """(64-byte CUDA IPC handle of t's allocation, byte offset of t in it)."""
    h = (ctypes.c_ubyte * 64)()
    off = ctypes.c_uint64(0)
    with _one_device(t):
        _check(lib().idg_ipc_handle(ctypes.c_void_p(t.data_ptr()), h, ctypes.byref(off)), "idg_ipc_handle")
    return bytes(h), int(off.value)


def ipc_open(handle: bytes, offset: int) -> int:
    """Map another process's allocation (current device); returns the device pointer at `offset`."""
    if len(handle) != 64:
        raise ValueError("a CUDA IPC handle has 64 bytes")
    p = ctypes.c_void_p()
    _check(lib().idg_ipc_open((ctypes.c_ubyte * 64).from_buffer_copy(handle), ctypes.c_uint64(offset),
                              ctypes.byref(p)), "idg_ipc_open")
    return int(p.value)


def ipc_close(ptr: int, offset: int):
    _check(lib().idg_ipc_close(ctypes.c_void_p(ptr), ctypes.c_uint64(offset)), "idg_ipc_close")


def _host(t, dtype, shape, name):
    import torch
    if not isinstance(t, torch.Tensor) or t.is_cuda:
        raise TypeError(f"{name} must be a CPU torch tensor (pinned for overlap)")
    if t.dtype != dtype or tuple(t.shape) != tuple(shape) or not t.is_contiguous():
        raise ValueError(f"{name} must be a contiguous {dtype} tensor of shape {tuple(shape)}")
    return ctypes.c_void_p(t.data_ptr())


def workspace(plan: Plan, device=None, full: bool = False, max_buffers: int = 0):
    """A device workspace for the host-streamed calls: the minimum (idg_host_workspace_size, three
    staging buffers per direction); with full=True one staging buffer per work group and direction
    (2 x the visibility bytes) so consecutive grid/degrid calls overlap completely; with max_buffers=k
    up to k staging buffers per direction (no more than one per work group)."""
    import torch
    n = plan.host_workspace_size()
    per_buffer = n // 6                        # idg_host_workspace_size = 2 directions x 3 buffers
    all_groups = 2 * plan.nr_baselines * plan.nr_timesteps * plan.nr_channels * 32 + (64 << 20)
    if full:
        n = max(n, all_groups)
    elif max_buffers > 3:
        n = max(n, min(all_groups, 2 * max_buffers * per_buffer))
    return torch.empty(max(1, n), dtype=torch.uint8, device=device or "cuda")


def _workspace_ok(ws):
    import torch
    if not isinstance(ws, torch.Tensor) or not ws.is_cuda or ws.dtype != torch.uint8 or not ws.is_contiguous():
        raise TypeError("ws must be a contiguous uint8 CUDA tensor (see workspace())")


def grid_host(plan: Plan, vis_host, uvw, aterms, taper, grid_out, ws, stream=None):
    """idg_grid_host: visibilities in (pinned) host memory, streamed through `ws`."""
    sh = _shapes(plan)
    args = [_host(vis_host, *sh["vis"], "vis_host"), _dev(uvw, *sh["uvw"], "uvw"),
            _dev(aterms, *sh["aterms"], "aterms"), _dev(taper, *sh["taper"], "taper"),
            _dev(grid_out, *sh["grid"], "grid")]
    _workspace_ok(ws)
    with _one_device(uvw, aterms, taper, grid_out, ws):
        _check(lib().idg_grid_host(plan.handle, *args, ctypes.c_void_p(ws.data_ptr()), ws.numel(),
                                   _stream(stream)), "idg_grid_host")
    return grid_out


def degrid_host(plan: Plan, grid_in, uvw, aterms, taper, vis_host_out, ws, stream=None):
    """idg_degrid_host: predicted visibilities streamed back into (pinned) host memory."""
    sh = _shapes(plan)
    args = [_dev(grid_in, *sh["grid"], "grid"), _dev(uvw, *sh["uvw"], "uvw"),
            _dev(aterms, *sh["aterms"], "aterms"), _dev(taper, *sh["taper"], "taper"),
            _host(vis_host_out, *sh["vis"], "vis_host_out")]
    _workspace_ok(ws)
    with _one_device(grid_in, uvw, aterms, taper, ws):
        _check(lib().idg_degrid_host(plan.handle, *args, ctypes.c_void_p(ws.data_ptr()), ws.numel(),
                                     _stream(stream)), "idg_degrid_host")
    return vis_host_out


def adder_workspace(plan: Plan, device=None, buffers: int = 3):
    """A device workspace for the host adder / splitter calls: `buffers` (>= 3) staging buffers per direction."""
    import torch
    n = plan.host_adder_workspace_size() * max(3, int(buffers)) // 3
    return torch.empty(max(1, n), dtype=torch.uint8, device=device or "cuda")


def grid_host_adder(plan: Plan, vis_host, uvw, aterms, taper, grid_host_out, ws, stream=None):
    """idg_grid_host_adder: visibilities and the grid in HOST memory; subgrids added on the host."""
    sh = _shapes(plan)
    args = [_host(vis_host, *sh["vis"], "vis_host"), _dev(uvw, *sh["uvw"], "uvw"),
            _dev(aterms, *sh["aterms"], "aterms"), _dev(taper, *sh["taper"], "taper"),
            _host(grid_host_out, *sh["grid"], "grid_host")]
    _workspace_ok(ws)
    with _one_device(uvw, aterms, taper, ws):
        _check(lib().idg_grid_host_adder(plan.handle, *args, ctypes.c_void_p(ws.data_ptr()), ws.numel(),
                                         _stream(stream)), "idg_grid_host_adder")
    return grid_host_out


def degrid_host_splitter(plan: Plan, grid_host, uvw, aterms, taper, vis_host_out, ws, stream=None):
    """idg_degrid_host_splitter: the model grid in HOST memory, subgrids split on the host."""
    sh = _shapes(plan)
    args = [_host(grid_host, *sh["grid"], "grid_host"), _dev(uvw, *sh["uvw"], "uvw"),
            _dev(aterms, *sh["aterms"], "aterms"), _dev(taper, *sh["taper"], "taper"),
            _host(vis_host_out, *sh["vis"], "vis_host_out")]
    _workspace_ok(ws)
    with _one_device(uvw, aterms, taper, ws):
        _check(lib().idg_degrid_host_splitter(plan.handle, *args, ctypes.c_void_p(ws.data_ptr()), ws.numel(),
                                              _stream(stream)), "idg_degrid_host_splitter")
    return vis_host_out


def rho_benchmark(rho: int = 17, iterations: int = 4096, stream=None, scalar: bool = False) -> tuple[float, float]:
    """The paper's FMA:sincos benchmark: returns (ops/s, seconds) at ratio rho.  FMAs as packed
    FFMA2 pairs (B200 form), or as scalar FFMA with scalar=True (the paper's form)."""
    ops, sec = ctypes.c_double(), ctypes.c_double()
    f = lib().idg_rho_benchmark_scalar if scalar else lib().idg_rho_benchmark
    _check(f(int(rho), int(iterations), _stream(stream), ctypes.byref(ops), ctypes.byref(sec)), "idg_rho_benchmark")
    return ops.value, sec.value


def profiling_enable(on: bool = True):
    _check(lib().idg_profiling_enable(1 if on else 0), "idg_profiling_enable")


def profiling_reset():
    _check(lib().idg_profiling_reset(), "idg_profiling_reset")


def profiling_read() -> dict:
    buf = (KernelTime * 32)()
    n = ctypes.c_int32()
    _check(lib().idg_profiling_read(buf, 32, ctypes.byref(n)), "idg_profiling_read")
    return {buf[i].name.decode(): {"launches": int(buf[i].launches), "total_ms": float(buf[i].total_ms)}
            for i in range(min(n.value, 32))}


def kernel_variants(which: str) -> list[str]:
    """Compiled launch-shape variants of the 'gridder' or 'degridder' (see IDG_*_VARIANT)."""
    return lib().idg_kernel_variants(0 if which == "gridder" else 1).decode().split()


def last_variant(which: str) -> str:
    """Variant the most recent 'gridder' / 'degridder' launch in this process used ('' before any)."""
    return lib().idg_last_variant(0 if which == "gridder" else 1).decode()


def launch_count() -> int:
    return int(lib().idg_launch_count())
