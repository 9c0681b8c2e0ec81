"""Multi-GPU IDG: one process per GPU, baseline shards, NCCL for the two real exchange steps.

Work items are independent (the subgrid work is "embarrassingly parallel"), and the plan
is built per baseline, so a rank that owns baselines [b0, b1) builds exactly the global plan's items of
those baselines (tested in tests/test_parallel.py).  The path has one exchange per direction:

  gridding:   every rank grids its shard into a private uv-grid; the grids are summed with a
              torch.distributed reduce to the destination rank (the adder across ranks);
  degridding: the model grid is broadcast from the source rank; every rank degrids its own shard.

Both collectives can be restricted to the band of grid rows the items cover ("reduce only
the uv bounding box of the coverage"): the union over ranks of [min y, max y + N~) is agreed with one
2-element all-reduce, and each contiguous [plane][pol] row slab is reduced / broadcast on its own.  Rows
outside the band are zero on every rank after gridding and read by no item when degridding, so the
result is identical to the full-grid collective with less traffic.

torch.distributed is plumbing only (NCCL over NVLink on B200, gloo for the CPU tests); every step of the
hot path runs in libidg_b200.so.

BandedGrid fuses both exchanges into the kernels instead: the grid is distributed by row bands (rank r owns
rows [r R, (r+1) R) of every [plane][pol]), every rank's gridder adds each subgrid row straight into its
owner's band through CUDA-IPC peer memory (NVLink / NVSwitch) and every degridder's splitter reads the
owners' bands, so there is no reduce and no broadcast -- only a barrier between the two phases.
"""
from __future__ import annotations

import numpy as np


def shard_range(nr_baselines: int, rank: int, world: int, weights: np.ndarray | None = None):
    """Contiguous baseline range [b0, b1) of `rank`.

    Without weights the baselines are split evenly: every baseline carries T*C visibilities and its
    (pixel, visibility) pairs are N~^2 times its assigned visibilities, so equal counts are equal work.
    With per-baseline weights (e.g. pairs from a global plan) the split balances the cumulative weight.
    """
    if weights is None:
        return (nr_baselines * rank) // world, (nr_baselines * (rank + 1)) // world
    w = np.asarray(weights, dtype=np.float64)
    cum = np.concatenate([[0.0], np.cumsum(w)])
    total = cum[-1]
    b0 = int(np.searchsorted(cum, total * rank / world, side="left"))
    b1 = int(np.searchsorted(cum, total * (rank + 1) / world, side="left"))
    if rank == world - 1:
        b1 = nr_baselines
    return min(b0, nr_baselines), min(b1, nr_baselines)


def shard_arrays(uvw: np.ndarray, baselines: np.ndarray, b0: int, b1: int):
    """The rank's slice of the per-baseline inputs (uvw [nbl][T][3], baselines [nbl][2])."""
    return np.ascontiguousarray(uvw[b0:b1]), np.ascontiguousarray(baselines[b0:b1])


def coverage_rows(item_y, subgrid_size: int, grid_size: int):
    """Grid rows [y0, y1) covered by items with corner rows `item_y` (empty: (grid_size, 0))."""
    y = np.asarray(item_y)
    if y.size == 0:
        return grid_size, 0
    return int(y.min()), int(y.max()) + subgrid_size


def union_rows(rows, device=None, group=None):
    """Union over ranks of the local row bands (one 2-element MAX all-reduce)."""
    import torch
    import torch.distributed as dist
    y0, y1 = rows
    if not dist.is_initialized() or dist.get_world_size(group) == 1:
        return y0, y1
    t = torch.tensor([-y0, y1], dtype=torch.int64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX, group=group)
    return int(-t[0]), int(t[1])


def _slabs(grid, rows):
    """Contiguous [plane][pol] row slabs grid[..., y0:y1, :] as fp32 views (the whole grid if rows is None)."""
    import torch
    if rows is None:
        return [torch.view_as_real(grid)]
    y0, y1 = rows
    if y1 <= y0:
        return []
    n = grid.shape[-1]
    planes = grid.reshape(-1, grid.shape[-2], n)
    return [torch.view_as_real(planes[k, y0:y1]) for k in range(planes.shape[0])]


def reduce_grid(grid, dst: int = 0, group=None, rows=None):
    """Sum the ranks' complex64 uv-grids onto `dst` (in place on dst).  Complex is reduced as fp32 pairs.
    `rows` = (y0, y1), the same on every rank: reduce only that band of every plane/polarisation."""
    import torch.distributed as dist
    if not dist.is_initialized() or dist.get_world_size(group) == 1:
        return grid
    for slab in _slabs(grid, rows):
        dist.reduce(slab, dst=dst, op=dist.ReduceOp.SUM, group=group)
    return grid


def broadcast_grid(grid, src: int = 0, group=None, rows=None):
    """Broadcast the model grid from `src` to every rank (in place); `rows` as for reduce_grid."""
    import torch.distributed as dist
    if not dist.is_initialized() or dist.get_world_size(group) == 1:
        return grid
    for slab in _slabs(grid, rows):
        dist.broadcast(slab, src=src, group=group)
    return grid


class ShardedIDG:
    """The rank-local plan plus the two collectives.  Inputs are the rank's baseline slice.
    With `bbox` (default) the collectives move only the union band of covered grid rows."""

    def __init__(self, plan, bbox: bool = True):
        self.plan = plan
        self.bbox = bbox
        self._rows = None

    def rows(self, device=None):
        """The agreed row band (collective on first use; every rank must call it)."""
        if not self.bbox:
            return None
        if self._rows is None:
            md = self.plan.metadata()
            local = coverage_rows(md["y"], self.plan.subgrid_size, self.plan.grid_size)
            self._rows = union_rows(local, device=device)
        return self._rows

    def grid(self, vis, uvw, aterms, taper, grid_out, dst: int = 0, stream=None):
        from . import idg
        idg.grid(self.plan, vis, uvw, aterms, taper, grid_out, stream=stream)
        return reduce_grid(grid_out, dst=dst, rows=self.rows(grid_out.device))

    def degrid(self, grid_in, uvw, aterms, taper, vis_out, src: int = 0, stream=None):
        from . import idg
        broadcast_grid(grid_in, src=src, rows=self.rows(grid_in.device))
        return idg.degrid(self.plan, grid_in, uvw, aterms, taper, vis_out, stream=stream)

    # host-streamed variants (visibilities in pinned host memory)
    def grid_host(self, vis_host, uvw, aterms, taper, grid_out, ws, dst: int = 0, stream=None):
        from . import idg
        idg.grid_host(self.plan, vis_host, uvw, aterms, taper, grid_out, ws, stream=stream)
        return reduce_grid(grid_out, dst=dst, rows=self.rows(grid_out.device))

    def degrid_host(self, grid_in, uvw, aterms, taper, vis_host_out, ws, src: int = 0, stream=None):
        from . import idg
        broadcast_grid(grid_in, src=src, rows=self.rows(grid_in.device))
        return idg.degrid_host(self.plan, grid_in, uvw, aterms, taper, vis_host_out, ws, stream=stream)


# ---- banded grid: the exchange fused into the kernels (idg_grid_bands / idg_degrid_bands) --------------

def band_rows(grid_size: int, world: int) -> int:
    """Rows per band R = ceil(N / world): rank r owns grid rows [r R, min((r+1) R, N))."""
    return -(-int(grid_size) // max(1, int(world)))


def band_range(grid_size: int, world: int, rank: int):
    R = band_rows(grid_size, world)
    return min(rank * R, grid_size), min((rank + 1) * R, grid_size)


def split_bands(full, world: int):
    """The bands [..., R, N] of a full grid [..., N, N] (the last band zero-padded to R rows); numpy or torch."""
    N = full.shape[-1]
    R = band_rows(N, world)
    out = []
    for r in range(world):
        y0, y1 = band_range(N, world, r)
        if hasattr(full, "new_zeros"):
            b = full.new_zeros(full.shape[:-2] + (R, N))
        else:
            b = np.zeros(full.shape[:-2] + (R, N), dtype=full.dtype)
        b[..., : y1 - y0, :] = full[..., y0:y1, :]
        out.append(b)
    return out


def join_bands(bands, grid_size: int):
    """The full grid [..., N, N] from the bands (inverse of split_bands); numpy or torch."""
    world = len(bands)
    b0 = bands[0]
    if hasattr(b0, "new_zeros"):
        full = b0.new_zeros(b0.shape[:-2] + (grid_size, grid_size))
    else:
        full = np.zeros(b0.shape[:-2] + (grid_size, grid_size), dtype=b0.dtype)
    for r, b in enumerate(bands):
        y0, y1 = band_range(grid_size, world, r)
        full[..., y0:y1, :] = b[..., : y1 - y0, :]
    return full


class BandedGrid:
    """This rank's band of the distributed uv-grid plus peer mappings of every other rank's band.

    Construction is collective (every rank of `group` must call it): the bands' CUDA-IPC handles are
    exchanged once with all_gather_object and mapped (idg_ipc_open); `ptrs` is the device array of the
    world's band pointers the kernels take.  Phases are separated by `sync()` (this rank's stream, then a
    barrier): zero -> sync -> grid -> sync -> degrid (-> sync before the next zero)."""

    def __init__(self, plan, device, group=None):
        import torch
        import torch.distributed as dist
        from . import idg
        self.plan, self.group = plan, group
        on = dist.is_initialized() and dist.get_world_size(group) > 1
        self.world = dist.get_world_size(group) if on else 1
        self.rank = dist.get_rank(group) if on else 0
        self.R = band_rows(plan.grid_size, self.world)
        self.band = torch.zeros((plan.nr_w_planes, 4, self.R, plan.grid_size), dtype=torch.complex64, device=device)
        self._opened = []
        ptrs = [0] * self.world
        ptrs[self.rank] = self.band.data_ptr()
        if on:
            handles = [None] * self.world
            dist.all_gather_object(handles, idg.ipc_handle(self.band), group=group)
            with torch.cuda.device(self.band.device):
                for r, (h, off) in enumerate(handles):
                    if r != self.rank:
                        ptrs[r] = idg.ipc_open(h, off)
                        self._opened.append((ptrs[r], off))
        self.ptrs = torch.tensor(ptrs, dtype=torch.int64, device=device)

    def sync(self, stream=None):
        """This rank's queued work is complete and so is every other rank's (stream sync, then barrier)."""
        import torch
        import torch.distributed as dist
        (torch.cuda.current_stream(self.band.device) if stream is None else stream).synchronize()
        if self.world > 1:
            dist.barrier(group=self.group)

    def grid(self, vis, uvw, aterms, taper, stream=None):
        """Add this rank's visibilities into the world's bands (idg_grid_bands)."""
        from . import idg
        idg.grid_bands(self.plan, vis, uvw, aterms, taper, self.ptrs, self.R, stream=stream)

    def degrid(self, uvw, aterms, taper, vis_out, stream=None):
        """Predict this rank's visibilities from the world's bands (idg_degrid_bands)."""
        from . import idg
        return idg.degrid_bands(self.plan, self.ptrs, self.R, uvw, aterms, taper, vis_out, stream=stream)

    def gather(self, dst: int = 0):
        """The full grid [nz][4][N][N] on rank `dst` (None elsewhere) -- for checks and the image step."""
        import torch.distributed as dist
        N = self.plan.grid_size
        if self.world == 1:
            return join_bands([self.band], N)
        parts = [None] * self.world if self.rank == dst else None
        dist.gather_object(self.band.cpu(), parts, dst=dst, group=self.group)
        return join_bands([p.to(self.band.device) for p in parts], N) if self.rank == dst else None

    def load(self, full):
        """Set this rank's band from a full grid [nz][4][N][N] (or [4][N][N]) every rank holds."""
        N = self.plan.grid_size
        y0, y1 = band_range(N, self.world, self.rank)
        f = full.reshape(self.band.shape[:2] + (N, N))
        self.band.zero_()
        self.band[:, :, : y1 - y0, :] = f[:, :, y0:y1, :]

    def close(self):
        from . import idg
        for p, off in self._opened:
            idg.ipc_close(p, off)
        self._opened = []
