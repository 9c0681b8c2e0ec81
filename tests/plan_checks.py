"""Property checks of an execution plan (Fig. 5; readings R-8..R-16 in DESIGN.md).

They do not re-run the greedy algorithm; they check what any correct plan must satisfy:
  * partition: every (baseline, time, channel) is in exactly one item, or is counted as dropped;
  * coverage: each item's uv footprint (all its timesteps x channels, in grid cells) plus the kernel
    support K fits in N~ (R-10), and the subgrid lies on the grid (R-12);
  * placement: the subgrid centre cell is within half a cell of the footprint centre (R-11);
  * T~ <= T~max; no item straddles an A-term slot and aterm_index is the slot of t0 (R-15);
  * greedy maximality: an item that could have been extended (same slot, below T~max, not at T)
    would NOT fit with one more timestep ("as many time steps as possible");
  * drops are forced: every visibility left out belongs to a (baseline, timestep, channel block) that
    cannot form an item on its own — its footprint + K exceeds N~ (R-13) or its subgrid falls off the
    grid (R-12) — so a plan cannot pass by dropping data it could have gridded.
Shared by the oracle-plan tests (CPU) and the library-plan tests.
"""
import numpy as np

C0 = 299792458.0


def uv_cells(obs):
    """[nbl][T][C] u and v in grid cells, evaluated as u * nu / c * L in fp64 (R-10)."""
    uvw = obs.uvw.astype(np.float64)
    f = obs.frequencies[None, None, :]
    u = uvw[:, :, 0:1] * f / C0 * obs.image_size
    v = uvw[:, :, 1:2] * f / C0 * obs.image_size
    return u, v


def check_plan(obs, items, nr_dropped, check_maximal=True):
    n, N, K = obs.subgrid_size, obs.grid_size, obs.kernel_size
    T, C = obs.nr_timesteps, obs.nr_channels
    offs = obs.aterm_offsets
    u, v = uv_cells(obs)
    cover = np.zeros((obs.nr_baselines, T, C), dtype=np.int32)
    for it in items:
        b, t0, nt = int(it["baseline"]), int(it["time_offset"]), int(it["nr_timesteps"])
        c0, c1 = int(it["channel_begin"]), int(it["channel_end"])
        x, y, slot = int(it["x"]), int(it["y"]), int(it["aterm_index"])
        assert 1 <= nt <= obs.max_timesteps_per_subgrid
        assert 0 <= c0 < c1 <= C and 0 <= t0 and t0 + nt <= T
        cover[b, t0:t0 + nt, c0:c1] += 1
        # A-term slot
        assert offs[slot] <= t0 and t0 + nt <= offs[slot + 1], (it, offs[slot], offs[slot + 1])
        uu, vv = u[b, t0:t0 + nt, c0:c1], v[b, t0:t0 + nt, c0:c1]
        assert (uu.max() - uu.min()) + K <= n and (vv.max() - vv.min()) + K <= n
        assert 0 <= x and x + n <= N and 0 <= y and y + n <= N
        cu = (uu.max() + uu.min()) / 2 + N / 2
        cv = (vv.max() + vv.min()) / 2 + N / 2
        assert abs(x + n / 2 - cu) <= 0.5 + 1e-9 and abs(y + n / 2 - cv) <= 0.5 + 1e-9
        nz = getattr(obs, "nr_w_planes", 1)
        if nz > 1:   # R-21: every timestep's w lies in the item's plane interval (edge planes unbounded)
            z = int(it["z"])
            assert 0 <= z < nz
            nu_ref = obs.frequencies[c0 + (c1 - c0) // 2]
            w = obs.uvw[b, t0:t0 + nt, 2].astype(np.float64) * nu_ref / C0
            w0 = obs.w_offset + (z - (nz - 1) / 2) * obs.w_step
            lo = -np.inf if z == 0 else w0 - obs.w_step / 2 - 1e-9 * obs.w_step
            hi = np.inf if z == nz - 1 else w0 + obs.w_step / 2 + 1e-9 * obs.w_step
            assert np.all((w >= lo) & (w <= hi)), (it, w.min(), w.max(), lo, hi)
        else:
            assert int(it["z"]) == 0
        if check_maximal:
            te = t0 + nt
            if te < T and te < offs[slot + 1] and nt < obs.max_timesteps_per_subgrid:
                uu, vv = u[b, t0:te + 1, c0:c1], v[b, t0:te + 1, c0:c1]
                fits = (uu.max() - uu.min()) + K <= n and (vv.max() - vv.min()) + K <= n
                if nz > 1:   # the next timestep may also start a new W-plane
                    wn = float(obs.uvw[b, te, 2]) * nu_ref / C0
                    fits = fits and (lo <= wn <= hi)
                assert not fits, f"item {it} is not maximal"
    assert cover.max(initial=0) <= 1, "visibility in two items"
    assert int((cover == 0).sum()) == nr_dropped, (int((cover == 0).sum()), nr_dropped)
    cb = obs.max_channels_per_subgrid or C
    for c0 in range(0, C, cb):
        c1 = min(C, c0 + cb)
        blk = cover[:, :, c0:c1]
        assert np.all((blk == 0).all(axis=2) | (blk == 1).all(axis=2)), "channel block split across items"
        for b, t in zip(*np.nonzero((blk == 0).all(axis=2))):
            uu, vv = u[b, t, c0:c1], v[b, t, c0:c1]
            too_wide = (uu.max() - uu.min()) + K > n or (vv.max() - vv.min()) + K > n
            x = np.floor((uu.max() + uu.min()) / 2 + N / 2 + 0.5) - n / 2
            y = np.floor((vv.max() + vv.min()) / 2 + N / 2 + 0.5) - n / 2
            off_grid = not (0 <= x and x + n <= N and 0 <= y and y + n <= N)
            assert too_wide or off_grid, f"baseline {b} timestep {t} channels [{c0},{c1}) dropped but fits"
    return cover
