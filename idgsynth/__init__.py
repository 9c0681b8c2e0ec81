"""Seeded synthetic inputs for IDG (shared by the oracle tests, the GPU tests and bench.py).

This module generates INPUTS only: station layouts, earth-rotation uvw tracks, channel frequencies,
baseline lists, A-term slot boundaries, A-term Jones matrices, a spheroidal taper and visibilities.
It contains none of the method's arithmetic (no plan, no phasor, no DFT, no gridding) and imports
neither ``oracle/`` nor the product package; both sides consume what it returns.

Workload shapes follow PAPER.md (P:n = /root/reference/PAPER.md line n):
  * visibilities V in C^{2x2} per (baseline, time, channel), 4 pols XX,XY,YX,YY;
  * uvw per (baseline, time) in metres, scaled per channel by nu/c;
  * SKA-1-low-like data set: 150 stations, T=8192 x 1 s, A-terms updated every 256 steps.
The concrete configs are SURVEY.md section 8(d) (restated in DESIGN.md "Input recipe").
"""
from __future__ import annotations

import dataclasses
import math

import numpy as np

SPEED_OF_LIGHT = 299792458.0
SIDEREAL_RATE = 2.0 * math.pi / 86164.0905  # rad/s


@dataclasses.dataclass
class Observation:
    """One synthetic observation: everything idg_plan_create/idg_grid/idg_degrid take as input."""
    name: str
    nr_stations: int
    baselines: np.ndarray        # int32 [nbl][2], station1 < station2 (lexicographic)
    uvw: np.ndarray              # float32 [nbl][T][3] metres
    frequencies: np.ndarray      # float64 [C] Hz
    aterm_offsets: np.ndarray    # int32 [slots+1], 0 ... T
    subgrid_size: int            # N~
    grid_size: int               # N
    image_size: float            # L (direction cosines); cell du = 1/L wavelengths
    kernel_size: int             # K (support reserved in the subgrid, Fig. 5)
    max_timesteps_per_subgrid: int   # T~max
    max_channels_per_subgrid: int    # C~ (0 = all channels)
    w_offset: float              # w0 (wavelengths)
    seed: int
    aterm_kind: str = "identity"     # "identity" | "random"
    nr_w_planes: int = 1             # W-stacking planes; 1 = none
    w_step: float = 0.0              # plane spacing (wavelengths)

    @property
    def nr_baselines(self) -> int:
        return int(self.baselines.shape[0])

    @property
    def nr_timesteps(self) -> int:
        return int(self.uvw.shape[1])

    @property
    def nr_channels(self) -> int:
        return int(self.frequencies.shape[0])

    @property
    def nr_aterm_slots(self) -> int:
        return int(self.aterm_offsets.shape[0] - 1)

    @property
    def nr_visibilities(self) -> int:
        return self.nr_baselines * self.nr_timesteps * self.nr_channels

    def plan_params(self) -> dict:
        return dict(subgrid_size=self.subgrid_size, grid_size=self.grid_size,
                    image_size=self.image_size, kernel_size=self.kernel_size,
                    max_timesteps_per_subgrid=self.max_timesteps_per_subgrid,
                    max_channels_per_subgrid=self.max_channels_per_subgrid,
                    w_offset=self.w_offset, nr_w_planes=self.nr_w_planes, w_step=self.w_step)

    def subset(self, nr_baselines: int | None = None, nr_timesteps: int | None = None,
               baseline_begin: int = 0) -> "Observation":
        """A deterministic slice (first baselines x first timesteps) with the SAME L, N, taper etc."""
        nb = self.nr_baselines - baseline_begin if nr_baselines is None else nr_baselines
        nt = self.nr_timesteps if nr_timesteps is None else nr_timesteps
        offs = [o for o in self.aterm_offsets.tolist() if o < nt] + [nt]
        return dataclasses.replace(
            self, name=f"{self.name}[bl{baseline_begin}+{nb},t{nt}]",
            baselines=np.ascontiguousarray(self.baselines[baseline_begin:baseline_begin + nb]),
            uvw=np.ascontiguousarray(self.uvw[baseline_begin:baseline_begin + nb, :nt]),
            aterm_offsets=np.asarray(offs, dtype=np.int32))

    def select(self, baselines, nr_timesteps: int | None = None, time_begin: int = 0) -> "Observation":
        """Any baselines (index list) over timesteps [time_begin, time_begin + nr_timesteps), with the SAME
        L, N, taper, stations (A-term rows) etc.; A-term slot boundaries are cut to the window."""
        idx = np.asarray(baselines, dtype=np.int64).reshape(-1)
        nt = self.nr_timesteps - time_begin if nr_timesteps is None else nr_timesteps
        t1 = time_begin + nt
        offs = [0] + [o - time_begin for o in self.aterm_offsets.tolist() if time_begin < o < t1] + [nt]
        return dataclasses.replace(
            self, name=f"{self.name}[bl{idx.tolist()},t{time_begin}+{nt}]",
            baselines=np.ascontiguousarray(self.baselines[idx]),
            uvw=np.ascontiguousarray(self.uvw[idx, time_begin:t1]),
            aterm_offsets=np.asarray(offs, dtype=np.int32))

    def longest_baselines(self, k: int) -> np.ndarray:
        """Indices of the k baselines reaching the largest |u|, |v| (the outer grid: |u| L near N/2)."""
        r = np.max(np.abs(self.uvw[:, :, :2]), axis=(1, 2))
        return np.sort(np.argsort(r)[::-1][:k])


# ----------------------------------------------------------------------------------------------
# station layouts (ENU metres)
# ----------------------------------------------------------------------------------------------

def _layout_square(rng, n, side):
    e = rng.uniform(-side / 2, side / 2, n)
    nn = rng.uniform(-side / 2, side / 2, n)
    return np.stack([e, nn, np.zeros(n)], axis=1)


def _layout_lofar(rng, n_core=24, n_remote=20, core_radius=1000.0, rmin=3000.0, rmax=60000.0):
    r = core_radius * np.sqrt(rng.uniform(0, 1, n_core))
    th = rng.uniform(0, 2 * np.pi, n_core)
    core = np.stack([r * np.cos(th), r * np.sin(th)], axis=1)
    rr = np.exp(rng.uniform(np.log(rmin), np.log(rmax), n_remote))
    th = rng.uniform(0, 2 * np.pi, n_remote)
    remote = np.stack([rr * np.cos(th), rr * np.sin(th)], axis=1)
    en = np.concatenate([core, remote])
    return np.concatenate([en, np.zeros((en.shape[0], 1))], axis=1)


def _layout_spiral(rng, n, core_fraction=0.5, core_radius=500.0, rmin=600.0, rmax=35000.0, arms=3):
    n_core = int(round(n * core_fraction))
    r = core_radius * np.sqrt(rng.uniform(0, 1, n_core))
    th = rng.uniform(0, 2 * np.pi, n_core)
    pts = [np.stack([r * np.cos(th), r * np.sin(th)], axis=1)]
    n_arm = n - n_core
    per_arm = [n_arm // arms + (1 if a < n_arm % arms else 0) for a in range(arms)]
    for a, k in enumerate(per_arm):
        rr = np.exp(np.linspace(np.log(rmin), np.log(rmax), k)) * rng.uniform(0.95, 1.05, k)
        th = a * 2 * np.pi / arms + 1.2 * np.log(rr / rmin) + rng.normal(0, 0.03, k)
        pts.append(np.stack([rr * np.cos(th), rr * np.sin(th)], axis=1))
    en = np.concatenate(pts)
    return np.concatenate([en, np.zeros((en.shape[0], 1))], axis=1)


def _enu_to_xyz(enu, lat):
    e, n, u = enu[:, 0], enu[:, 1], enu[:, 2]
    sl, cl = math.sin(lat), math.cos(lat)
    return np.stack([-sl * n + cl * u, e, cl * n + sl * u], axis=1)


def baselines_for(nr_stations: int) -> np.ndarray:
    """All station pairs p<q, lexicographic, no autocorrelations (150 stations -> 11,175)."""
    p, q = np.triu_indices(nr_stations, k=1)
    return np.stack([p, q], axis=1).astype(np.int32)


def earth_rotation_uvw(xyz, baselines, nr_timesteps, dt, dec):
    """uvw [nbl][T][3] metres for baseline vector b = xyz[q] - xyz[p] over hour angles centred on transit."""
    b = xyz[baselines[:, 1]] - xyz[baselines[:, 0]]           # [nbl][3]
    H = (np.arange(nr_timesteps) - nr_timesteps / 2) * dt * SIDEREAL_RATE
    sH, cH = np.sin(H)[None, :], np.cos(H)[None, :]
    X, Y, Z = b[:, 0:1], b[:, 1:2], b[:, 2:3]
    sd, cd = math.sin(dec), math.cos(dec)
    u = sH * X + cH * Y
    v = -sd * cH * X + sd * sH * Y + cd * Z
    w = cd * cH * X - cd * sH * Y + sd * Z
    return np.stack([u, v, w], axis=2).astype(np.float32)


MAX_IMAGE_SIZE = 0.3


def image_size_for(uvw, frequencies, grid_size, subgrid_size):
    """L = (N/2 - N~) / max|u_lambda, v_lambda| so that no subgrid falls off the grid,
    capped at 0.3 (a ~17 degree field) so that small station subsets still image a physical sky."""
    umax = float(np.max(np.abs(uvw[:, :, :2]).astype(np.float64))) * float(np.max(frequencies)) / SPEED_OF_LIGHT
    return min(MAX_IMAGE_SIZE, (grid_size / 2 - subgrid_size) / umax)


# ----------------------------------------------------------------------------------------------
# named configs (BASELINE.json configs[0..4]; recipe in SURVEY.md 8(d))
# ----------------------------------------------------------------------------------------------

CONFIGS = {
    # name: (stations layout, nr_stations, lat deg, dec deg, C, f0, df, T, dt, Ns, N, K, Tmax, slot_len, aterms, seed)
    "tiny": dict(layout="square", nr_stations=4, lat=52.91, dec=60.0, C=1, f0=150e6, df=0.0, T=64, dt=30.0,
                 Ns=16, N=256, K=5, Tmax=64, slot=64, aterms="identity", seed=1001),
    "lofar": dict(layout="lofar", nr_stations=44, lat=52.91, dec=60.0, C=16, f0=150e6, df=12.207e3, T=8192,
                  dt=1.0, Ns=24, N=2048, K=7, Tmax=128, slot=256, aterms="identity", seed=1002),
    "lofar_dde": dict(layout="lofar", nr_stations=44, lat=52.91, dec=60.0, C=16, f0=150e6, df=12.207e3, T=8192,
                      dt=1.0, Ns=24, N=2048, K=7, Tmax=128, slot=256, aterms="random", seed=1003, w_offset="half_median"),
    # small parity case with everything switched on (channels, random A-terms, slots, w0, taper)
    "small_dde": dict(layout="lofar", nr_stations=8, lat=52.91, dec=60.0, C=4, f0=150e6, df=195.3e3, T=96,
                      dt=20.0, Ns=16, N=256, K=5, Tmax=24, slot=40, aterms="random", seed=1010,
                      w_offset="half_median"),
    # short-item stress variant of configs[1] (not a BASELINE config): 8 s integration over 18 h on an 8192^2
    # grid, so the uv tracks cross subgrids ~16x faster per time step -- mean T~ 46, median 24 (P:254:
    # "performance is data dependent")
    "lofar_short": dict(layout="lofar", nr_stations=44, lat=52.91, dec=60.0, C=16, f0=150e6, df=12.207e3, T=8192,
                        dt=8.0, Ns=24, N=8192, K=7, Tmax=128, slot=256, aterms="identity", seed=1006),
    "ska": dict(layout="spiral", nr_stations=150, lat=-26.82, dec=-30.0, C=32, f0=140e6, df=24.414e3, T=8192,
                dt=1.0, Ns=32, N=8192, K=9, Tmax=128, slot=256, aterms="identity", seed=1004),
    "predict": dict(layout="spiral_ext", nr_stations=512, lat=-26.82, dec=-30.0, C=16, f0=140e6, df=24.414e3,
                    T=1024, dt=1.0, Ns=32, N=8192, K=9, Tmax=128, slot=256, aterms="identity", seed=1005),
}


def make_observation(name: str, **overrides) -> Observation:
    """Build config `name`; `overrides` replace recipe entries (T, nr_stations, C, Ns, N, K, Tmax, slot,
    aterms, dt, w_offset, seed, ...) -- same recipe, same seed unless overridden."""
    cfg = dict(CONFIGS[name])
    for k, v in overrides.items():
        if k not in cfg and k not in ("w_offset", "C_block", "w_planes", "channels"):
            raise KeyError(k)
        cfg[k] = v
    rng = np.random.default_rng(cfg["seed"])
    S = cfg["nr_stations"]
    lay = cfg["layout"]
    if lay == "square":
        enu = _layout_square(rng, S, 1000.0)
    elif lay == "lofar":
        n_core = min(24, S)
        enu = _layout_lofar(rng, n_core=n_core, n_remote=S - n_core)
    elif lay == "spiral":
        enu = _layout_spiral(rng, S)
    elif lay == "spiral_ext":
        enu = _layout_spiral(rng, S, core_radius=1000.0, rmax=50000.0)
    else:
        raise ValueError(lay)
    xyz = _enu_to_xyz(enu, math.radians(cfg["lat"]))
    bl = baselines_for(S)
    T = cfg["T"]
    uvw = earth_rotation_uvw(xyz, bl, T, cfg["dt"], math.radians(cfg["dec"]))
    freqs = cfg["f0"] + cfg["df"] * np.arange(cfg["C"], dtype=np.float64)
    if cfg.get("channels", "uniform") == "gap_jitter":
        # a real channel table: one channel missing (flagged / split band) and +-1 kHz jitter, so the
        # spacing is not uniform and the kernels that rotate phasors across channels may not be used
        full = cfg["f0"] + cfg["df"] * np.arange(cfg["C"] + 1, dtype=np.float64)
        full = np.delete(full, (cfg["C"] + 1) // 3)
        jit = np.random.default_rng(cfg["seed"] + 17).uniform(-1e3, 1e3, cfg["C"])
        freqs = full + jit
    L = image_size_for(uvw, freqs, cfg["N"], cfg["Ns"])
    slot = cfg["slot"]
    offs = np.asarray(list(range(0, T, slot)) + [T], dtype=np.int32)
    w0 = cfg.get("w_offset", 0.0)
    if w0 == "half_median":
        w0 = 0.5 * float(np.median(np.abs(uvw[:, :, 2]))) * float(freqs[0]) / SPEED_OF_LIGHT
    nz, w_step = int(cfg.get("w_planes", 1)), 0.0
    if nz > 1:   # planes spanning the |w| range of the observation at the middle frequency
        wmax = float(np.max(np.abs(uvw[:, :, 2]))) * float(freqs[len(freqs) // 2]) / SPEED_OF_LIGHT
        w_step = 2.0 * wmax / nz
    return Observation(name=name, nr_stations=S, baselines=bl, uvw=uvw, frequencies=freqs,
                       aterm_offsets=offs, subgrid_size=cfg["Ns"], grid_size=cfg["N"], image_size=L,
                       kernel_size=cfg["K"], max_timesteps_per_subgrid=cfg["Tmax"],
                       max_channels_per_subgrid=int(cfg.get("C_block", 0)), w_offset=float(w0),
                       nr_w_planes=nz, w_step=w_step, seed=cfg["seed"], aterm_kind=cfg["aterms"])


# ----------------------------------------------------------------------------------------------
# A-terms, taper, visibilities, grids
# ----------------------------------------------------------------------------------------------

def make_aterms(obs: Observation, kind: str | None = None, seed_offset: int = 7) -> np.ndarray:
    """complex64 [slots][S][N~][N~][4]; identity, or smooth random per-station Jones."""
    kind = obs.aterm_kind if kind is None else kind
    n, S, ns = obs.subgrid_size, obs.nr_stations, obs.nr_aterm_slots
    a = np.zeros((ns, S, n, n, 4), dtype=np.complex64)
    if kind == "identity":
        a[..., 0] = 1
        a[..., 3] = 1
        return a
    rng = np.random.default_rng(obs.seed + seed_offset)
    x = (np.arange(n) - n / 2) / (n / 2)
    lp, mp = np.meshgrid(x, x)                  # [y][x]: l varies with x, m with y
    basis = np.stack([np.ones_like(lp), lp, mp, lp * mp, lp * lp, mp * mp])   # [6][n][n]
    coef = (rng.standard_normal((ns, S, 6, 4)) + 1j * rng.standard_normal((ns, S, 6, 4))) * 0.1
    gain = np.exp(1j * rng.uniform(0, 2 * np.pi, (ns, S))) * rng.uniform(0.8, 1.2, (ns, S))
    pert = np.einsum("bskp,kyx->bsyxp", coef, basis)
    ident = np.array([1, 0, 0, 1], dtype=np.complex128)
    a[:] = (gain[:, :, None, None, None] * (ident + pert)).astype(np.complex64)
    return a


def _grdsf(nu: np.ndarray) -> np.ndarray:
    """Schwab (1984) rational approximation of the prolate spheroidal wave function (m=6, alpha=1)."""
    P = np.array([[8.203343e-2, -3.644705e-1, 6.278660e-1, -5.335581e-1, 2.312756e-1],
                  [4.028559e-3, -3.697768e-2, 1.021332e-1, -1.201436e-1, 6.412774e-2]])
    Q = np.array([[1.0, 8.212018e-1, 2.078043e-1],
                  [1.0, 9.599102e-1, 2.918724e-1]])
    nu = np.abs(np.asarray(nu, dtype=np.float64))
    part = (nu >= 0.75).astype(int)
    nuend = np.where(part == 0, 0.75, 1.0)
    d = nu * nu - nuend * nuend
    top = sum(P[part, k] * d ** k for k in range(5))
    bot = sum(Q[part, k] * d ** k for k in range(3))
    return np.where(nu <= 1.0, top / bot, 0.0)


def make_taper(subgrid_size: int, kind: str = "spheroidal") -> np.ndarray:
    """float32 [N~][N~] = taper[y][x], the image-domain taper (the 'spheroidal'); separable,
    positive, peak 1.  kind="asymmetric" tilts it along x only (s(y) s(x) (1 + 0.2 x')), so that a
    [y][x] <-> [x][y] slip anywhere (oracle or kernels) changes the result."""
    n = subgrid_size
    if kind == "ones":
        return np.ones((n, n), dtype=np.float32)
    nu = np.abs(np.arange(n) - n / 2) / (n / 2 + 1)
    s = _grdsf(nu) * (1 - nu * nu)
    s = s / s.max()
    if kind == "asymmetric":
        xx = (np.arange(n) - n / 2) / (n / 2)
        return np.outer(s, s * (1 + 0.2 * xx)).astype(np.float32)
    if kind != "spheroidal":
        raise ValueError(kind)
    return np.outer(s, s).astype(np.float32)


def make_visibilities(obs: Observation, seed_offset: int = 11) -> np.ndarray:
    """complex64 [nbl][T][C][4], complex Gaussian (values do not affect run time; uvw does)."""
    rng = np.random.default_rng(obs.seed + seed_offset)
    shape = (obs.nr_baselines, obs.nr_timesteps, obs.nr_channels, 4)
    v = np.empty(shape, dtype=np.complex64)
    f = v.view(np.float32)
    f[...] = rng.standard_normal(f.shape, dtype=np.float32) * np.float32(math.sqrt(0.5))
    return v


def make_grid(obs: Observation, seed_offset: int = 13) -> np.ndarray:
    """complex64 [4][N][N] (or [nz][4][N][N] with W-stacking) random model grid (degridding input)."""
    rng = np.random.default_rng(obs.seed + seed_offset)
    N = obs.grid_size
    shape = (4, N, N) if obs.nr_w_planes <= 1 else (obs.nr_w_planes, 4, N, N)
    g = np.empty(shape, dtype=np.complex64)
    f = g.view(np.float32)
    f[...] = rng.standard_normal(f.shape, dtype=np.float32) * np.float32(math.sqrt(0.5))
    return g


def torch_visibilities(obs: Observation, device, seed_offset: int = 11):
    """Same distribution as make_visibilities, drawn on `device` with a seeded torch generator (bench)."""
    import torch
    g = torch.Generator(device=device)
    g.manual_seed(obs.seed + seed_offset)
    n = obs.nr_visibilities * 4 * 2
    f = torch.empty(n, device=device, dtype=torch.float32)
    f.normal_(0.0, math.sqrt(0.5), generator=g)           # in place: no temporaries at 94 GB sizes
    return f.view(torch.complex64).view(obs.nr_baselines, obs.nr_timesteps, obs.nr_channels, 4)


def torch_grid(obs: Observation, device, seed_offset: int = 13):
    import torch
    g = torch.Generator(device=device)
    g.manual_seed(obs.seed + seed_offset)
    N = obs.grid_size
    f = torch.empty(4 * N * N * 2, device=device, dtype=torch.float32)
    f.normal_(0.0, math.sqrt(0.5), generator=g)
    return f.view(torch.complex64).view(4, N, N)
