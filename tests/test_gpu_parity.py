"""GPU parity: the sm_100a path (through the C ABI) against the fp64 oracle, element by element.

Bar (BASELINE.json north_star): relative RMS error ||x - x_oracle||_2 / ||x_oracle||_2 <= 1e-4 on grids
(all cells x pols) and on visibilities (all visibilities x pols); the plan is bit-exact (test_abi_plan).
Sizes span several work items, ragged channel blocks, every subgrid size (16/24/32) and both grid sizes
of the configs; full-size configs are checked on sampled work items (the oracle computes them one by
one) and through the adjoint identity, which holds at any size.
"""
import numpy as np
import pytest

import idgsynth
import oracle

torch = pytest.importorskip("torch")
import paper_conf_ipps_veenboerpr17_b200 as idg

pytestmark = pytest.mark.gpu
TOL = 1e-4


def rel_rms(x, ref):
    x = np.asarray(x).astype(np.complex128).reshape(-1)
    ref = np.asarray(ref).astype(np.complex128).reshape(-1)
    return float(np.linalg.norm(x - ref) / np.linalg.norm(ref))


def _inputs(obs, aterm_kind=None, taper_kind="spheroidal"):
    vis = idgsynth.make_visibilities(obs)
    aterms = idgsynth.make_aterms(obs, aterm_kind)
    taper = idgsynth.make_taper(obs.subgrid_size, taper_kind)
    return vis, aterms, taper


def _dev(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


def gpu_grid(obs, vis, aterms, taper, plan=None):
    plan = plan or idg.Plan.from_observation(obs)
    g = torch.zeros(oracle.grid_shape(obs), dtype=torch.complex64, device="cuda")
    idg.grid(plan, _dev(vis), _dev(obs.uvw), _dev(aterms), _dev(taper), g)
    torch.cuda.synchronize()
    return g


def gpu_degrid(obs, grid_np_or_t, aterms, taper, plan=None):
    plan = plan or idg.Plan.from_observation(obs)
    g = grid_np_or_t if isinstance(grid_np_or_t, torch.Tensor) else _dev(grid_np_or_t)
    v = torch.full((obs.nr_baselines, obs.nr_timesteps, obs.nr_channels, 4), complex(7, 7),
                   dtype=torch.complex64, device="cuda")
    idg.degrid(plan, g, _dev(obs.uvw), _dev(aterms), _dev(taper), v)
    torch.cuda.synchronize()
    return v


CASES = [
    ("tiny", {}, "identity", "ones"),
    ("tiny", {}, "identity", "asymmetric"),
    ("small_dde", {}, None, "asymmetric"),
    ("small_dde", dict(C=7, C_block=3), None, "spheroidal"),          # ragged channel blocks
    ("small_dde", dict(C=12), None, "spheroidal"),                   # 12 channels: V=4 degridder
    ("small_dde", dict(C=8), None, "asymmetric"),                    # 8 channels: rot8 degridder
    ("lofar", dict(T=640, nr_stations=5), None, "asymmetric"),       # N~=24, N=2048, 16 ch
    ("lofar_dde", dict(T=512, nr_stations=5), None, "spheroidal"),   # + random A-terms, w0
    ("ska", dict(T=384, nr_stations=4), None, "asymmetric"),         # N~=32, N=8192, 32 ch
    ("predict", dict(T=256, nr_stations=4), None, "asymmetric"),     # N~=32, 16 ch
    ("predict", dict(T=256, nr_stations=4, C=8), None, "spheroidal"),  # N~=32, 8 ch: one k-block/timestep
    ("small_dde", dict(C=24, C_block=8), None, "spheroidal"),       # 3 channel blocks of 8
    ("small_dde", dict(w_planes=4), None, "asymmetric"),            # W-stacking (NEXT-1, R-21)
    ("lofar_dde", dict(T=512, nr_stations=5, w_planes=3), None, "spheroidal"),
    ("small_dde", dict(C=64), None, "spheroidal"),                   # 2 blocks of 32 channels per timestep
    ("small_dde", dict(C=40, C_block=24), None, "spheroidal"),      # 24 + 16 channels: mixed item widths
    ("lofar", dict(T=256, nr_stations=5, channels="gap_jitter"), None, "asymmetric"),  # real channel table
    ("tiny", dict(T=1), "identity", "asymmetric"),                   # degenerate: one timestep, one channel
    ("small_dde", dict(nr_stations=2), None, "asymmetric"),          # degenerate: a single baseline
    ("small_dde", dict(T=1, C=1), None, "spheroidal"),              # one visibility per baseline
]


KINDS = {
    "default": (None, None),   # default: rotation kernels where the channel layout allows, else direct
    "tc": ("tc", "tc"),        # direct tensor-core kernels (one sincos per pair, any channel table)
    "simt": ("simt", "simt"),  # CUDA-core kernels (the paper's structure)
    "umma": ("gridder_umma_rot<*", ""),  # tcgen05 / TMEM rotation gridder, cluster pair (N~ = 32, 16 / 32 ch)
    "fx16": ("", "degridder_rot16<*"),  # 16-row degridders with the f16 fixed-point split (default: integer form)
}


@pytest.fixture(params=list(KINDS))
def kind(request, monkeypatch):
    """Kernel family under test (the variant environment overrides of include/idg.h).  Families a
    case is not eligible for (e.g. tensor-core gridders need C~ % 8 == 0) fall back to the default."""
    g, d = KINDS[request.param]
    if g or d:
        monkeypatch.setenv("IDG_GRIDDER_VARIANT", g)
        monkeypatch.setenv("IDG_DEGRIDDER_VARIANT", d)
    return request.param


@pytest.mark.parametrize("name,kw,aterm,taper", CASES)
def test_grid_matches_oracle(name, kw, aterm, taper, kind):
    obs = idgsynth.make_observation(name, **kw)
    vis, aterms, tap = _inputs(obs, aterm, taper)
    items, _ = oracle.plan(obs)
    ref = oracle.grid(obs, items, vis, aterms, tap)
    got = gpu_grid(obs, vis, aterms, tap).cpu().numpy()
    err = rel_rms(got, ref)
    print(f"grid[{kind}] {name} {kw}: rel rms {err:.3e}")
    assert err <= TOL, err


@pytest.mark.parametrize("name,kw,aterm,taper", CASES)
def test_degrid_matches_oracle(name, kw, aterm, taper, kind):
    obs = idgsynth.make_observation(name, **kw)
    _, aterms, tap = _inputs(obs, aterm, taper)
    G = idgsynth.make_grid(obs)
    items, dropped = oracle.plan(obs)
    ref = oracle.scatter_visibilities(obs, items, oracle.degrid(obs, items, G, aterms, tap))
    got = gpu_degrid(obs, G, aterms, tap).cpu().numpy()
    err = rel_rms(got, ref)
    print(f"degrid[{kind}] {name} {kw}: rel rms {err:.3e}")
    assert err <= TOL, err


def test_grid_accumulates_and_degrid_zeroes_dropped(kind):
    import dataclasses
    obs = idgsynth.make_observation("small_dde")
    obs = dataclasses.replace(obs, image_size=obs.image_size * 6)     # long baselines fall off the grid
    vis, aterms, tap = _inputs(obs)
    items, dropped = oracle.plan(obs)
    assert dropped > 0
    plan = idg.Plan.from_observation(obs)
    g = gpu_grid(obs, vis, aterms, tap, plan)
    idg.grid(plan, _dev(vis), _dev(obs.uvw), _dev(aterms), _dev(tap), g)    # second call accumulates
    ref = 2 * oracle.grid(obs, items, vis, aterms, tap)
    assert rel_rms(g.cpu().numpy(), ref) <= TOL
    G = idgsynth.make_grid(obs)
    got = gpu_degrid(obs, G, aterms, tap, plan).cpu().numpy()
    ref = oracle.scatter_visibilities(obs, items, oracle.degrid(obs, items, G, aterms, tap))
    assert rel_rms(got, ref) <= TOL
    covered = oracle.scatter_visibilities(obs, items, np.ones(int(np.sum(
        items["nr_timesteps"] * (items["channel_end"] - items["channel_begin"]))) * 4))
    assert np.all(got[covered == 0] == 0)                              # dropped -> exactly 0


def _inner_t(a, b, chunk=1 << 26):
    """sum conj(a) b in complex128, in chunks (the full-size arrays are up to 94 GB)."""
    a, b = a.reshape(-1), b.reshape(-1)
    acc = 0j
    for i in range(0, a.numel(), chunk):
        acc += torch.vdot(a[i:i + chunk].to(torch.complex128), b[i:i + chunk].to(torch.complex128)).item()
    return acc


@pytest.mark.parametrize("name", ["lofar_dde", "lofar"])
def test_full_size_adjoint_and_sampled_items(name, kind):
    """Full LOFAR-shaped set in the bench launch configuration: <degrid(G),V> = <G,grid(V)> on the GPU,
    and degridded visibilities of sampled work items against the oracle computing just those items."""
    obs = idgsynth.make_observation(name)
    aterms = idgsynth.make_aterms(obs)
    tap = idgsynth.make_taper(obs.subgrid_size)
    plan = idg.Plan.from_observation(obs)
    uvw, at, tp = _dev(obs.uvw), _dev(aterms), _dev(tap)
    V = idgsynth.torch_visibilities(obs, "cuda")
    G = idgsynth.torch_grid(obs, "cuda")
    gV = torch.zeros_like(G)
    idg.grid(plan, V, uvw, at, tp, gV)
    DG = torch.empty_like(V)
    idg.degrid(plan, G, uvw, at, tp, DG)
    torch.cuda.synchronize()
    lhs, rhs = _inner_t(DG, V), _inner_t(G, gV)
    assert abs(lhs - rhs) / abs(lhs) < 1e-4, (lhs, rhs)
    # sampled items through the oracle
    items, _ = oracle.plan(obs)
    rng = np.random.default_rng(0)
    sel = items[np.sort(rng.choice(len(items), 24, replace=False))]
    Gh = G.cpu().numpy()
    ref = oracle.degrid(obs, sel, Gh, aterms, tap)
    got = oracle.gather_visibilities(obs, sel, DG.cpu().numpy())
    assert rel_rms(got, ref) <= TOL


@pytest.mark.parametrize("name,kw,chunk,drop", [("small_dde", {}, 60000, False),
                                                ("lofar", dict(T=640, nr_stations=6), 300000, False),
                                                ("small_dde", dict(C=7, C_block=3), 40000, False),
                                                ("small_dde", dict(w_planes=3), 60000, False),
                                                ("small_dde", {}, 50000, True)])
def test_host_streamed_calls(name, kw, chunk, drop, monkeypatch):
    """idg_grid_host / idg_degrid_host (work groups through triple-buffered staging) against the
    oracle, and against the device-resident calls (degridding bit-identical).  drop: long baselines fall
    off the grid, so some work groups hold dropped runs (zeroed on the device) or no items at all."""
    import dataclasses
    monkeypatch.setenv("IDG_HOST_CHUNK_BYTES", str(chunk))     # several work groups even at small sizes
    obs = idgsynth.make_observation(name, **kw)
    if drop:
        obs = dataclasses.replace(obs, image_size=obs.image_size * 6)
    vis, aterms, tap = _inputs(obs, None, "asymmetric")
    items, dropped = oracle.plan(obs)
    assert (dropped > 0) == drop
    plan = idg.Plan.from_observation(obs)
    ws = idg.workspace(plan)
    uvw, at, tp = _dev(obs.uvw), _dev(aterms), _dev(tap)
    vis_h = torch.from_numpy(vis).pin_memory()
    g_host = torch.zeros(oracle.grid_shape(obs), dtype=torch.complex64, device="cuda")
    idg.grid_host(plan, vis_h, uvw, at, tp, g_host, ws)
    idg.grid_host(plan, vis_h, uvw, at, tp, g_host, ws)      # accumulates, buffers reused across calls
    torch.cuda.synchronize()
    ref = 2 * oracle.grid(obs, items, vis, aterms, tap)
    assert rel_rms(g_host.cpu().numpy(), ref) <= TOL
    G = idgsynth.make_grid(obs)
    refv = oracle.scatter_visibilities(obs, items, oracle.degrid(obs, items, G, aterms, tap))
    Gd = _dev(G)
    v_host = torch.full((obs.nr_baselines, obs.nr_timesteps, obs.nr_channels, 4), complex(3, 3),
                        dtype=torch.complex64).pin_memory()
    idg.degrid_host(plan, Gd, uvw, at, tp, v_host, ws)
    torch.cuda.synchronize()
    assert rel_rms(v_host.numpy(), refv) <= TOL
    if drop:
        assert np.all(v_host.numpy()[refv == 0] == 0)          # dropped -> exactly 0
    v_dev = gpu_degrid(obs, G, aterms, tap, plan)
    assert torch.equal(v_host, v_dev.cpu())


@pytest.mark.parametrize("name,kw,chunk,drop", [("small_dde", {}, 50000, False),
                                                ("small_dde", dict(w_planes=3), 60000, False),
                                                ("lofar", dict(T=640, nr_stations=6), 300000, False),
                                                ("ska", dict(T=256, nr_stations=4), 2000000, False),
                                                ("small_dde", {}, 50000, True)])
def test_host_adder_and_splitter(name, kw, chunk, drop, monkeypatch):
    """The grid in host memory (option 2): subgrids stream to / from the host and host threads add
    them into / split them out of the grid.  Against the oracle, and degridding bit-identical to the
    device-resident call (same kernels, same subgrids)."""
    import dataclasses
    monkeypatch.setenv("IDG_HOST_CHUNK_BYTES", str(chunk))     # several work groups
    monkeypatch.setenv("IDG_HOST_THREADS", "5")                # rows interleaved over an odd thread count
    obs = idgsynth.make_observation(name, **kw)
    if drop:
        obs = dataclasses.replace(obs, image_size=obs.image_size * 6)
    vis, aterms, tap = _inputs(obs, None, "asymmetric")
    items, dropped = oracle.plan(obs)
    assert (dropped > 0) == drop
    plan = idg.Plan.from_observation(obs)
    ws = idg.adder_workspace(plan, buffers=4)
    uvw, at, tp = _dev(obs.uvw), _dev(aterms), _dev(tap)
    vis_h = torch.from_numpy(vis).pin_memory()
    g_host = torch.zeros(oracle.grid_shape(obs), dtype=torch.complex64)
    idg.grid_host_adder(plan, vis_h, uvw, at, tp, g_host, ws)
    idg.grid_host_adder(plan, vis_h, uvw, at, tp, g_host, ws)      # accumulates
    ref = 2 * oracle.grid(obs, items, vis, aterms, tap)
    err = rel_rms(g_host.numpy(), ref)
    print(f"host adder {name} {kw}: rel rms {err:.3e}")
    assert err <= TOL, err
    G = idgsynth.make_grid(obs)
    refv = oracle.scatter_visibilities(obs, items, oracle.degrid(obs, items, G, aterms, tap))
    v_host = torch.full((obs.nr_baselines, obs.nr_timesteps, obs.nr_channels, 4), complex(3, 3),
                        dtype=torch.complex64).pin_memory()
    idg.degrid_host_splitter(plan, torch.from_numpy(G), uvw, at, tp, v_host, ws)
    torch.cuda.synchronize()
    assert rel_rms(v_host.numpy(), refv) <= TOL
    v_dev = gpu_degrid(obs, G, aterms, tap, plan)
    assert torch.equal(v_host, v_dev.cpu())


@pytest.mark.parametrize("name,kw", [("ska", dict(T=256, nr_stations=4)), ("predict", dict(T=128, nr_stations=4))])
def test_host_adder_tcgen05_gridder(name, kw, monkeypatch):
    """The cluster-pair tcgen05 gridder writes its two polarisation halves into the host adder's subgrid
    buffer (slot = the item's position in the order, not the CTA index)."""
    monkeypatch.setenv("IDG_HOST_CHUNK_BYTES", "2000000")
    monkeypatch.setenv("IDG_GRIDDER_VARIANT", "gridder_umma_rot<*")
    obs = idgsynth.make_observation(name, **kw)
    vis, aterms, tap = _inputs(obs, "random", "asymmetric")
    items, _ = oracle.plan(obs)
    plan = idg.Plan.from_observation(obs)
    ws = idg.adder_workspace(plan, buffers=3)
    g_host = torch.zeros(oracle.grid_shape(obs), dtype=torch.complex64)
    idg.grid_host_adder(plan, torch.from_numpy(vis).pin_memory(), _dev(obs.uvw), _dev(aterms), _dev(tap),
                        g_host, ws)
    assert idg.last_variant("gridder").startswith("gridder_umma_rot<")
    err = rel_rms(g_host.numpy(), oracle.grid(obs, items, vis, aterms, tap))
    print(f"host adder [umma] {name} {kw}: rel rms {err:.3e}")
    assert err <= TOL, err


def test_host_streamed_upload_waits_for_the_callers_stream():
    """A non-blocking device->host copy into vis_h queued on the caller's stream right before
    idg_grid_host (no synchronize in between): the uploads must see the new host data."""
    obs = idgsynth.make_observation("small_dde")
    vis, aterms, tap = _inputs(obs, None, "asymmetric")
    plan = idg.Plan.from_observation(obs)
    ws = idg.workspace(plan)
    uvw, at, tp = _dev(obs.uvw), _dev(aterms), _dev(tap)
    items, _ = oracle.plan(obs)
    ref = oracle.grid(obs, items, vis, aterms, tap)
    s = torch.cuda.Stream()
    vis_d = _dev(vis)
    for _ in range(3):
        vis_h = torch.zeros(vis.shape, dtype=torch.complex64).pin_memory()
        g = torch.zeros(oracle.grid_shape(obs), dtype=torch.complex64, device="cuda")
        with torch.cuda.stream(s):
            torch.cuda._sleep(50_000_000)                    # keep the stream busy: the copy lands late
            vis_h.copy_(vis_d, non_blocking=True)
            idg.grid_host(plan, vis_h, uvw, at, tp, g, ws, stream=s)
        s.synchronize()
        assert rel_rms(g.cpu().numpy(), ref) <= TOL


@pytest.mark.slow
@pytest.mark.parametrize("name", ["ska", "predict"])
def test_full_size_configs_sampled(name):
    """The SKA-low-shaped (N=8192, N~=32, C=32, T=8192: 2.9e9 visibilities, 94 GB) and predict-shaped
    (512 stations, N=8192: 2.1e9 visibilities) configs at full size in the bench launch configuration:
    degridded visibilities of sampled work items against the oracle, and the grid <-> degrid adjoint
    identity (on the full set when two visibility arrays fit in HBM, else on the first half of time)."""
    obs = idgsynth.make_observation(name)
    aterms = idgsynth.make_aterms(obs)
    tap = idgsynth.make_taper(obs.subgrid_size)
    plan = idg.Plan.from_observation(obs)
    assert plan.stats()["nr_vis_dropped"] == 0
    uvw, at, tp = _dev(obs.uvw), _dev(aterms), _dev(tap)
    G = idgsynth.torch_grid(obs, "cuda")
    DG = torch.empty((obs.nr_baselines, obs.nr_timesteps, obs.nr_channels, 4), dtype=torch.complex64,
                     device="cuda")
    idg.degrid(plan, G, uvw, at, tp, DG)
    torch.cuda.synchronize()
    items = plan.metadata()
    rng = np.random.default_rng(1)
    sel = np.asarray(items[np.sort(rng.choice(len(items), 16, replace=False))]).astype(oracle.ITEM_DTYPE)
    ref = oracle.degrid(obs, sel, G.cpu().numpy(), aterms, tap)
    got = np.concatenate([DG[int(it["baseline"]), int(it["time_offset"]):int(it["time_offset"]) + int(it["nr_timesteps"]),
                             int(it["channel_begin"]):int(it["channel_end"])].cpu().numpy().reshape(-1) for it in sel])
    assert rel_rms(got, ref) <= TOL
    free, _ = torch.cuda.mem_get_info()
    if free < obs.nr_visibilities * 32 + (8 << 30):           # second full array does not fit: half of time
        del DG
        torch.cuda.empty_cache()
        obs = obs.subset(nr_timesteps=obs.nr_timesteps // 2)
        plan = idg.Plan.from_observation(obs)
        uvw = _dev(obs.uvw)
        DG = torch.empty((obs.nr_baselines, obs.nr_timesteps, obs.nr_channels, 4), dtype=torch.complex64,
                         device="cuda")
        idg.degrid(plan, G, uvw, at[: obs.nr_aterm_slots], tp, DG)
    V = idgsynth.torch_visibilities(obs, "cuda")
    gV = torch.zeros_like(G)
    idg.grid(plan, V, uvw, at[: obs.nr_aterm_slots], tp, gV)
    torch.cuda.synchronize()
    lhs, rhs = _inner_t(DG, V), _inner_t(G, gV)
    assert abs(lhs - rhs) / abs(lhs) < 1e-4, (lhs, rhs)


# ------------------------------------------------------------------------------------------------
# the full-size uv regime: long baselines of the FULL observations (same L, N, channels), so the
# subgrids sit near the grid edge (|u| L > 90 % of N/2) where fp32 phase formation is hardest
# ------------------------------------------------------------------------------------------------
_FULL = {}


def _full_obs(name):
    if name not in _FULL:
        _FULL[name] = idgsynth.make_observation(name)
    return _FULL[name]


# (config, longest baselines, time window): windows where the longest tracks reach their extreme |u|
FULL_L = [("lofar", 4, 0), ("ska", 3, 3072), ("predict", 3, 0)]


def _full_l_subset(name, k, t0):
    full = _full_obs(name)
    obs = full.select(full.longest_baselines(k), nr_timesteps=1024, time_begin=t0)
    assert obs.image_size == full.image_size
    f = obs.frequencies.max() / idgsynth.SPEED_OF_LIGHT
    reach = float(np.abs(obs.uvw[:, :, :2]).max()) * f * obs.image_size / (obs.grid_size / 2)
    assert reach > 0.9, reach            # the subset exercises the outer grid
    return obs


def _window(items, n, N):
    """Grid rows / columns [y0, y1) x [x0, x1) the items cover (the GPU grid is 0 elsewhere)."""
    return (int(items["y"].min()), int(items["y"].max()) + n, int(items["x"].min()), int(items["x"].max()) + n)


@pytest.mark.parametrize("name,k,t0", FULL_L)
def test_grid_full_l_subset_matches_oracle(name, k, t0, kind):
    obs = _full_l_subset(name, k, t0)
    vis = idgsynth.make_visibilities(obs)
    aterms = idgsynth.make_aterms(obs, "random")
    tap = idgsynth.make_taper(obs.subgrid_size, "asymmetric")
    items, dropped = oracle.plan(obs)
    assert dropped == 0
    ref = oracle.grid(obs, items, vis, aterms, tap)
    got = gpu_grid(obs, vis, aterms, tap)
    y0, y1, x0, x1 = _window(items, obs.subgrid_size, obs.grid_size)
    win = got[..., y0:y1, x0:x1]
    assert abs(float(torch.linalg.vector_norm(got)) - float(torch.linalg.vector_norm(win))) <= 1e-6 * float(
        torch.linalg.vector_norm(win))
    err = rel_rms(win.cpu().numpy(), ref[..., y0:y1, x0:x1])
    print(f"grid[{kind}] full-L {name}: {len(items)} items, rel rms {err:.3e}")
    assert err <= TOL, err


@pytest.mark.parametrize("name,k,t0", FULL_L)
def test_degrid_full_l_subset_matches_oracle(name, k, t0, kind):
    obs = _full_l_subset(name, k, t0)
    aterms = idgsynth.make_aterms(obs, "random")
    tap = idgsynth.make_taper(obs.subgrid_size, "asymmetric")
    items, _ = oracle.plan(obs)
    y0, y1, x0, x1 = _window(items, obs.subgrid_size, obs.grid_size)
    G = np.zeros(oracle.grid_shape(obs), dtype=np.complex64)       # random inside the covered window
    rng = np.random.default_rng(obs.seed + 13)
    shape = G[..., y0:y1, x0:x1].shape
    G[..., y0:y1, x0:x1] = (rng.standard_normal(shape) + 1j * rng.standard_normal(shape)) * np.sqrt(0.5)
    ref = oracle.scatter_visibilities(obs, items, oracle.degrid(obs, items, G, aterms, tap))
    got = gpu_degrid(obs, G, aterms, tap).cpu().numpy()
    err = rel_rms(got, ref)
    print(f"degrid[{kind}] full-L {name}: rel rms {err:.3e}")
    assert err <= TOL, err


def test_nonuniform_channels_use_direct_kernels():
    """A real channel table (one channel missing, +-1 kHz jitter): the rotation kernels need uniformly
    spaced channels, so the default dispatch must leave them, and the result still matches the oracle."""
    full = _full_obs("lofar")
    obs = idgsynth.make_observation("lofar", channels="gap_jitter").select(full.longest_baselines(3),
                                                                          nr_timesteps=512)
    assert np.ptp(np.diff(obs.frequencies)) > 1e3
    vis = idgsynth.make_visibilities(obs)
    aterms = idgsynth.make_aterms(obs, "random")
    tap = idgsynth.make_taper(obs.subgrid_size, "asymmetric")
    items, _ = oracle.plan(obs)
    ref = oracle.grid(obs, items, vis, aterms, tap)
    got = gpu_grid(obs, vis, aterms, tap).cpu().numpy()
    assert idg.last_variant("gridder").startswith("gridder_tc<"), idg.last_variant("gridder")
    assert rel_rms(got, ref) <= TOL
    G = idgsynth.make_grid(obs)
    refv = oracle.scatter_visibilities(obs, items, oracle.degrid(obs, items, G, aterms, tap))
    gotv = gpu_degrid(obs, G, aterms, tap).cpu().numpy()
    assert idg.last_variant("degridder").startswith("degridder_tc"), idg.last_variant("degridder")   # tc / tci
    assert rel_rms(gotv, refv) <= TOL


@pytest.mark.parametrize("name,kw", [("lofar", dict(T=640, nr_stations=5)), ("ska", dict(T=384, nr_stations=4))])
def test_small_amplitudes_after_a_zero_batch(name, kw, kind):
    """Visibilities of ~1e-4 (absolute units must not matter) whose first time steps are all zero (flagged):
    the per-batch f16 range scale must not be pinned by the empty batch."""
    obs = idgsynth.make_observation(name, **kw)
    vis = idgsynth.make_visibilities(obs) * np.float32(1e-4)
    vis[:, :200] = 0
    aterms = idgsynth.make_aterms(obs, "random")
    tap = idgsynth.make_taper(obs.subgrid_size, "asymmetric")
    items, _ = oracle.plan(obs)
    ref = oracle.grid(obs, items, vis, aterms, tap)
    err = rel_rms(gpu_grid(obs, vis, aterms, tap).cpu().numpy(), ref)
    print(f"grid[{kind}] small amplitudes {name}: rel rms {err:.3e}")
    assert err <= TOL, err


def test_short_items_match_oracle():
    """Long baselines of the short-item workload (lofar_short: 8 s integration, N = 8192): items of ~9 time
    steps, so most warp units are ragged tails; the default dispatch picks the 8-row degridder for plans
    whose mean T~ is <= 64.  Both directions against the oracle."""
    full = _full_obs("lofar_short")
    obs = full.select(full.longest_baselines(3), nr_timesteps=512, time_begin=2048)
    vis, aterms, tap = _inputs(obs, "random", "asymmetric")
    items, _ = oracle.plan(obs)
    assert float(items["nr_timesteps"].mean()) < 16
    ref = oracle.grid(obs, items, vis, aterms, tap)
    got = gpu_grid(obs, vis, aterms, tap)
    y0, y1, x0, x1 = _window(items, obs.subgrid_size, obs.grid_size)
    assert rel_rms(got[..., y0:y1, x0:x1].cpu().numpy(), ref[..., y0:y1, x0:x1]) <= TOL
    G = np.zeros(oracle.grid_shape(obs), dtype=np.complex64)
    rng = np.random.default_rng(obs.seed + 13)
    shape = G[..., y0:y1, x0:x1].shape
    G[..., y0:y1, x0:x1] = (rng.standard_normal(shape) + 1j * rng.standard_normal(shape)) * np.sqrt(0.5)
    refv = oracle.scatter_visibilities(obs, items, oracle.degrid(obs, items, G, aterms, tap))
    gotv = gpu_degrid(obs, G, aterms, tap).cpu().numpy()
    assert idg.last_variant("degridder").startswith("degridder_rot8"), idg.last_variant("degridder")
    err = rel_rms(gotv, refv)
    print(f"short items: {len(items)} items, mean T~ {items['nr_timesteps'].mean():.1f}, degrid rel rms {err:.3e}")
    assert err <= TOL, err


def test_items_beyond_shared_memory_fall_back():
    """Items of 8192 time steps: the tensor-core degridders stage per-timestep coefficients in shared
    memory (32 B per step) and do not fit; the dispatcher must pick a kernel that does (not fail)."""
    obs = idgsynth.make_observation("tiny", T=8192, dt=0.01, Tmax=8192, slot=8192)
    items, _ = oracle.plan(obs)
    assert int(items["nr_timesteps"].max()) > 7000
    _, aterms, tap = _inputs(obs, "random", "asymmetric")
    G = idgsynth.make_grid(obs)
    ref = oracle.scatter_visibilities(obs, items, oracle.degrid(obs, items, G, aterms, tap))
    got = gpu_degrid(obs, G, aterms, tap).cpu().numpy()
    assert idg.last_variant("degridder").startswith("degridder<"), idg.last_variant("degridder")
    assert rel_rms(got, ref) <= TOL


def test_tolerance_is_discriminating():
    """The 1e-4 bar is tight enough to see small systematic errors: the kernels' own error is far below
    it, while a 2e-5 relative uvw scale error, a one-timestep shift of the visibilities or two swapped
    polarisations -- fed to the same GPU path -- exceed it."""
    obs = idgsynth.make_observation("lofar_dde", T=512, nr_stations=5)
    vis, aterms, taper = _inputs(obs)
    items, _ = oracle.plan(obs)
    ref = oracle.grid(obs, items, vis, aterms, taper)
    plan = idg.Plan.from_observation(obs)
    good = rel_rms(gpu_grid(obs, vis, aterms, taper, plan).cpu().numpy(), ref)
    assert good < TOL / 5, good

    def err_with(uvw=None, v=None):
        g = torch.zeros(oracle.grid_shape(obs), dtype=torch.complex64, device="cuda")
        idg.grid(plan, _dev(vis if v is None else v), _dev(obs.uvw if uvw is None else uvw), _dev(aterms),
                 _dev(taper), g)
        torch.cuda.synchronize()
        return rel_rms(g.cpu().numpy(), ref)

    assert err_with(uvw=(obs.uvw * (1 + 2e-5)).astype(np.float32)) > TOL
    assert err_with(v=np.roll(vis, 1, axis=1)) > TOL
    assert err_with(v=vis[..., [0, 2, 1, 3]]) > TOL


@pytest.mark.parametrize("name,kw", [("small_dde", {}), ("ska", dict(T=128, nr_stations=4))])
def test_degrid_amplitude_scaling(name, kw, kind):
    """The operand forms scale by per-item powers of two, so degrid(2^k G) is exactly 2^k degrid(G)
    (bitwise) for the fixed-point and integer degridders; a zero grid predicts exact zeros; a grid at
    1e-20 or 1e+20 amplitude (no power of two) still matches the oracle to the parity bar."""
    obs = idgsynth.make_observation(name, **kw)
    _, aterms, tap = _inputs(obs, "random", "asymmetric")
    G = idgsynth.make_grid(obs)
    base = gpu_degrid(obs, G, aterms, tap).cpu().numpy()
    for k in (-40, 37):
        got = gpu_degrid(obs, (G * np.float32(2.0 ** k)).astype(np.complex64), aterms, tap).cpu().numpy()
        assert np.array_equal(got, (base * np.float32(2.0 ** k)).astype(np.complex64)), k
    zero = gpu_degrid(obs, np.zeros_like(G), aterms, tap).cpu().numpy()
    assert not np.any(zero)
    items, _ = oracle.plan(obs)
    for s in (1e-20, 1e20):
        Gs = (G * s).astype(np.complex64)
        ref = oracle.scatter_visibilities(obs, items, oracle.degrid(obs, items, Gs, aterms, tap))
        err = rel_rms(gpu_degrid(obs, Gs, aterms, tap).cpu().numpy(), ref)
        print(f"degrid[{kind}] {name} amplitude {s:g}: rel rms {err:.3e}")
        assert err <= TOL, (s, err)
