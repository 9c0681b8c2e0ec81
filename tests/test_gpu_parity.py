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
    ("tiny", {}, "identity", "spheroidal"),
    ("small_dde", {}, None, "spheroidal"),
    ("small_dde", dict(C=7, C_block=3), None, "spheroidal"),          # ragged channel blocks
    ("small_dde", dict(C=12), None, "spheroidal"),                   # 12 channels: V=4 degridder
    ("lofar", dict(T=640, nr_stations=5), None, "spheroidal"),       # N~=24, N=2048, 16 ch
    ("lofar_dde", dict(T=512, nr_stations=5), None, "spheroidal"),   # + random A-terms, w0
    ("ska", dict(T=384, nr_stations=4), None, "spheroidal"),         # N~=32, N=8192, 32 ch
    ("predict", dict(T=256, nr_stations=4, C=8), None, "spheroidal"),  # N~=32, 8 ch: one k-block/timestep
    ("small_dde", dict(C=24, C_block=8), None, "spheroidal"),       # 3 channel blocks of 8
    ("small_dde", dict(w_planes=4), None, "spheroidal"),            # W-stacking (NEXT-1, R-21)
    ("lofar_dde", dict(T=512, nr_stations=5, w_planes=3), None, "spheroidal"),
    ("small_dde", dict(C=64), None, "spheroidal"),                   # 2 blocks of 32 channels per timestep
    ("small_dde", dict(C=40, C_block=24), None, "spheroidal"),      # 24 + 16 channels: rotation J = 3 and 2
]


KINDS = {
    "default": (None, None),                       # default tensor-core kernels (split-f16 mma)
    "tc": ("tc", "tc"),                            # direct tensor-core kernels (no channel recurrence)
    "rec": ("gridder_tcr<*", "degridder_tc<*"),    # split-f16 gridder with the channel recurrence
    "rot": ("gridder_rot<*", "degridder_rot<*"),   # accumulator / phasor rotation over channel groups
    "rot2": ("gridder_rot2<*", "degridder_rot<*"), # rotation with E_t derived from the slot phasors
    "rot8": ("gridder_rot2<*", "degridder_rot8<*"), # degridder: 8 channel rows per lane (0.25 sincos/pair)
    "rot16": ("gridder_rot2<*", "degridder_rot16<*"), # degridder: 16 channel rows per lane
    "rot16t": ("gridder_rot2<*", "degridder_rot16t<*"), # + lo(A) B_hi as tf32 mma
    "tc2": ("gridder_rot2<*", "degridder_tc2<*"), # degridder: row-split phase (m per row, l in registers)
    "poly": ("gridder_rot2<*", "degridder_tcp<*"), # degridder with part of the sincos on the FMA pipe
    "tf32": ("gridder_tf32*", "degridder_tf32*"),  # split-tf32 tensor-core kernels
    "umma": ("gridder_umma*", "degridder_tc<*"),    # tcgen05 / TMEM gridder
    "simt": ("simt", "simt"),                      # CUDA-core kernels (the paper's structure)
}


@pytest.fixture(params=list(KINDS))
def kind(request, monkeypatch):
    """Kernel family under test (the variant environment overrides of include/idg.h).  Families a
    case is not eligible for (e.g. tensor-core gridders need C~ % 8 == 0) fall back to the default."""
    g, d = KINDS[request.param]
    if g:
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


@pytest.mark.parametrize("name,kw,chunk", [("small_dde", {}, 60000), ("lofar", dict(T=640, nr_stations=6), 300000),
                                           ("small_dde", dict(C=7, C_block=3), 40000),
                                           ("small_dde", dict(w_planes=3), 60000)])
def test_host_streamed_calls(name, kw, chunk, monkeypatch):
    """idg_grid_host / idg_degrid_host (work groups through triple-buffered staging) give the
    device-resident results: degridding bit-identical, gridding equal up to atomic summation order."""
    monkeypatch.setenv("IDG_HOST_CHUNK_BYTES", str(chunk))     # several work groups even at small sizes
    obs = idgsynth.make_observation(name, **kw)
    vis, aterms, tap = _inputs(obs)
    plan = idg.Plan.from_observation(obs)
    ws = idg.workspace(plan)
    uvw, at, tp = _dev(obs.uvw), _dev(aterms), _dev(tap)
    vis_h = torch.from_numpy(vis).pin_memory()
    g_dev = gpu_grid(obs, vis, aterms, tap, plan)
    g_host = torch.zeros_like(g_dev)
    idg.grid_host(plan, vis_h, uvw, at, tp, g_host, ws)
    idg.grid_host(plan, vis_h, uvw, at, tp, g_host, ws)      # accumulates, buffers reused across calls
    torch.cuda.synchronize()
    assert rel_rms(g_host.cpu().numpy(), 2 * g_dev.cpu().numpy()) < 1e-6
    G = _dev(idgsynth.make_grid(obs))
    v_dev = gpu_degrid(obs, G, aterms, tap, plan)
    v_host = torch.full(v_dev.shape, complex(3, 3), dtype=torch.complex64).pin_memory()
    idg.degrid_host(plan, G, uvw, at, tp, v_host, ws)
    torch.cuda.synchronize()
    assert torch.equal(v_host, v_dev.cpu())


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
