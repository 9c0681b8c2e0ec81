"""Pins of the fp64 oracle against what the paper and the mathematics fix (no GPU).

P:n = /root/reference/PAPER.md line n.  Each pin is chosen so that a plausible slip in the oracle
(a dropped term, a wrong sign or index, a transposed operand, a swapped station) fails at least one:

  * centred subgrid DFT  == checkerboard . numpy.fft.fft2 . checkerboard      (library routine)
  * degrid of the model grid of ONE point source == Eq. (1) closed form, with random per-station
    A-terms, a non-trivial taper, w-term and w0  (A_p B A_q^H, e^{-2 pi i (ul+vm+wn)})
  * adjoint identity <degrid(G), V> == <G, grid(V)> for random G, V, A, taper, w0
  * identity A-terms, unit taper, w=0, on-cell uv: grid == N~^2 x nearest-cell gridding
  * one off-cell visibility spreads as the Dirichlet kernel D(dx) D(dy) (closed-form geometric sum)
"""
import dataclasses
import math

import numpy as np
import pytest

import idgsynth
import oracle

C0 = 299792458.0


def _inner(a, b):
    return np.vdot(a.reshape(-1), b.reshape(-1))   # sum conj(a) b


# ------------------------------------------------------------------------------------------------
# subgrid FFT (a4 / a7)
# ------------------------------------------------------------------------------------------------

@pytest.mark.parametrize("n", [16, 18, 24, 32])
def test_centred_dft_is_checkerboard_fft(n):
    rng = np.random.default_rng(n)
    a = rng.standard_normal((n, n)) + 1j * rng.standard_normal((n, n))
    cb = np.fromfunction(lambda y, x: (-1.0) ** (x + y), (n, n))
    fwd = oracle.centred_dft(a, -1)
    np.testing.assert_allclose(fwd, cb * np.fft.fft2(cb * a), rtol=0, atol=1e-11 * n * n)
    inv = oracle.centred_dft(a, +1)
    np.testing.assert_allclose(inv, cb * np.fft.ifft2(cb * a) * n * n, rtol=0, atol=1e-11 * n * n)


def test_centred_dft_delta_lands_on_centre():
    # a constant image transforms to N~^2 at the centre cell (k = N~/2): the zero frequency is centred
    n = 24
    out = oracle.centred_dft(np.ones((n, n), dtype=complex), -1)
    expect = np.zeros((n, n), dtype=complex)
    expect[n // 2, n // 2] = n * n
    np.testing.assert_allclose(out, expect, atol=1e-9)


# ------------------------------------------------------------------------------------------------
# degrid: point source through Eq. (1)
# ------------------------------------------------------------------------------------------------

def _point_source_case(obs, x0, y0, B, taper, aterms):
    """Model grid of a point source of brightness B (2x2) at subgrid pixel (x0,y0), divided by the
    taper at that pixel (the 'simple correction'), and the Eq. (1) visibilities it predicts."""
    n, N, L = obs.subgrid_size, obs.grid_size, obs.image_size
    l0 = (x0 - n / 2) * L / n
    m0 = (y0 - n / 2) * L / n
    n0 = 1 - math.sqrt(1 - l0 * l0 - m0 * m0)
    g = np.arange(N) - N / 2
    # G(gy,gx) = B/sph0 * exp(-2 pi i (u_g l0 + v_g m0)), u_g = (gx - N/2) du, du = 1/L
    ph = np.exp(-2j * np.pi * (g[None, :] * l0 + g[:, None] * m0) / L)
    sph0 = float(taper[y0, x0])
    grid = B.reshape(4)[:, None, None] / sph0 * ph[None]          # complex128: exact model
    return grid, (l0, m0, n0)


def _eq1_visibilities(obs, items, aterms, x0, y0, B, lmn):
    """V = N~^2 A_p B A_q^H exp(-2 pi i (u l0 + v m0 + (w - w0) n0))  (Eq. 1, discretised)."""
    l0, m0, n0 = lmn
    n = obs.subgrid_size
    out = []
    for it in items:
        p, q = obs.baselines[it["baseline"]]
        Ap = aterms[it["aterm_index"], p, y0, x0].astype(np.complex128).reshape(2, 2)
        Aq = aterms[it["aterm_index"], q, y0, x0].astype(np.complex128).reshape(2, 2)
        M = Ap @ B @ Aq.conj().T
        t0, nt = int(it["time_offset"]), int(it["nr_timesteps"])
        c0, c1 = int(it["channel_begin"]), int(it["channel_end"])
        uvw = obs.uvw[it["baseline"], t0:t0 + nt].astype(np.float64)          # [nt][3]
        k = obs.frequencies[c0:c1] / C0                                        # [nc]
        u, v, w = (uvw[:, i:i + 1] * k[None, :] for i in range(3))
        ph = np.exp(-2j * np.pi * (u * l0 + v * m0 + (w - obs.w_offset) * n0))
        out.append((n * n * ph[:, :, None] * M.reshape(4)[None, None, :]).reshape(-1))
    return np.concatenate(out)


@pytest.mark.parametrize("pix", [(11, 6), (3, 13), (8, 8)])
def test_degrid_point_source_matches_eq1(pix):
    obs = idgsynth.make_observation("small_dde")
    assert obs.w_offset != 0.0
    items, dropped = oracle.plan(obs)
    assert dropped == 0 and len(items) > 50
    items = items[::7]                                   # a spread of items keeps the test fast
    taper = idgsynth.make_taper(obs.subgrid_size, "asymmetric")
    aterms = idgsynth.make_aterms(obs, "random")
    rng = np.random.default_rng(5)
    B = rng.standard_normal((2, 2)) + 1j * rng.standard_normal((2, 2))
    x0, y0 = pix
    grid, lmn = _point_source_case(obs, x0, y0, B, taper, aterms)
    got = oracle.degrid(obs, items, grid, aterms, taper)
    want = _eq1_visibilities(obs, items, aterms, x0, y0, B, lmn)
    err = np.linalg.norm(got - want) / np.linalg.norm(want)
    assert err < 1e-11, err


def test_degrid_point_source_catches_w_sign():
    # the same check with w0 -> -w0 in the expectation must fail: the pin is sensitive to the w-term
    obs = idgsynth.make_observation("small_dde")
    items, _ = oracle.plan(obs)
    items = items[::11]
    taper = idgsynth.make_taper(obs.subgrid_size, "asymmetric")
    aterms = idgsynth.make_aterms(obs, "random")
    B = np.array([[1.0, 0.3j], [-0.2, 0.7]])
    grid, (l0, m0, n0) = _point_source_case(obs, 12, 3, B, taper, aterms)
    got = oracle.degrid(obs, items, grid, aterms, taper)
    wrong = _eq1_visibilities(obs, items, aterms, 12, 3, B, (l0, m0, -n0))
    assert np.linalg.norm(got - wrong) / np.linalg.norm(wrong) > 1e-3


# ------------------------------------------------------------------------------------------------
# adjoint identity grid <-> degrid
# ------------------------------------------------------------------------------------------------

def test_adjoint_identity():
    obs = idgsynth.make_observation("small_dde")
    items, _ = oracle.plan(obs)
    items = items[::3]
    taper = idgsynth.make_taper(obs.subgrid_size, "asymmetric")
    aterms = idgsynth.make_aterms(obs, "random")
    vis = idgsynth.make_visibilities(obs)
    G = idgsynth.make_grid(obs)
    DG = oracle.degrid(obs, items, G, aterms, taper)                       # flat, item order
    V = oracle.gather_visibilities(obs, items, vis).astype(np.complex128)
    gV = oracle.grid(obs, items, vis, aterms, taper)
    lhs = _inner(DG, V)
    rhs = _inner(G.astype(np.complex128), gV)
    assert abs(lhs - rhs) / abs(lhs) < 1e-12, (lhs, rhs)


# ------------------------------------------------------------------------------------------------
# gridding reduces to plain gridding (identity A, unit taper, w = 0)
# ------------------------------------------------------------------------------------------------

def _handmade_observation(cells_u, cells_v, N=256, n=16, K=5, Tmax=32):
    """C=1 at nu = c (so u_lambda = u metres) and L = 1/64: u = 64 * cell metres is exact in fp32."""
    nbl, T = cells_u.shape
    L = 1.0 / 64
    uvw = np.zeros((nbl, T, 3), dtype=np.float32)
    uvw[:, :, 0] = cells_u / L
    uvw[:, :, 1] = cells_v / L
    base = idgsynth.make_observation("tiny")
    return dataclasses.replace(
        base, name="handmade", nr_stations=nbl + 1,
        baselines=np.stack([np.zeros(nbl), np.arange(1, nbl + 1)], axis=1).astype(np.int32),
        uvw=uvw, frequencies=np.array([C0]), aterm_offsets=np.array([0, T], dtype=np.int32),
        subgrid_size=n, grid_size=N, image_size=L, kernel_size=K, max_timesteps_per_subgrid=Tmax,
        max_channels_per_subgrid=0, w_offset=0.0, aterm_kind="identity")


def test_on_cell_gridding_is_nearest_cell_times_n2():
    rng = np.random.default_rng(3)
    nbl, T = 5, 40
    cu = np.cumsum(rng.integers(-1, 2, (nbl, T)), axis=1) + rng.integers(-80, 80, (nbl, 1))
    cv = np.cumsum(rng.integers(-1, 2, (nbl, T)), axis=1) + rng.integers(-80, 80, (nbl, 1))
    obs = _handmade_observation(cu.astype(np.float64), cv.astype(np.float64))
    items, dropped = oracle.plan(obs)
    assert dropped == 0 and len(items) >= nbl
    vis = idgsynth.make_visibilities(obs)
    aterms = idgsynth.make_aterms(obs, "identity")
    taper = idgsynth.make_taper(obs.subgrid_size, "ones")
    got = oracle.grid(obs, items, vis, aterms, taper)
    N, n = obs.grid_size, obs.subgrid_size
    want = np.zeros_like(got)
    for b in range(nbl):
        for t in range(T):
            want[:, cv[b, t] + N // 2, cu[b, t] + N // 2] += n * n * vis[b, t, 0, :]
    err = np.linalg.norm(got - want) / np.linalg.norm(want)
    assert err < 1e-11, err


def test_off_cell_visibility_spreads_as_dirichlet_kernel():
    n, N = 16, 256
    du_off, dv_off = 0.37, -0.21
    cu = np.array([[20.0 + du_off]])
    cv = np.array([[-33.0 + dv_off]])
    obs = _handmade_observation(cu, cv, N=N, n=n)
    items, _ = oracle.plan(obs)
    assert len(items) == 1
    it = items[0]
    vis = np.zeros((1, 1, 1, 4), dtype=np.complex64)
    vis[0, 0, 0] = [1 + 2j, -0.5j, 0.25, 3 - 1j]
    aterms = idgsynth.make_aterms(obs, "identity")
    taper = idgsynth.make_taper(n, "ones")
    sub = oracle.gridder_item(obs, it, vis, aterms, taper)                    # [4][n][n]
    u_rel = float(obs.uvw[0, 0, 0]) * obs.image_size - (int(it["x"]) + n / 2 - N / 2)
    v_rel = float(obs.uvw[0, 0, 1]) * obs.image_size - (int(it["y"]) + n / 2 - N / 2)
    k = np.arange(n) - n / 2

    def dirichlet(delta):   # sum_{x=0}^{n-1} exp(2 pi i (x - n/2) delta / n), closed form
        r = np.exp(2j * np.pi * delta / n)
        return np.exp(-1j * np.pi * delta) * (r ** n - 1) / (r - 1)

    want = dirichlet(v_rel - k)[:, None] * dirichlet(u_rel - k)[None, :]
    for pol in range(4):
        np.testing.assert_allclose(sub[pol], complex(vis[0, 0, 0, pol]) * want, rtol=1e-10, atol=1e-10)


# ------------------------------------------------------------------------------------------------
# W-stacking (reading R-21): per-plane w0 and grid copies
# ------------------------------------------------------------------------------------------------

def test_w_stacking_point_source_matches_eq1_with_full_w_term():
    """With W-planes the model of plane z carries exp(-2 pi i w0_z n0); degridding every item from its
    own plane then reproduces Eq. (1) with the FULL w-term (no w0 left)."""
    obs = idgsynth.make_observation("small_dde", w_planes=4)
    assert obs.nr_w_planes == 4
    items, dropped = oracle.plan(obs)
    assert dropped == 0 and len(set(items["z"].tolist())) >= 3
    items = items[::5]
    taper = idgsynth.make_taper(obs.subgrid_size, "asymmetric")
    aterms = idgsynth.make_aterms(obs, "random")
    B = np.array([[0.7 + 0.1j, -0.3j], [0.2, 1.1 - 0.4j]])
    x0, y0 = 10, 5
    g1, (l0, m0, n0) = _point_source_case(obs, x0, y0, B, taper, aterms)
    nz = obs.nr_w_planes
    w0s = obs.w_offset + (np.arange(nz) - (nz - 1) / 2) * obs.w_step
    grid = np.stack([g1 * np.exp(-2j * np.pi * w0 * n0) for w0 in w0s])
    got = oracle.degrid(obs, items, grid, aterms, taper)
    flat = dataclasses.replace(obs, w_offset=0.0)           # Eq. (1) with the full w-term
    want = _eq1_visibilities(flat, items, aterms, x0, y0, B, (l0, m0, n0))
    err = np.linalg.norm(got - want) / np.linalg.norm(want)
    assert err < 1e-11, err


def test_w_stacking_adjoint_identity():
    obs = idgsynth.make_observation("small_dde", w_planes=3)
    items, _ = oracle.plan(obs)
    items = items[::3]
    taper = idgsynth.make_taper(obs.subgrid_size, "asymmetric")
    aterms = idgsynth.make_aterms(obs, "random")
    vis = idgsynth.make_visibilities(obs)
    G = idgsynth.make_grid(obs)
    assert G.shape[0] == 3
    DG = oracle.degrid(obs, items, G, aterms, taper)
    V = oracle.gather_visibilities(obs, items, vis).astype(np.complex128)
    gV = oracle.grid(obs, items, vis, aterms, taper)
    lhs, rhs = _inner(DG, V), _inner(G.astype(np.complex128), gV)
    assert abs(lhs - rhs) / abs(lhs) < 1e-12, (lhs, rhs)
