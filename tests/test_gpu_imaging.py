"""Imaging-cycle harness (NEXT-3, paper Fig. 2) on the GPU path: point sources through
grid -> iFFT -> dirty image -> peak -> model -> FFT -> degrid -> residual visibilities."""
import math

import numpy as np
import pytest

import idgsynth

torch = pytest.importorskip("torch")
import paper_conf_ipps_veenboerpr17_b200 as idg
from paper_conf_ipps_veenboerpr17_b200 import imaging

pytestmark = pytest.mark.gpu
C0 = 299792458.0


def _sky_vis(obs, sources):
    """Eq. (1) with identity A-terms: V_pol = sum_s B_s[pol] exp(-2 pi i (u l + v m + w n))."""
    uvw = obs.uvw.astype(np.float64)
    k = obs.frequencies / C0
    u, v, w = (uvw[:, :, None, i] * k[None, None, :] for i in range(3))
    vis = np.zeros((obs.nr_baselines, obs.nr_timesteps, obs.nr_channels, 4), dtype=np.complex128)
    for (l0, m0, flux) in sources:
        n0 = 1 - math.sqrt(1 - l0 * l0 - m0 * m0)
        vis += (flux * np.exp(-2j * np.pi * (u * l0 + v * m0 + w * n0)))[..., None] * np.array([1, 0, 0, 1])
    return vis.astype(np.complex64)


def _taper_image(obs, device):
    """The generator's separable PSWF taper evaluated on the N x N image pixels."""
    N, n = obs.grid_size, obs.subgrid_size
    nu = np.abs((np.arange(N) - N / 2) * n / N) / (n / 2 + 1)   # same nu(l) as idgsynth.make_taper
    s = idgsynth._grdsf(nu) * (1 - nu * nu)
    nu0 = np.abs(np.arange(n) - n / 2) / (n / 2 + 1)
    s = s / (idgsynth._grdsf(nu0) * (1 - nu0 * nu0)).max()
    return torch.from_numpy(np.outer(s, s)).to(device)


@pytest.mark.parametrize("w_planes", [1, 3])
def test_point_sources_image_and_predict(w_planes):
    obs = idgsynth.make_observation("small_dde", aterms="identity", w_planes=w_planes)
    N, n, L = obs.grid_size, obs.subgrid_size, obs.image_size
    step = N // n                                   # image pixels per subgrid pixel: the exact lattice
    pix = [(N // 2 + 3 * step, N // 2 - 2 * step, 1.0), (N // 2 - 5 * step, N // 2 + 4 * step, 0.6)]
    sources = [((x - N / 2) * L / N, (y - N / 2) * L / N, f) for (x, y, f) in pix]
    vis = _sky_vis(obs, sources)
    dev = torch.device("cuda")
    plan = idg.Plan.from_observation(obs)
    uvw = torch.from_numpy(obs.uvw).to(dev)
    at = torch.from_numpy(idgsynth.make_aterms(obs, "identity")).to(dev)
    tp = torch.from_numpy(idgsynth.make_taper(n)).to(dev)
    timg = _taper_image(obs, dev)
    dirty = imaging.dirty_image(plan, torch.from_numpy(vis).to(dev), uvw, at, tp, timg)
    val, y, x = imaging.find_peak(dirty, pol=0)
    assert (y, x) == (pix[0][1], pix[0][0]), (y, x, pix[0])
    assert abs(val - 1.0) < 0.2, val                # PSF sidelobes of the second source only
    # predict the exact two-source model: identical to Eq. (1) (lattice pixels are exact in IDG)
    model = torch.zeros((4, N, N), dtype=torch.complex64, device=dev)
    for (xx, yy, f) in pix:
        model[0, yy, xx] = f
        model[3, yy, xx] = f
    pred = torch.empty((obs.nr_baselines, obs.nr_timesteps, obs.nr_channels, 4), dtype=torch.complex64,
                       device=dev)
    imaging.predict(plan, model, uvw, at, tp, timg, pred)
    p = pred.cpu().numpy()
    err = np.linalg.norm(p - vis) / np.linalg.norm(vis)
    assert err < 1e-4, err
    # a one-component CLEAN step: subtracting the brightest source removes its power
    model[:, pix[1][1], pix[1][0]] = 0
    imaging.predict(plan, model, uvw, at, tp, timg, pred)
    res = vis - pred.cpu().numpy()
    assert np.linalg.norm(res) < 0.75 * np.linalg.norm(vis)


def test_imaging_cycle_breakdown():
    """One timed imaging cycle (Fig. 9 analogue): every stage reports a time, the stages add up to the
    total, and the residual of a cycle whose model is its own dirty image is the data minus its prediction."""
    obs = idgsynth.make_observation("lofar", T=256, nr_stations=6)
    plan = idg.Plan.from_observation(obs)
    dev = torch.device("cuda")
    vis = torch.from_numpy(idgsynth.make_visibilities(obs)).to(dev)
    uvw = torch.from_numpy(obs.uvw).to(dev)
    at = torch.from_numpy(idgsynth.make_aterms(obs)).to(dev)
    tp = torch.from_numpy(idgsynth.make_taper(obs.subgrid_size)).to(dev)
    out = torch.empty_like(vis)
    t = imaging.imaging_cycle(plan, vis, uvw, at, tp, _taper_image(obs, dev), out)
    stages = ["grid", "ifft", "image", "model", "degrid", "residual"]
    assert all(t[k] >= 0 for k in stages) and t["grid"] > 0 and t["degrid"] > 0
    assert abs(sum(t[k] for k in stages) - t["total_ms"]) < 1e-3 * t["total_ms"] + 1e-3
    assert torch.isfinite(torch.view_as_real(out)).all()
