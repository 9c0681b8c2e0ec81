"""Imaging-cycle harness around the hot path (paper Fig. 2 / Fig. 4).

    visibilities --grid()--> uv-grid(s) --iFFT, corrections--> dirty image        ("imaging")
    model image --corrections, FFT--> model uv-grid(s) --degrid()--> visibilities ("predict")

The gridding and degridding are the library's (libidg_b200.so); the full-grid FFT is cuFFT through
torch.fft (off-path glue, as BASELINE.json's north star allows).  Conventions follow the library:
grid cell g <-> u = (g - N/2)/L, image pixel p <-> l = (p - N/2) L/N, n = 1 - sqrt(1 - l^2 - m^2),
the image is the centred DFT of the grid, and the subgrid transform carries the scale N~^2 (R-5).

"Up to a simple correction": IDG applies the spheroidal taper in the image domain of every
subgrid, and the phases are taken relative to w0 (per W-plane with W-stacking, R-21), so the dirty image
of plane z is divided by the taper on the full image (`taper_image`, the caller's taper function sampled
at the N x N image pixels) and multiplied by exp(+2 pi i w0_z n); prediction applies the inverse.
"""
from __future__ import annotations

import math

import torch

from . import idg


def _centred_ifft2(grid):
    """sum_g G(g) exp(+2 pi i (g - N/2)(p - N/2) / N), unnormalised, over the last two axes."""
    return torch.fft.fftshift(torch.fft.ifft2(torch.fft.ifftshift(grid, dim=(-2, -1)), norm="forward"),
                              dim=(-2, -1))


def _centred_fft2(image):
    """sum_p I(p) exp(-2 pi i (g - N/2)(p - N/2) / N), unnormalised, over the last two axes."""
    return torch.fft.fftshift(torch.fft.fft2(torch.fft.ifftshift(image, dim=(-2, -1)), norm="backward"),
                              dim=(-2, -1))


def image_lmn(plan: idg.Plan, device):
    """(l, m, n) of the N x N image pixels (n in the cancellation-free form of P:43)."""
    N, L = plan.grid_size, plan.params.image_size
    c = (torch.arange(N, device=device, dtype=torch.float64) - N / 2) * L / N
    m, l = torch.meshgrid(c, c, indexing="ij")
    r2 = l * l + m * m
    return l, m, r2 / (1 + torch.sqrt(1 - r2))


def _plane_w0(plan: idg.Plan):
    p = plan.params
    nz = plan.nr_w_planes
    return [p.w_offset + (z - (nz - 1) / 2) * p.w_step for z in range(nz)]


def dirty_image(plan: idg.Plan, vis, uvw, aterms, taper, taper_image, stream=None):
    """Grid `vis`, transform, correct: the dirty image [4][N][N] (complex64 per polarisation),
    normalised by N~^2 x the number of gridded visibilities (a unit point source peaks at ~1)."""
    N = plan.grid_size
    shape = (4, N, N) if plan.nr_w_planes == 1 else (plan.nr_w_planes, 4, N, N)
    g = torch.zeros(shape, dtype=torch.complex64, device=vis.device)
    idg.grid(plan, vis, uvw, aterms, taper, g, stream=stream)
    _, _, n = image_lmn(plan, vis.device)
    planes = g.reshape(plan.nr_w_planes, 4, N, N)
    img = torch.zeros((4, N, N), dtype=torch.complex128, device=vis.device)
    for z, w0 in enumerate(_plane_w0(plan)):
        img += _centred_ifft2(planes[z].to(torch.complex128)) * torch.exp(2j * math.pi * w0 * n)
    nvis = max(1, plan.stats()["nr_vis_assigned"])
    return (img / (taper_image.to(torch.float64) * (nvis * plan.subgrid_size ** 2))).to(torch.complex64)


def model_grid(plan: idg.Plan, model_image, taper_image):
    """Model uv-grid(s) of a model image [4][N][N] for degridding (the degridder re-applies the taper
    per subgrid and the phases relative to w0_z)."""
    _, _, n = image_lmn(plan, model_image.device)
    base = model_image.to(torch.complex128) / taper_image.to(torch.float64)
    grids = [_centred_fft2(base * torch.exp(-2j * math.pi * w0 * n)) for w0 in _plane_w0(plan)]
    G = torch.stack(grids).to(torch.complex64)
    return G[0] if plan.nr_w_planes == 1 else G


def predict(plan: idg.Plan, model_image, uvw, aterms, taper, taper_image, vis_out, stream=None):
    """Visibilities of a model image (degridding), scaled so that a unit point source at a pixel
    of the subgrid lattice predicts exp(-2 pi i (u l + v m + w n)) (Eq. 1 with identity A-terms)."""
    idg.degrid(plan, model_grid(plan, model_image, taper_image), uvw, aterms, taper, vis_out, stream=stream)
    vis_out /= plan.subgrid_size ** 2
    return vis_out


def find_peak(image, pol: int = 0):
    """(value, y, x) of the brightest pixel of the real part of one polarisation (the source finder of a
    one-component CLEAN step)."""
    re = image[pol].real
    idx = int(torch.argmax(re))
    y, x = divmod(idx, re.shape[-1])
    return float(re[y, x]), y, x


def imaging_cycle(plan: idg.Plan, vis, uvw, aterms, taper, taper_image, vis_out, stream=None, residual=True):
    """One full imaging cycle (Fig. 2) in production precision (complex64 throughout), timed per
    stage with CUDA events on `stream` -- the analogue of the paper's runtime breakdown (Fig. 9):

      grid      zero the uv-grid(s) + idg_grid (gridder, A-term/taper, subgrid FFT, adder: one fused kernel)
      ifft      centred inverse FFT of every polarisation / W-plane (cuFFT via torch.fft)
      image     taper + w0 corrections -> dirty image (elementwise)
      model     the dirty image stands in for the deconvolved model (deconvolution is out of scope):
                corrections + centred FFT back to the model grid(s)
      degrid    idg_degrid (splitter, subgrid iFFT, taper/A-term, degridder: one fused kernel)
      residual  vis - predicted (elementwise; skipped when vis_out aliases vis)

    Returns {stage: ms} plus 'total_ms'.  vis_out receives the residual (the unnormalised predictions, x N~^2,
    when it aliases vis)."""
    s = torch.cuda.current_stream(vis.device) if stream is None else stream
    N = plan.grid_size
    nz = plan.nr_w_planes
    shape = (4, N, N) if nz == 1 else (nz, 4, N, N)
    ev = {}

    def mark(name):
        e = torch.cuda.Event(enable_timing=True)
        e.record(s)
        ev[name] = e

    with torch.cuda.stream(s):
        _, _, n = image_lmn(plan, vis.device)
        n = n.to(torch.float32)
        w0s = _plane_w0(plan)
        tap = taper_image.to(torch.float32)
        nvis = max(1, plan.stats()["nr_vis_assigned"])
        g = torch.empty(shape, dtype=torch.complex64, device=vis.device)
        mark("start")
        g.zero_()
        idg.grid(plan, vis, uvw, aterms, taper, g, stream=s)
        mark("grid")
        planes = g.reshape(nz, 4, N, N)
        img_planes = _centred_ifft2(planes)
        mark("ifft")
        img = torch.zeros((4, N, N), dtype=torch.complex64, device=vis.device)
        for z, w0 in enumerate(w0s):
            img += img_planes[z] * torch.exp(2j * math.pi * w0 * n) if w0 != 0.0 else img_planes[z]
        img /= tap * (nvis * plan.subgrid_size ** 2)
        mark("image")
        base = img / tap
        model = torch.stack([base * torch.exp(-2j * math.pi * w0 * n) if w0 != 0.0 else base for w0 in w0s])
        G = _centred_fft2(model)
        G = G[0] if nz == 1 else G
        mark("model")
        idg.degrid(plan, G.contiguous(), uvw, aterms, taper, vis_out, stream=s)
        mark("degrid")
        if residual and vis_out.data_ptr() != vis.data_ptr():
            vis_out.sub_(vis).neg_()          # residual = vis - predicted
        mark("residual")
    ev["residual"].synchronize()
    names = ["grid", "ifft", "image", "model", "degrid", "residual"]
    out, prev = {}, "start"
    for k in names:
        out[k] = ev[prev].elapsed_time(ev[k])
        prev = k
    out["total_ms"] = ev["start"].elapsed_time(ev["residual"])
    return out
