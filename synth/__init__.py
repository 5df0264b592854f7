"""Seeded synthetic sample generators shared by the oracle tests, the GPU tests and bench.py.

This module holds NO arithmetic of the method (no encoding, no decoding, no
log transform, no normalisation).  It only produces raw samples shaped like the
paper's two workloads, plus per-channel statistics a training pipeline would
use for normalisation.  Recipes are stated in DESIGN.md §"Input recipe".

* CosmoFlow (§V.B, lines 96-100; Fig. 5 caption line 124): int16
  particle counts ``[4, D, H, W]`` (CDHW; four redshifts).  A lognormal density
  driven by one Gaussian random field shared across redshifts, Poisson counts
  drawn by inverse CDF through a Gaussian copula so the four redshifts are
  coupled ("highly coupled", line 98): few hundred unique values, tens of
  thousands of unique 4-groups, power-law value histogram.
* DeepCAM (§IV line 56, §V.A lines 72-92): fp32 ``[16, H, W]``
  (CHW), smooth along x (line 72, Fig. 2 caption line 76), sensor noise, ~2%
  area of abrupt localised "events" (lines 72, 82), a sparse
  precipitation-like channel with exact zeros and tiny bursts (line 92).
"""
from __future__ import annotations

import numpy as np
from scipy import special

__all__ = ["gen_cosmo", "gen_deepcam", "COSMO_PRESETS", "DEEPCAM_CHANNELS",
           "deepcam_stats", "gen_deepcam_labels", "gen_cosmo_labels"]

# name -> (lam, sigma, rho_c); paper = calibrated to P:98 (|U|~558, G~36,944)
COSMO_PRESETS = {
    "paper": (2.0, 2.0, 0.7),
    "sparse": (0.05, 2.0, 0.9),
    "verysparse": (0.01, 2.0, 0.7),
    "unit": (1.0, 2.0, 0.7),
    "dense": (16.0, 2.0, 0.0),
    "verydense": (64.0, 2.0, 0.0),
    "independent": (2.0, 2.0, 0.0),
    "coupled": (2.0, 2.0, 0.9),
}

_GROWTH = (0.4, 0.6, 0.8, 1.0)  # redshift growth factors D_r (high z -> today)


def _grf(rng: np.random.Generator, shape, slope: float, aniso=None) -> np.ndarray:
    """Unit-variance Gaussian random field with power spectrum P(k) ~ k**slope."""
    white = rng.standard_normal(shape)
    F = np.fft.rfftn(white)
    ks = []
    for ax, n in enumerate(shape):
        k = np.fft.rfftfreq(n) if ax == len(shape) - 1 else np.fft.fftfreq(n)
        if aniso is not None:
            k = k * aniso[ax]
        sh = [1] * len(shape)
        sh[ax] = k.size
        ks.append(k.reshape(sh))
    k2 = sum(k * k for k in ks)
    k2.flat[0] = np.inf
    F *= k2 ** (slope / 4.0)
    g = np.fft.irfftn(F, s=shape, axes=tuple(range(len(shape))))
    g -= g.mean()
    g /= g.std()
    return g


def _poisson_icdf(u: np.ndarray, lam: np.ndarray) -> np.ndarray:
    """Poisson inverse CDF, vectorised; normal approximation above lam=200."""
    out = np.zeros(u.shape, dtype=np.int64)
    big = lam > 200.0
    if big.any():
        z = special.ndtri(np.clip(u[big], 1e-300, 1 - 1e-16))
        lb = lam[big]
        out[big] = np.maximum(0, np.floor(lb + np.sqrt(lb) * z + 0.5)).astype(np.int64)
    idx = np.nonzero(~big)[0]
    uu = u[idx]
    ll = lam[idx]
    p = np.exp(-ll)
    cdf = p.copy()
    k = 0
    while idx.size:
        act = uu > cdf
        idx, uu, ll, p, cdf = idx[act], uu[act], ll[act], p[act], cdf[act]
        if not idx.size:
            break
        k += 1
        p = p * ll / k
        cdf = cdf + p
        out[idx] = k
        if k > 4000:  # numerical floor of the cdf; never reached for lam<=200
            break
    return out


def gen_cosmo(seed: int, preset: str = "paper", n: int = 128, *, lam=None,
              sigma=None, rho_c=None) -> np.ndarray:
    """int16 counts [4, n, n, n] (CDHW).  Deterministic in (seed, preset, n)."""
    plam, psig, prho = COSMO_PRESETS[preset]
    lam = plam if lam is None else lam
    sigma = psig if sigma is None else sigma
    rho_c = prho if rho_c is None else rho_c
    rng = np.random.default_rng(seed)
    g = _grf(rng, (n, n, n), slope=-2.0).ravel()
    z0 = rng.standard_normal(g.size)
    out = np.empty((4, g.size), dtype=np.int16)
    for r, D in enumerate(_GROWTH):
        s = sigma * D
        rho = lam * np.exp(s * g - 0.5 * s * s)
        zr = rng.standard_normal(g.size)
        u = special.ndtr(np.sqrt(rho_c) * z0 + np.sqrt(1.0 - rho_c) * zr)
        c = _poisson_icdf(u, rho)
        out[r] = np.minimum(c, 32767).astype(np.int16)
    return out.reshape(4, n, n, n)


# DeepCAM channel mix: (kind, mean, amplitude, noise)
DEEPCAM_CHANNELS = (
    ("temperature", 250.0, 30.0, 1e-3), ("temperature", 220.0, 20.0, 1e-3),
    ("temperature", 270.0, 25.0, 1e-3), ("temperature", 288.0, 15.0, 1e-3),
    ("wind", 0.0, 20.0, 1e-3), ("wind", 0.0, 15.0, 1e-3),
    ("wind", 0.0, 10.0, 1e-3), ("wind", 0.0, 8.0, 1e-3),
    ("geopotential", 12000.0, 800.0, 1e-4), ("geopotential", 5500.0, 300.0, 1e-4),
    ("geopotential", 100.0, 60.0, 1e-4),
    ("pressure", 1.0e5, 2.0e3, 1e-5), ("pressure", 1.01e5, 1.5e3, 1e-5),
    ("humidity", 0.01, 0.01, 1e-3), ("water", 30.0, 30.0, 1e-3),
    ("precipitation", 0.0, 1e-4, 0.0),
)


def gen_deepcam(seed: int, H: int = 768, W: int = 1152, C: int = 16,
                noise_scale: float = 1.0, event_frac: float = 0.02) -> np.ndarray:
    """fp32 [C, H, W] (CHW).  Deterministic in (seed, H, W, C)."""
    rng = np.random.default_rng(seed)
    out = np.empty((C, H, W), dtype=np.float32)
    yy, xx = np.mgrid[0:H, 0:W].astype(np.float64)
    # localised abrupt events (cyclone-like discs) shared by all channels
    n_ev = max(1, int(round(event_frac * H * W / (np.pi * (0.03 * H) ** 2))))
    ev_mask = np.zeros((H, W), dtype=bool)
    ev_field = np.zeros((H, W))
    for _ in range(n_ev):
        cy, cx = rng.uniform(0, H), rng.uniform(0, W)
        r = rng.uniform(0.015, 0.045) * H
        d = np.hypot(yy - cy, xx - cx)
        m = d < r
        ev_mask |= m
        ev_field[m] += rng.choice([-1.0, 1.0]) * (1.0 - d[m] / r) + rng.standard_normal(m.sum()) * 0.3
    for c in range(C):
        kind, mean, amp, noise = DEEPCAM_CHANNELS[c % len(DEEPCAM_CHANNELS)]
        # smoother along x (latitude lines) than along y: anisotropic spectrum
        g = _grf(rng, (H, W), slope=-3.5, aniso=(1.0, 0.5))
        if kind == "precipitation":
            f = np.where(g > 1.6, (g - 1.6) ** 2 * amp, 0.0)
            f = np.where(ev_mask & (ev_field > 0.2), f + ev_field * amp * 5.0, f)
            f = np.maximum(f, 0.0)
        elif kind in ("humidity", "water"):
            f = np.maximum(mean + amp * g, 0.0)
        else:
            f = mean + amp * g
        if kind != "precipitation":
            f = f + amp * 0.5 * ev_field  # abrupt changes at extreme events
            f = f + noise_scale * noise * amp * rng.standard_normal((H, W))
            if kind in ("humidity", "water"):
                f = np.maximum(f, 0.0)
        out[c] = f.astype(np.float32)
    return out


def deepcam_stats(x: np.ndarray):
    """Per-channel (mean, 1/std) as fp32: a training pipeline's normalisation
    constants (reading S18).  Statistics only, not the method."""
    m = x.reshape(x.shape[0], -1).astype(np.float64)
    mean = m.mean(axis=1)
    std = m.std(axis=1)
    std[std == 0] = 1.0
    return mean.astype(np.float32), (1.0 / std).astype(np.float32)


def gen_deepcam_labels(seed: int, H: int = 768, W: int = 1152) -> np.ndarray:
    """uint8 [H, W] per-pixel class mask shaped like DeepCAM's segmentation
    labels (PAPER.md P:56 semantic segmentation of extreme weather; classes as
    in the MLPerf DeepCAM dataset: 0 background, 1 tropical cyclone, 2
    atmospheric river): a few cyclone discs and a few long, thin, meandering
    river bands on a background that covers most of the image."""
    rng = np.random.default_rng(seed)
    yy, xx = np.mgrid[0:H, 0:W].astype(np.float64)
    m = np.zeros((H, W), dtype=np.uint8)
    for _ in range(int(rng.integers(1, 4))):                   # atmospheric rivers
        x0, x1 = np.sort(rng.uniform(0, W, 2))
        x1 = max(x1, x0 + 0.2 * W)
        y0 = rng.uniform(0.1, 0.9) * H
        amp, lam, ph = rng.uniform(0.02, 0.1) * H, rng.uniform(0.2, 0.6) * W, rng.uniform(0, 2 * np.pi)
        slope = rng.uniform(-0.3, 0.3)
        thick = rng.uniform(0.008, 0.025) * H
        yc = y0 + slope * (xx - x0) + amp * np.sin(2 * np.pi * xx / lam + ph)
        m[(np.abs(yy - yc) < thick) & (xx >= x0) & (xx < x1)] = 2
    for _ in range(int(rng.integers(1, 6))):                   # tropical cyclones
        cy, cx = rng.uniform(0.1, 0.9) * H, rng.uniform(0, W)
        r = rng.uniform(0.01, 0.025) * H
        m[np.hypot(yy - cy, xx - cx) < r] = 1
    return m


def gen_cosmo_labels(seed: int) -> np.ndarray:
    """fp32 [4]: the four cosmological parameters a CosmoFlow sample is
    labelled with, drawn uniformly from plausible ranges."""
    rng = np.random.default_rng(seed)
    lo = np.array([0.25, 0.70, 0.90, 0.60])
    hi = np.array([0.35, 0.90, 1.00, 0.80])
    return (lo + (hi - lo) * rng.random(4)).astype(np.float32)
