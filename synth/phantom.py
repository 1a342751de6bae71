"""Phantoms and noisy parallel-beam sinograms.

Units: mm and mm^-1.  mu_water = 0.02 mm^-1.  Field of view 256 mm, pixel pitch
dxy = 256/N, detector pitch dc = N*dxy/M (the detector spans the image width).
Views theta_k = k*pi/V.  Channel i covers [t0 + i*dc, t0 + (i+1)*dc),
t0 = -M*dc/2 + center_offset*dc.

Sinogram: p_i = mean over `subrays` equally spaced rays inside channel i of the analytic
line integral of the phantom; counts lambda_i ~ Poisson(lambda0 * exp(-p_i)) from a numpy
generator seeded per slice by (noise seed, z);
y_i = ln(lambda0 / max(lambda_i, 1)), w_i = max(lambda_i, 1) (inverse variance of y_i).
"""
from __future__ import annotations

import math
from dataclasses import dataclass, field

import numpy as np

MU_WATER = 0.02
FOV_MM = 256.0

# Kak & Slaney 2-D Shepp-Logan: (x0, y0, a, b, phi_deg, relative density)
_SL2D = [
    (0.0, 0.0, 0.69, 0.92, 0.0, 2.0),
    (0.0, -0.0184, 0.6624, 0.874, 0.0, -0.98),
    (0.22, 0.0, 0.11, 0.31, -18.0, -0.02),
    (-0.22, 0.0, 0.16, 0.41, 18.0, -0.02),
    (0.0, 0.35, 0.21, 0.25, 0.0, 0.01),
    (0.0, 0.1, 0.046, 0.046, 0.0, 0.01),
    (0.0, -0.1, 0.046, 0.046, 0.0, 0.01),
    (-0.08, -0.605, 0.046, 0.023, 0.0, 0.01),
    (0.0, -0.605, 0.023, 0.023, 0.0, 0.01),
    (0.06, -0.605, 0.023, 0.046, 0.0, 0.01),
]

# Kak & Slaney 3-D Shepp-Logan: (x0, y0, z0, a, b, c, phi_deg about z, relative density)
_SL3D = [
    (0.0, 0.0, 0.0, 0.69, 0.92, 0.9, 0.0, 2.0),
    (0.0, 0.0, 0.0, 0.6624, 0.874, 0.88, 0.0, -0.98),
    (-0.22, 0.0, -0.25, 0.41, 0.16, 0.21, 108.0, -0.02),
    (0.22, 0.0, -0.25, 0.31, 0.11, 0.22, 72.0, -0.02),
    (0.0, 0.35, -0.25, 0.21, 0.25, 0.5, 0.0, 0.01),
    (0.0, 0.1, -0.25, 0.046, 0.046, 0.046, 0.0, 0.01),
    (-0.08, -0.65, -0.25, 0.046, 0.023, 0.02, 0.0, 0.01),
    (0.06, -0.65, -0.25, 0.046, 0.023, 0.02, 90.0, 0.01),
    (0.06, -0.105, 0.0625, 0.056, 0.04, 0.1, 90.0, 0.02),
    (0.0, 0.1, 0.0625, 0.056, 0.056, 0.1, 0.0, -0.02),
]


def shepp_logan_2d():
    """Ellipses in mm: (x0, y0, a, b, phi_rad, mu) with mu in mm^-1."""
    r = FOV_MM / 2
    return [(x0 * r, y0 * r, a * r, b * r, math.radians(p), d * MU_WATER)
            for (x0, y0, a, b, p, d) in _SL2D]


def shepp_logan_3d(z_norm: float):
    """The ellipses cut by the plane z = z_norm (normalised head coordinates)."""
    r = FOV_MM / 2
    out = []
    for (x0, y0, z0, a, b, c, p, d) in _SL3D:
        t = 1.0 - ((z_norm - z0) / c) ** 2
        if t <= 0:
            continue
        s = math.sqrt(t)
        out.append((x0 * r, y0 * r, a * s * r, b * s * r, math.radians(p), d * MU_WATER))
    return out


def baggage_phantom(seed: int, n_objects: int = 6):
    """Security-scan-like slice (P:273 TO3 is baggage): random objects in air, a few dense
    inclusions (3-10 mu_w), large air fraction -- exercises zero-skipping."""
    rng = np.random.default_rng(seed)
    r = FOV_MM / 2
    ells = []
    for _ in range(n_objects):
        x0, y0 = rng.uniform(-0.55, 0.55, 2) * r
        a, b = rng.uniform(0.05, 0.25, 2) * r
        ells.append((x0, y0, a, b, rng.uniform(0, math.pi), rng.uniform(0.3, 1.5) * MU_WATER))
    for _ in range(2):
        x0, y0 = rng.uniform(-0.5, 0.5, 2) * r
        a, b = rng.uniform(0.01, 0.04, 2) * r
        ells.append((x0, y0, a, b, rng.uniform(0, math.pi), rng.uniform(3, 10) * MU_WATER))
    return ells


def _line_integrals(ells, theta, t):
    """Analytic line integrals of a sum of uniform ellipses.
    theta: [V], t: [V, R] detector coordinates (mm).  Returns [V, R] (dimensionless)."""
    c = np.cos(theta)[:, None]
    s = np.sin(theta)[:, None]
    out = np.zeros(t.shape, np.float64)
    for (x0, y0, a, b, phi, mu) in ells:
        ct = np.cos(theta - phi)[:, None]
        st = np.sin(theta - phi)[:, None]
        r2 = a * a * ct * ct + b * b * st * st
        sp = t - (x0 * c + y0 * s)
        disc = r2 - sp * sp
        out += np.where(disc > 0, mu * 2.0 * a * b * np.sqrt(np.maximum(disc, 0.0)) / r2, 0.0)
    return out


def sinogram(ells, nviews: int, nchannels: int, dchannel: float, center_offset: float = 0.0,
             subrays: int = 4):
    """Noise-free projection p [V, M] averaged over `subrays` rays per channel."""
    theta = np.arange(nviews, dtype=np.float64) * math.pi / nviews
    t0 = -0.5 * nchannels * dchannel + center_offset * dchannel
    sub = (np.arange(subrays) + 0.5) / subrays
    t = t0 + (np.arange(nchannels)[:, None] + sub[None, :]).reshape(-1) * dchannel
    tt = np.broadcast_to(t[None, :], (nviews, t.size))
    p = _line_integrals(ells, theta, tt)
    return p.reshape(nviews, nchannels, subrays).mean(axis=2)


def phantom_image(ells, n: int, supersample: int = 4):
    """Pixel-averaged phantom on the N x N grid (for RMSE-to-truth, sigma tuning)."""
    d = FOV_MM / n
    sub = (np.arange(supersample) + 0.5) / supersample - 0.5
    coords = ((np.arange(n) - (n - 1) / 2)[:, None] + sub[None, :]).reshape(-1) * d
    X, Y = np.meshgrid(coords, coords)  # [iy, ix]
    img = np.zeros_like(X)
    for (x0, y0, a, b, phi, mu) in ells:
        xr = (X - x0) * math.cos(phi) + (Y - y0) * math.sin(phi)
        yr = -(X - x0) * math.sin(phi) + (Y - y0) * math.cos(phi)
        img += np.where((xr / a) ** 2 + (yr / b) ** 2 <= 1.0, mu, 0.0)
    return img.reshape(n, supersample, n, supersample).mean(axis=(1, 3))


@dataclass
class WorkloadConfig:
    """One BASELINE.json config, made concrete."""
    name: str
    n: int
    nz: int
    nviews: int
    nchannels: int
    sv_side: int
    nbhd: int
    sigma: float
    phantom: str = "shepp_logan"
    lambda0: float = 1.0e4
    center_offset: float = 0.0
    fov: float = FOV_MM  # image width in mm (dxy = fov / n); the phantom is always FOV_MM wide

    @property
    def dxy(self):
        return self.fov / self.n

    @property
    def dchannel(self):
        return self.n * self.dxy / self.nchannels


# sigma_x (mm^-1) per config: DESIGN.md "Input recipe" (tuned once on cfg1, scaled by dxy)
CONFIGS = {
    "cfg1": WorkloadConfig("cfg1", 64, 1, 90, 96, 9, 8, 0.002),
    "cfg2": WorkloadConfig("cfg2", 256, 8, 360, 384, 9, 26, 0.004),
    "cfg3": WorkloadConfig("cfg3", 512, 1, 720, 1024, 9, 8, 0.005),
    "cfg4": WorkloadConfig("cfg4", 512, 64, 720, 1024, 9, 26, 0.005),
}


def slice_ellipses(cfg: WorkloadConfig, z: int, phantom_seed: int):
    """The ellipses of global slice z of a config's phantom (2-D Shepp-Logan, a slab of the 3-D
    head with slices sampling z in [-0.25, 0.25], or a baggage scene)."""
    if cfg.phantom == "baggage":
        return baggage_phantom(phantom_seed * 1000 + z)
    if cfg.nz == 1:
        return shepp_logan_2d()
    return shepp_logan_3d(-0.25 + 0.5 * (z + 0.5) / cfg.nz)


def noisy_counts(p: np.ndarray, lambda0: float, noise_seed: int, z: int):
    """Poisson counts of slice z: lambda ~ Poisson(lambda0 exp(-p)) from a generator seeded by
    (noise_seed, z), so any slab of a volume is the same whoever computes it; returns (y, w)
    float32 with y = ln(lambda0 / max(lambda, 1)), w = max(lambda, 1)."""
    rng = np.random.default_rng([noise_seed, z])
    lam = np.maximum(rng.poisson(lambda0 * np.exp(-p)), 1).astype(np.float64)
    return np.log(lambda0 / lam).astype(np.float32), lam.astype(np.float32)


def make_sinogram_torch(cfg: WorkloadConfig, case_id: int = 0, device="cuda", z0: int = 0,
                        z1: int | None = None):
    """The make_case recipe for the large bench configs: the analytic projections (double) are
    computed with torch on `device`, the Poisson counts with the same per-slice numpy generator
    as make_case (noisy_counts), so the result equals make_case(cfg, case_id) slice by slice.
    Returns float32 tensors y, w [z1-z0, V, M] on `device` for global slices [z0, z1)."""
    import torch
    V, M, nz = cfg.nviews, cfg.nchannels, cfg.nz
    z1 = nz if z1 is None else z1
    dev = torch.device(device)
    theta = torch.arange(V, dtype=torch.float64, device=dev) * math.pi / V
    t0 = -0.5 * M * cfg.dchannel + cfg.center_offset * cfg.dchannel
    sub = (torch.arange(4, dtype=torch.float64, device=dev) + 0.5) / 4
    t = t0 + (torch.arange(M, dtype=torch.float64, device=dev)[:, None] + sub[None, :]).reshape(-1) * cfg.dchannel
    c, s = torch.cos(theta)[:, None], torch.sin(theta)[:, None]
    y = torch.empty((z1 - z0, V, M), dtype=torch.float32, device=dev)
    w = torch.empty_like(y)
    for z in range(z0, z1):
        p = torch.zeros((V, t.numel()), dtype=torch.float64, device=dev)
        for (x0, y0, a, b, phi, mu) in slice_ellipses(cfg, z, 1000 + case_id):
            ct = torch.cos(theta - phi)[:, None]
            st = torch.sin(theta - phi)[:, None]
            r2 = a * a * ct * ct + b * b * st * st
            sp = t[None, :] - (x0 * c + y0 * s)
            disc = r2 - sp * sp
            p += torch.where(disc > 0, mu * 2.0 * a * b * torch.sqrt(disc.clamp_min(0.0)) / r2, 0.0)
        p = p.reshape(V, M, 4).mean(dim=2)
        yz, wz = noisy_counts(p.cpu().numpy(), cfg.lambda0, 2000 + case_id, z)
        y[z - z0] = torch.from_numpy(yz).to(dev)
        w[z - z0] = torch.from_numpy(wz).to(dev)
    return y, w


@dataclass
class Case:
    cfg: WorkloadConfig
    y: np.ndarray          # [nz, V, M] float32
    w: np.ndarray          # [nz, V, M] float32
    truth: np.ndarray      # [nz, N, N] float64 (pixel-averaged phantom)
    meta: dict = field(default_factory=dict)


def make_case(cfg: WorkloadConfig, case_id: int = 0, *, phantom_seed=None, noise_seed=None,
              with_truth: bool = True) -> Case:
    """Seeds: phantom 1000+case, noise 2000+case."""
    ps = 1000 + case_id if phantom_seed is None else phantom_seed
    ns = 2000 + case_id if noise_seed is None else noise_seed
    V, M, nz = cfg.nviews, cfg.nchannels, cfg.nz
    y = np.empty((nz, V, M), np.float32)
    w = np.empty((nz, V, M), np.float32)
    truth = np.empty((nz, cfg.n, cfg.n)) if with_truth else None
    for z in range(nz):
        ells = slice_ellipses(cfg, z, ps)
        p = sinogram(ells, V, M, cfg.dchannel, cfg.center_offset)
        y[z], w[z] = noisy_counts(p, cfg.lambda0, ns, z)
        if with_truth:
            truth[z] = phantom_image(ells, cfg.n)
    return Case(cfg, y, w, truth, {"phantom_seed": ps, "noise_seed": ns})


# sigma_x for the sweep by image size (the cfg1/cfg3 values scaled with the pixel pitch)
SWEEP_SIGMA = {64: 0.002, 128: 0.003, 256: 0.004}


def sweep_configs(n_cases: int = 200, seed: int = 5000, sizes=(128, 256), sides=(5, 7, 9), prefix="sweep"):
    """BASELINE.json configs[4]: synthetic 2-D cases varying phantom, dose, view count and SV side
    (the paper's 3200-case suite, in miniature), sampled without replacement from the
    grid phantom {Shepp-Logan, 3 baggage seeds} x lambda0 {1e3, 1e4, 1e5} x V {90, 180, 360, 720}
    x side {5, 7, 9} x N `sizes`, M = 2N (the paper's channel:pixel ratio, so dc = dxy/2).
    The 200-case sample keeps sides {5, 7, 9}; sides 11 and 13 of the survey's grid (two-window
    bands, 2-CTA clusters) form a supplementary sample: sweep_configs(40, 5001, sides=(11, 13),
    prefix="sweepL").  Returns [(WorkloadConfig, case_id)]."""
    rng = np.random.default_rng(seed)
    grid = [(ph, lam, v, s, n) for ph in ("shepp_logan", "baggage:0", "baggage:1", "baggage:2")
            for lam in (1e3, 1e4, 1e5) for v in (90, 180, 360, 720) for s in sides for n in sizes]
    pick = rng.choice(len(grid), size=min(n_cases, len(grid)), replace=False)
    out = []
    for i, gi in enumerate(sorted(pick)):
        ph, lam, v, s, n = grid[gi]
        base, _, bseed = ph.partition(":")
        cfg = WorkloadConfig(f"{prefix}{i}", n, 1, v, 2 * n, s, 8, SWEEP_SIGMA[n], phantom=base, lambda0=lam)
        out.append((cfg, 100 + (int(bseed) if bseed else 0)))
    return out
