"""Seeded synthetic input generators (models, geometry, source series).

This module holds NONE of the method's arithmetic: it only builds the inputs
that both the CUDA path and the fp64 oracle consume (velocity/density models,
source and receiver positions, the injected sample series s[n]).  The recipes
are the ones stated in DESIGN.md §4 (= SURVEY.md §8d); the paper gives no model,
size or step count ("one shot profile"), so every workload here is
ours, shaped like the paper's propagators.

All random media use ``numpy.random.default_rng(seed)`` with the default seed
20150207 (the paper's conference date, PMAM'15).
"""
from __future__ import annotations

import math
from dataclasses import dataclass, field
from typing import Optional

import numpy as np

SEED = 20150207


# ----------------------------------------------------------- source (O10/O11)
def ricker(t, fp, t0=None):
    """Ricker wavelet w(t) = (1 - 2 pi^2 fp^2 (t-t0)^2) exp(-pi^2 fp^2 (t-t0)^2), t0 = 1.5/fp.
    The paper names no wavelet ("f is the point source"); Ricker is BASELINE.json's."""
    t0 = 1.5 / fp if t0 is None else t0
    a = (math.pi * fp * (np.asarray(t, dtype=np.float64) - t0)) ** 2
    return (1.0 - 2.0 * a) * np.exp(-a)


def ricker_integral(t, fp, t0=None):
    """Exact antiderivative of the Ricker wavelet: G(t) = (t - t0) exp(-pi^2 fp^2 (t-t0)^2).
    Used for Eq 2's rho v^2 d_t^{-1} f source term."""
    t0 = 1.5 / fp if t0 is None else t0
    tt = np.asarray(t, dtype=np.float64) - t0
    return tt * np.exp(-((math.pi * fp * tt) ** 2))


def source_series(kind: str, nt: int, dt: float, fp: float, t0=None) -> np.ndarray:
    """Injected samples s[n], n = 0..nt-1, as fp32 (the API's wavelet array, O11):
    ISO s[n] = w(n dt); ACOUSTIC / ELASTIC s[n] = G((n + 1/2) dt)."""
    dt = float(np.float32(dt))
    n = np.arange(nt, dtype=np.float64)
    if kind == "iso":
        s = ricker(n * dt, fp, t0)
    elif kind in ("acoustic", "elastic"):
        s = ricker_integral((n + 0.5) * dt, fp, t0)
    else:
        raise ValueError(kind)
    return s.astype(np.float32)


# --------------------------------------------------------------- models
def gardner(vp):
    """Gardner density rho = 310 vp^0.25 (kg/m^3)."""
    return (310.0 * np.asarray(vp, dtype=np.float64) ** 0.25).astype(np.float32)


def homogeneous(shape, v, rho=None, vs=None):
    vp = np.full(shape, v, dtype=np.float32)
    out = {"vp": vp}
    if rho is not None:
        out["rho"] = np.full(shape, rho, dtype=np.float32)
    if vs is not None:
        out["vs"] = np.full(shape, vs, dtype=np.float32)
    return out


def random_media(shape, seed=SEED, elastic=False):
    """Random heterogeneous medium for tests: vp ~ U(1500,4500), rho ~ U(1000,2600),
    vs = vp/sqrt(3) * U(0.8,1)."""
    rng = np.random.default_rng(seed)
    vp = rng.uniform(1500.0, 4500.0, size=shape).astype(np.float32)
    rho = rng.uniform(1000.0, 2600.0, size=shape).astype(np.float32)
    out = {"vp": vp, "rho": rho}
    if elastic:
        out["vs"] = (vp / np.sqrt(3.0) * rng.uniform(0.8, 1.0, size=shape)).astype(np.float32)
    return out


def _undulation(nx, ny, scale):
    x = np.arange(nx, dtype=np.float64)
    y = np.arange(ny, dtype=np.float64)
    L = 256.0 * scale
    return 10.0 * scale * np.sin(2 * np.pi * x[None, :] / L) * np.cos(2 * np.pi * y[:, None] / L)


def layered_acoustic(nx, ny, nz, scale=None, z0=0, nzl=None):
    """C2 recipe: interfaces at z = 40,120,220,320,420 (of 512, scaled to nz) with
    undulation 10 sin(2 pi x/256) cos(2 pi y/256) points; vp = 1500 (water, rho 1000),
    1800, 2200, 2700, 3200, 3800; Gardner density below the water.
    z0, nzl: generate only the planes [z0, z0 + nzl) of the nz-deep model (one rank's z-slab;
    each plane depends on its global z only, so slabs concatenate to the whole model)."""
    s = nz / 512.0 if scale is None else scale
    nzl = nz - z0 if nzl is None else nzl
    iface = [40, 120, 220, 320, 420]
    vps = [1500.0, 1800.0, 2200.0, 2700.0, 3200.0, 3800.0]
    und = _undulation(nx, ny, s)  # [ny][nx]
    vp = np.empty((nzl, ny, nx), dtype=np.float32)
    rho = np.empty((nzl, ny, nx), dtype=np.float32)
    table = np.asarray(vps, dtype=np.float32)
    depth = [zi * s + und for zi in iface]
    for k in range(nzl):  # plane by plane (bounded host memory at 1024^3)
        layer = np.zeros((ny, nx), dtype=np.int32)
        for dz in depth:
            layer += (float(z0 + k) >= dz).astype(np.int32)
        vp[k] = table[layer]
        rho[k] = gardner(vp[k])
        rho[k][layer == 0] = 1000.0
    return {"vp": vp, "rho": rho}


def salt_acoustic(nx, ny, nz):
    """C4 recipe: the C2 layers plus a salt body (vp 4500, rho 2150): ellipsoid centred at
    (256,256,250) with semi-axes (150,120,80) points plus a stem cylinder of radius 40 from
    z = 140 to 250 (all scaled by n/512)."""
    m = layered_acoustic(nx, ny, nz)
    sx, sy, sz = nx / 512.0, ny / 512.0, nz / 512.0
    y = np.arange(ny, dtype=np.float64)[:, None]
    x = np.arange(nx, dtype=np.float64)[None, :]
    cx, cy, cz = 256 * sx, 256 * sy, 250 * sz
    exy = ((x - cx) / (150 * sx)) ** 2 + ((y - cy) / (120 * sy)) ** 2
    disc = ((x - cx) / sx) ** 2 + ((y - cy) / sy) ** 2 <= 40.0 ** 2
    for k in range(nz):  # plane by plane (bounded host memory at 1024^3)
        z = float(k)
        salt = exy + ((z - cz) / (80 * sz)) ** 2 <= 1.0
        if 140 * sz <= z <= 250 * sz:
            salt = salt | disc
        m["vp"][k][salt] = 4500.0
        m["rho"][k][salt] = 2150.0
    return m


def smooth(model, sigma):
    """Migration model: 3D Gaussian smoothing (sigma in points) of a true model."""
    from scipy.ndimage import gaussian_filter

    return {k: gaussian_filter(v.astype(np.float32), sigma=sigma, mode="nearest").astype(np.float32)
            for k, v in model.items()}


def smooth_torch(model, sigma, device):
    """The same migration model as smooth() -- separable 3D Gaussian, sigma in points, 'nearest'
    edges -- computed with torch on `device` (1024^3 grids; input preparation, not the method)."""
    import torch

    r = int(4 * sigma + 0.5)
    x = torch.arange(-r, r + 1, dtype=torch.float32, device=device)
    w = torch.exp(-0.5 * (x / sigma) ** 2)
    w = (w / w.sum()).view(1, 1, -1)
    F = torch.nn.functional
    out_model = {}
    for key, a in model.items():
        t = torch.from_numpy(np.ascontiguousarray(a, dtype=np.float32)).to(device)
        nz, ny, nx = t.shape
        out = torch.empty_like(t)
        for k in range(nz):  # x and y, plane by plane (small temporaries)
            p = t[k]
            p = F.conv1d(F.pad(p.view(ny, 1, nx), (r, r), mode="replicate"), w).view(ny, nx)
            p = F.conv1d(F.pad(p.t().contiguous().view(nx, 1, ny), (r, r), mode="replicate"), w).view(nx, ny).t()
            out[k] = p
        del t
        for j0 in range(0, ny, 64):  # z, per block of rows
            blk = out[:, j0:j0 + 64, :].permute(1, 2, 0).contiguous()  # [yb][nx][nz]
            yb = blk.shape[0]
            b = F.conv1d(F.pad(blk.view(yb * nx, 1, nz), (r, r), mode="replicate"), w)
            out[:, j0:j0 + 64, :] = b.view(yb, nx, nz).permute(2, 0, 1)
        out_model[key] = out.cpu().numpy()
        del out
        torch.cuda.empty_cache()
    return out_model


def layered_elastic(nx, ny, nz):
    """C3 recipe: layers at z = 60, 160, 280 (of 384, scaled): (vp, vs, rho) =
    (2000,1000,2000), (2800,1600,2200), (3500,2000,2400), (4500,2600,2600)."""
    s = nz / 384.0
    iface = [60 * s, 160 * s, 280 * s]
    props = np.asarray([[2000, 1000, 2000], [2800, 1600, 2200], [3500, 2000, 2400],
                        [4500, 2600, 2600]], dtype=np.float32)
    z = np.arange(nz, dtype=np.float64)
    layer = np.zeros(nz, dtype=np.int32)
    for zi in iface:
        layer += (z >= zi).astype(np.int32)
    col = props[layer]  # [nz][3]
    shape = (nz, ny, nx)
    return {"vp": np.broadcast_to(col[:, 0, None, None], shape).copy(),
            "vs": np.broadcast_to(col[:, 1, None, None], shape).copy(),
            "rho": np.broadcast_to(col[:, 2, None, None], shape).copy()}


# --------------------------------------------------------------- workloads
@dataclass
class Workload:
    """One synthetic workload: grid + model + shot (all host arrays)."""
    name: str
    kind: str                      # "iso" | "acoustic" | "elastic"
    nx: int
    ny: int
    nz: int
    h: float
    dt: float
    nt: int
    nb: int
    fp: float
    src: tuple
    rec: np.ndarray                # [nrec][3] int32 (x, y, z)
    model: dict
    free_surface: int = 0
    pml_R: float = 1e-3
    snap: int = 1
    rec_component: int = 2
    wavelet: Optional[np.ndarray] = field(default=None)

    def __post_init__(self):
        if self.wavelet is None:
            self.wavelet = source_series(self.kind, self.nt, self.dt, self.fp)

    @property
    def npts(self):
        return self.nx * self.ny * self.nz


def _line_x(x0, x1, y, z, step=1):
    xs = np.arange(x0, x1 + 1, step, dtype=np.int32)
    return np.stack([xs, np.full_like(xs, y), np.full_like(xs, z)], axis=1)


def _carpet(lo, hi, step, z):
    v = np.arange(lo, hi + 1, step, dtype=np.int32)
    yy, xx = np.meshgrid(v, v, indexing="ij")
    return np.stack([xx.ravel(), yy.ravel(), np.full(xx.size, z, dtype=np.int32)], axis=1)


def c1(n=64, nt=200, nb=0):
    """C1: ISO 64^3 homogeneous v = 2000, h 10 m, dt 1 ms, Ricker 15 Hz at the centre;
    receivers at r = 5, 10, 15 h on +x and on the diagonal (6,6,6), plus an x-line."""
    c = n // 2
    pts = [(c + 5, c, c), (c + 10, c, c), (c + 15, c, c), (c + 6, c + 6, c + 6)]
    line = _line_x(max(0, c - 24), min(n - 1, c + 24), c, max(0, c - 8), 2)
    rec = np.concatenate([np.asarray(pts, dtype=np.int32), line], axis=0)
    return Workload("C1", "iso", n, n, n, 10.0, 1e-3, nt, nb, 15.0, (c, c, c), rec,
                    homogeneous((n, n, n), 2000.0))


def c2(n=512, nt=2000, nb=20, model=True):
    """C2: acoustic layered n^3, 2000 steps of 0.8 ms, C-PML (6 faces), Ricker 10 Hz at
    (n/2, n/2, 24 s), receiver line z = 24 s, y = n/2, x = 20 s .. n-21 s.
    model=False: geometry only (the caller builds the model, e.g. one z-slab per rank)."""
    s = n / 512.0
    zr = max(nb + 1, int(round(24 * s)))
    x0, x1 = int(round(20 * s)), n - 1 - int(round(20 * s))
    rec = _line_x(x0, x1, n // 2, zr)
    return Workload("C2", "acoustic", n, n, n, 10.0, 8e-4, nt, nb, 10.0, (n // 2, n // 2, zr), rec,
                    layered_acoustic(n, n, n) if model else {})


def c3(n=384, nt=1500, nb=20):
    """C3: elastic layered n^3, 1500 steps of 0.7 ms, free surface on top, C-PML on the other
    5 faces, explosive Ricker 10 Hz at (n/2, n/2, 10 s); surface receiver line (vz, k = 0)."""
    s = n / 384.0
    zs = max(1, int(round(10 * s)))
    x0, x1 = int(round(20 * s)), n - 1 - int(round(20 * s))
    rec = _line_x(x0, x1, n // 2, 0)
    return Workload("C3", "elastic", n, n, n, 10.0, 7e-4, nt, nb, 10.0, (n // 2, n // 2, zs), rec,
                    layered_elastic(n, n, n), free_surface=1, rec_component=2)


def c4(n=512, nt=2000, nb=20, snap=20, carpet_step=4):
    """C4: acoustic RTM n^3 on the salt model: observed data from the true model, migration
    on the Gaussian-smoothed (sigma 5 points) model; receiver carpet at z = 24 s,
    x, y in 20 s .. n-21 s step 4 s; snapshots every `snap` steps."""
    s = n / 512.0
    zr = max(nb + 1, int(round(24 * s)))
    step = max(1, int(round(carpet_step * s)))
    lo, hi = int(round(20 * s)), n - 1 - int(round(20 * s))
    rec = _carpet(lo, hi, step, zr)
    return Workload("C4", "acoustic", n, n, n, 10.0, 8e-4, nt, nb, 10.0, (n // 2, n // 2, zr), rec,
                    salt_acoustic(n, n, n), snap=snap)


def recommended_snap(dt, fp):
    """snap_period = floor(1 / (2 f_max dt)), f_max = 2.5 fp ("depends on the maximum
    frequency")."""
    return max(1, int(math.floor(1.0 / (2.0 * 2.5 * fp * dt))))


def c5(n=1024, nt=1000, nb=20, snap=20):
    """C5: acoustic RTM 1024^3 -- the C4 geometry scaled x2 in points (same h): salt model,
    1000 steps of 0.8 ms, source at (n/2, n/2, 48), receiver carpet at z = 48, x, y in
    40 .. n-41 step 8 (13 924 receivers), snapshots every 20 steps (49)."""
    wl = c4(n=n, nt=nt, nb=nb, snap=snap, carpet_step=4)
    wl.name = "C5"
    return wl
