"""Pin of the free surface's surface row (O16) -- CPU only.

The normal-incidence test in test_oracle_schemes.py pins the stress-imaging mirror but cannot
exercise the surface-row rule dz vz = -lam/(lam + 2 mu)(dx vx + dy vy), which only acts on
waves travelling ALONG the surface.  Lamb's problem does: an explosion just below the free
surface of a homogeneous Poisson solid (nu = 1/4, vp = sqrt(3) vs) excites a Rayleigh wave,
whose speed is the root of the Rayleigh equation, 0.919402 vs for nu = 1/4 (SURVEY §8c O16
pin: "the Rayleigh phase velocity along the surface line is within 2% of 0.9194 vs").
The surface vz records are cross-correlated between two offsets; the lag gives the speed.
"""
import numpy as np
import pytest
from scipy.optimize import brentq

import oracle
from paper_conf_ppopp_qawasmehchc15_b200 import inputs


def _rayleigh_ratio(nu=0.25):
    """Root c/vs in (0, 1) of the Rayleigh equation
    (2 - c^2)^2 = 4 sqrt(1 - c^2) sqrt(1 - c^2 k^2),  k = vs/vp (closed form, textbook)."""
    k2 = (1 - 2 * nu) / (2 * (1 - nu))
    f = lambda c: (2 - c * c) ** 2 - 4 * np.sqrt(1 - c * c) * np.sqrt(1 - k2 * c * c)
    return brentq(f, 0.5, 0.999)


def _lag(a, b, dt):
    """Delay of b relative to a: cross-correlation peak with a parabolic sub-sample refinement."""
    c = np.correlate(b, a, mode="full")
    i = int(np.argmax(c))
    y0, y1, y2 = c[i - 1], c[i], c[i + 1]
    return (i + 0.5 * (y0 - y2) / (y0 - 2 * y1 + y2) - (len(a) - 1)) * dt


def test_rayleigh_root_is_textbook_value():
    assert _rayleigh_ratio() == pytest.approx(0.919402, abs=2e-6)


@pytest.mark.slow
def test_surface_wave_travels_at_the_rayleigh_speed():
    nx, ny, nz, h, dt, fp = 128, 40, 40, 10.0, 1e-3, 8.0
    vs0 = 1000.0
    shape = (nz, ny, nx)
    vp = np.full(shape, np.sqrt(3.0) * vs0, np.float32)
    vs = np.full(shape, vs0, np.float32)
    rho = np.full(shape, 2000.0, np.float32)
    g = oracle.Grid(nx, ny, nz, h, dt, nb=12, free_surface=1, pml_f=fp)
    nt = 1050
    w = inputs.source_series("elastic", nt, dt, fp)
    xs = np.asarray([55, 95])  # 300 m and 700 m from the source at x = 25
    rec = np.stack([xs, np.full(2, ny // 2), np.zeros(2, int)], 1).astype(np.int32)
    seis = oracle.el_run(g, vp, vs, rho, oracle.el_state(g), 0, nt, [(25, ny // 2, 1)], w[:, None], rec,
                         component=2)  # vz on the surface row (k + 1/2 = 1/2)
    v = (xs[1] - xs[0]) * h / _lag(seis[:, 0], seis[:, 1], dt)
    ratio = v / vs0
    # the Rayleigh wave (0.9194 vs), not the S wave (vs) nor the P wave (1.73 vs)
    assert abs(ratio - _rayleigh_ratio()) < 0.02 * _rayleigh_ratio()
