"""Pins of the oracle's RTM (Algorithm 1; imaging P:111) — CPU only.

* linearity of the image in the data, zero data => image unchanged, two calls
  accumulate (the sum over shots of P:111);
* brute force on a 16^3 grid, nt = 40, against an INDEPENDENT NumPy
  implementation of Eq 1 + the damping layer + Algorithm 1 (no oracle code);
* the acoustic migrate loop equals a manual composition of pinned single steps;
* physics: a flat reflector under a homogeneous overburden images at its depth.
"""
import math

import numpy as np
import pytest

import oracle
from paper_conf_ppopp_qawasmehchc15_b200 import inputs

# exact rationals of the 8th-order centred stencil (tests/golden/stencil_coefficients.txt)
_C = [-205 / 72, 8 / 5, -1 / 5, 8 / 315, -1 / 560]
C32 = [float(np.float32(c)) for c in _C]


def _setup(kind, n=16, nt=40, nb=3, seed=7):
    m = inputs.random_media((n, n, n), seed=seed)
    g = oracle.Grid(n, n, n, h=10.0, dt=6e-4, nb=nb, pml_f=30.0)
    w = inputs.source_series(kind, nt, 6e-4, 30.0)
    src = (8, 7, 5)
    rec = np.asarray([(3, 4, 4), (12, 9, 4), (6, 12, 4), (6, 12, 4)], np.int32)  # one duplicate
    rng = np.random.default_rng(seed + 1)
    data = rng.standard_normal((nt, rec.shape[0]))
    return m, g, w, src, rec, data


@pytest.mark.parametrize("kind", ["iso", "acoustic"])
def test_image_linear_in_data_and_accumulates(kind):
    m, g, w, src, rec, data = _setup(kind)
    rho = m["rho"] if kind == "acoustic" else None
    I1 = oracle.migrate(g, kind, m["vp"], rho, src, w, rec, data, 4)
    d2 = np.cos(data)
    I2 = oracle.migrate(g, kind, m["vp"], rho, src, w, rec, d2, 4)
    I12 = oracle.migrate(g, kind, m["vp"], rho, src, w, rec, 2.0 * data - 3.0 * d2, 4)
    assert np.abs(I12 - (2 * I1 - 3 * I2)).max() <= 1e-12 * np.abs(I12).max()
    # zero data leaves the image unchanged (bitwise)
    base = np.random.default_rng(3).standard_normal(g.shape)
    I0 = oracle.migrate(g, kind, m["vp"], rho, src, w, rec, np.zeros_like(data), 4, image=base.copy())
    assert np.array_equal(I0, base)
    # two calls accumulate (sum over shots) up to the rounding of the running sum
    acc = oracle.migrate(g, kind, m["vp"], rho, src, w, rec, data, 4)
    acc = oracle.migrate(g, kind, m["vp"], rho, src, w, rec, data, 4, image=acc)
    assert np.abs(acc - 2.0 * I1).max() <= 1e-14 * np.abs(I1).max()


# --------------------------------------------------- independent NumPy ISO RTM
def _np_iso_step(up, uc, m, eta, dt, amp_field):
    p = np.pad(uc, 4)
    n0, n1, n2 = uc.shape
    lap = 3 * C32[0] * uc
    for mm in range(1, 5):
        lap = lap + C32[mm] * (p[4 + mm:4 + mm + n0, 4:4 + n1, 4:4 + n2] + p[4 - mm:4 - mm + n0, 4:4 + n1, 4:4 + n2]
                               + p[4:4 + n0, 4 + mm:4 + mm + n1, 4:4 + n2] + p[4:4 + n0, 4 - mm:4 - mm + n1, 4:4 + n2]
                               + p[4:4 + n0, 4:4 + n1, 4 + mm:4 + mm + n2] + p[4:4 + n0, 4:4 + n1, 4 - mm:4 - mm + n2])
    return (2 * uc - (1 - eta * dt) * up + m * lap + amp_field) / (1 + eta * dt)


def _np_eta(n, nb, h, vmax, R):
    emax = 3 * vmax * math.log(1 / R) / (2 * nb * h)
    i = np.arange(n, dtype=np.float64)
    xi = np.maximum(0, np.maximum(nb - i, i - (n - 1 - nb))) / nb
    return emax * xi ** 2


def _np_iso_migrate(g, vp, src, w, rec, data, snap):
    h, dt = float(np.float32(g.h)), float(np.float32(g.dt))
    v = vp.astype(np.float64)
    m = v * v * dt * dt / (h * h)
    e1 = _np_eta(g.nx, g.nb, h, v.max(), float(np.float32(g.pml_R)))
    eta = e1[None, None, :] + e1[None, :, None] + e1[:, None, None]
    nt = len(w)

    def inj_field(pos_amp):
        f = np.zeros(g.shape)
        for (x, y, z), a in pos_amp:
            f[z, y, x] += v[z, y, x] ** 2 * dt * dt * a / h ** 3
        return f

    up, uc = np.zeros(g.shape), np.zeros(g.shape)
    S = {}
    for n in range(nt):
        un = _np_iso_step(up, uc, m, eta, dt, inj_field([(src, float(w[n]))]))
        up, uc = uc, un
        if (n + 1) % snap == 0 and n + 1 <= nt - 1:
            S[n + 1] = uc.copy()
    I = np.zeros(g.shape)
    up, uc = np.zeros(g.shape), np.zeros(g.shape)
    for mstep in range(nt):
        j = nt - mstep
        if j in S:
            I += S[j] * uc
        un = _np_iso_step(up, uc, m, eta, dt,
                          inj_field([(tuple(r), data[nt - 1 - mstep, i]) for i, r in enumerate(rec)]))
        up, uc = uc, un
    return I


def test_iso_migrate_matches_independent_numpy_bruteforce():
    m, g, w, src, rec, data = _setup("iso", n=16, nt=40, nb=3)
    I_or = oracle.migrate(g, "iso", m["vp"], None, src, w, rec, data, 4)
    I_np = _np_iso_migrate(g, m["vp"], src, w.astype(np.float64), rec, data, 4)
    assert np.abs(I_np).max() > 0
    assert np.abs(I_or - I_np).max() <= 1e-12 * np.abs(I_np).max()


def test_acoustic_migrate_equals_composition_of_steps():
    """Algorithm 1's loop (snapshot levels j = snap..nt-1, reversed data, imaging of
    S_j with R^{m+1}, j = nt-1-m; O14/O15) rebuilt from single pinned steps."""
    m, g, w, src, rec, data = _setup("acoustic", n=14, nt=30, nb=3)
    snap = 3
    I_or = oracle.migrate(g, "acoustic", m["vp"], m["rho"], src, w, rec, data, snap)
    st = oracle.ac_state(g)
    S = {}
    nt = len(w)
    for n in range(nt):
        oracle.ac_run(g, m["vp"], m["rho"], st, n, 1, [src], w[:, None])
        if (n + 1) % snap == 0 and n + 1 <= nt - 1:
            S[n + 1] = st["p"].copy()
    st = oracle.ac_state(g)
    back = data[::-1].copy()
    I = np.zeros(g.shape)
    for mm in range(nt):
        oracle.ac_run(g, m["vp"], m["rho"], st, mm, 1, rec, back)
        j = nt - 1 - mm
        if j in S:
            I += S[j] * st["p"]
    assert np.abs(I).max() > 0
    assert np.abs(I_or - I).max() <= 1e-12 * np.abs(I).max()


@pytest.mark.slow
def test_flat_reflector_images_at_its_depth():
    """Physics: reflector at z_r = 24 under a homogeneous overburden; data = shot on the true
    model minus shot on the smooth (reflector-free) model; migrate on the smooth model.
    The laterally summed image peaks within +-2 points of z_r."""
    n, zr, nt = 40, 24, 240
    h, dt, fp = 10.0, 1e-3, 20.0
    vp_true = np.full((n, n, n), 2000.0, np.float32)
    rho_true = np.full((n, n, n), 1000.0, np.float32)
    vp_true[zr:] = 2600.0
    rho_true[zr:] = 1600.0
    vp_s = np.full((n, n, n), 2000.0, np.float32)
    rho_s = np.full((n, n, n), 1000.0, np.float32)
    g = oracle.Grid(n, n, n, h=h, dt=dt, nb=8, pml_f=fp)
    w = inputs.source_series("acoustic", nt, dt, fp)
    src = (n // 2, n // 2, 9)
    xs = np.arange(9, n - 9, 2, dtype=np.int32)
    yy, xx = np.meshgrid(xs, xs, indexing="ij")
    rec = np.stack([xx.ravel(), yy.ravel(), np.full(xx.size, 9, np.int32)], axis=1)
    d_true, _ = oracle.forward_model(g, "acoustic", vp_true, rho=rho_true, src=src, wavelet=w, rec=rec)
    d_s, _ = oracle.forward_model(g, "acoustic", vp_s, rho=rho_s, src=src, wavelet=w, rec=rec)
    # the acoustic receiver injection uses the source scaling dt K d / h^3, i.e. it treats its
    # samples as d_t^{-1} of the wanted pressure (O11/O15): pass the time-integrated residual so
    # the receiver wavefield is in phase with the source wavefield.
    resid = np.cumsum(d_true - d_s, axis=0) * float(np.float32(dt))
    I = oracle.migrate(g, "acoustic", vp_s, rho_s, src, w, rec, resid, 4)
    prof = np.abs(I[:, 10:n - 10, 10:n - 10]).sum(axis=(1, 2))
    prof[:12] = 0  # exclude the source/receiver depth band
    assert abs(int(np.argmax(prof)) - zr) <= 2


def test_elastic_rtm_fluid_limit_equals_acoustic_rtm():
    """Elastic RTM (f3; pressure imaging, explosive receiver injection) with vs = 0 reduces
    exactly to acoustic RTM (O9 fluid limit applied to Algorithm 1)."""
    m, g, w, src, rec, data = _setup("acoustic", n=14, nt=30, nb=3)
    I_ac = oracle.migrate(g, "acoustic", m["vp"], m["rho"], src, w, rec, data, 3)
    I_el = oracle.migrate(g, "elastic", m["vp"], m["rho"], src, w, rec, data, 3,
                          vs=np.zeros_like(m["vp"]))
    assert np.abs(I_ac).max() > 0
    assert np.abs(I_el - I_ac).max() <= 1e-12 * np.abs(I_ac).max()


def test_elastic_rtm_linear_and_accumulates():
    m, g, w, src, rec, data = _setup("elastic", n=14, nt=30, nb=3)
    me = inputs.random_media((14, 14, 14), seed=7, elastic=True)
    I1 = oracle.migrate(g, "elastic", me["vp"], me["rho"], src, w, rec, data, 3, vs=me["vs"])
    I2 = oracle.migrate(g, "elastic", me["vp"], me["rho"], src, w, rec, 2.0 * data, 3, vs=me["vs"])
    assert np.abs(I1).max() > 0
    assert np.abs(I2 - 2 * I1).max() <= 1e-12 * np.abs(I2).max()
