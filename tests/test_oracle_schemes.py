"""Pins of the oracle's time-stepping schemes against closed forms and invariants — CPU only.

Equations: Eq 1 (§3.3.1), Eq 2 (§3.3.2), Eq 3
(§3.3.3).  None of these checks re-types the oracle's update: each
one is a different mathematical statement the update must satisfy --
* exact discrete plane waves (numerical-dispersion relation, O4),
* discrete energy conservation with absorbing boundaries off (O3, O8, O9),
* source-receiver reciprocity (O3, O8),
* the homogeneous-medium analytic Green's function (O3, O8; also pins the
  recording convention O13 and the source scaling O11),
* the elastic fluid limit mu = 0 == acoustic (O9).
"""
import math

import numpy as np
import pytest

import oracle
from paper_conf_ppopp_qawasmehchc15_b200 import inputs


def _c():
    return oracle.coef()


# ------------------------------------------------------------ dispersion (O4)
def test_iso_dispersion_exact_plane_wave():
    """u^n = cos(k.x - w n dt) with sin^2(w dt/2) = (v dt/2)^2 sum_d -(c0 + 2 sum c_m cos(m k_d h))/h^2
    is an exact solution of the leapfrog scheme on a periodic grid."""
    n, h, dt, v = 16, 10.0, 1e-3, 2000.0
    g = oracle.Grid(n, n, n, h=h, dt=dt, periodic=1)
    h, dt = float(np.float32(h)), float(np.float32(dt))
    c, _ = _c()
    jk = (1, 2, 3)
    k = [2 * math.pi * j / (n * h) for j in jk]
    sym = sum(-(c[0] + 2 * sum(c[m] * math.cos(m * kd * h) for m in range(1, 5))) / h ** 2 for kd in k)
    w = 2.0 / dt * math.asin(v * dt / 2.0 * math.sqrt(sym))
    z, y, x = np.meshgrid(np.arange(n) * h, np.arange(n) * h, np.arange(n) * h, indexing="ij")
    phase = k[0] * x + k[1] * y + k[2] * z
    st = {"u_prev": np.cos(phase + w * dt), "u_cur": np.cos(phase)}
    vp = np.full((n, n, n), v, np.float32)
    nsteps = 500
    oracle.iso_run(g, vp, st, 0, nsteps)
    ref = np.cos(phase - w * nsteps * dt)
    assert np.abs(st["u_cur"] - ref).max() < 1e-10


def _stag_S(d, kd, h):
    return sum(d[m - 1] * math.sin((m - 0.5) * kd * h) for m in range(1, 5))


def test_acoustic_dispersion_exact_plane_wave():
    """p^n = cos(k.x - w n dt), q_d^{n-1/2} = Q_d cos(k.(x + h/2 e_d) - w (n-1/2) dt) with
    sin(w dt/2) = (v dt/h) sqrt(sum_d S_d^2), S_d = sum_m d_m sin((m-1/2) k_d h),
    Q_d = -b (dt/h) S_d / sin(w dt/2): exact on a periodic grid (O4)."""
    n, h, dt, v, rho = 16, 10.0, 8e-4, 3000.0, 1800.0
    g = oracle.Grid(n, n, n, h=h, dt=dt, periodic=1)
    h, dt = float(np.float32(h)), float(np.float32(dt))
    _, d = _c()
    jk = (1, 3, 2)
    k = [2 * math.pi * j / (n * h) for j in jk]
    S = [_stag_S(d, kd, h) for kd in k]
    s = v * dt / h * math.sqrt(sum(x * x for x in S))
    w = 2.0 / dt * math.asin(s)
    b = 1.0 / float(np.float32(rho))
    z, y, x = np.meshgrid(np.arange(n) * h, np.arange(n) * h, np.arange(n) * h, indexing="ij")
    X = [x, y, z]
    phase = k[0] * x + k[1] * y + k[2] * z
    Q = [-b * (dt / h) * Sd / math.sin(w * dt / 2) for Sd in S]
    st = oracle.ac_state(g)
    st["p"][:] = np.cos(phase)
    for ax, key in enumerate(("qx", "qy", "qz")):
        st[key][:] = Q[ax] * np.cos(phase + k[ax] * h / 2 + w * dt / 2)
    vp = np.full((n, n, n), v, np.float32)
    rr = np.full((n, n, n), rho, np.float32)
    nsteps = 500
    oracle.ac_run(g, vp, rr, st, 0, nsteps)
    assert np.abs(st["p"] - np.cos(phase - w * nsteps * dt)).max() < 1e-10
    for ax, key in enumerate(("qx", "qy", "qz")):
        ref = Q[ax] * np.cos(phase + k[ax] * h / 2 - w * (nsteps - 0.5) * dt)
        assert np.abs(st[key] - ref).max() < 1e-10 * max(abs(Q[ax]), 1e-30) + 1e-18


# field index in the elastic state and its staggering offset (x, y, z)
EL = {"vx": (0, (0.5, 0, 0)), "vy": (1, (0, 0.5, 0)), "vz": (2, (0, 0, 0.5)),
      "sxx": (3, (0, 0, 0)), "syy": (4, (0, 0, 0)), "szz": (5, (0, 0, 0)),
      "sxy": (6, (0.5, 0.5, 0)), "sxz": (7, (0.5, 0, 0.5)), "syz": (8, (0, 0.5, 0.5))}


@pytest.mark.parametrize("axis", [0, 1, 2])
@pytest.mark.parametrize("wave", ["P", "S1", "S2"])
def test_elastic_dispersion_exact_plane_wave(axis, wave):
    """Elastic plane waves along each axis: sin(w dt/2) = (c dt/h) S_axis with c = vp (P) or
    vs (S, both polarisations); amplitude ratios from the staggered system (O4, O9)."""
    nl, nt_, h, dt = 16, 4, 10.0, 6e-4
    vp_, vs_, rho_ = 3000.0, 1700.0, 2200.0
    dims = [nt_, nt_, nt_]
    dims[axis] = nl
    nx, ny, nz = dims
    g = oracle.Grid(nx, ny, nz, h=h, dt=dt, periodic=1)
    h, dt = float(np.float32(h)), float(np.float32(dt))
    vp32, vs32, r32 = (float(np.float32(a)) for a in (vp_, vs_, rho_))
    mu = r32 * vs32 ** 2
    lam = r32 * (vp32 ** 2 - 2 * vs32 ** 2)
    _, d = _c()
    kk = 2 * math.pi * 2 / (nl * h)
    S = _stag_S(d, kk, h)
    ax = "xyz"[axis]
    c = vp32 if wave == "P" else vs32
    w = 2.0 / dt * math.asin(c * dt / h * S)
    sn = math.sin(w * dt / 2)
    # stress amplitude 1 on the driving stress, velocity amplitude from dv/dt = b D sigma
    if wave == "P":
        vel = "v" + ax
        drive = {"s" + ax + ax: 1.0}
        others = {"s" + o + o: lam / (lam + 2 * mu) for o in "xyz" if o != ax}
        drive.update(others)
        V = -(dt / h) * S / sn / r32  # from the s_aa equation
    else:
        pol = [o for o in "xyz" if o != ax][0 if wave == "S1" else 1]
        vel = "v" + pol
        key = "s" + "".join(sorted(ax + pol))
        drive = {key: 1.0}
        V = -(dt / h) * S / sn / r32
    z, y, x = np.meshgrid(np.arange(nz), np.arange(ny), np.arange(nx), indexing="ij")
    coords = [x, y, z]
    st = oracle.el_state(g)

    def field(name, amp, t):
        idx, off = EL[name]
        pos = (coords[axis] + off[axis]) * h
        return amp * np.cos(kk * pos - w * t)

    # sigma at t = 0, v at t = -dt/2
    for name, amp in drive.items():
        st["f"][EL[name][0]] = field(name, amp, 0.0)
    st["f"][EL[vel][0]] = field(vel, V, -dt / 2)
    vpa = np.full(g.shape, vp_, np.float32)
    vsa = np.full(g.shape, vs_, np.float32)
    ra = np.full(g.shape, rho_, np.float32)
    nsteps = 300
    oracle.el_run(g, vpa, vsa, ra, st, 0, nsteps)
    T = nsteps * dt
    for name, amp in drive.items():
        assert np.abs(st["f"][EL[name][0]] - field(name, amp, T)).max() < 1e-9, name
    assert np.abs(st["f"][EL[vel][0]] - field(vel, V, T - dt / 2)).max() < 1e-9 * abs(V)
    for name, (idx, _) in EL.items():
        if name not in drive and name != vel:
            assert np.abs(st["f"][idx]).max() == 0.0, name


# ---------------------------------------------------------------- energy
def _np_lap(u, c):
    """Independent NumPy 25-point Laplacian (zero ghosts) for the energy functional."""
    p = np.pad(u, 4)
    n0, n1, n2 = u.shape
    out = 3 * c[0] * u
    for m in range(1, 5):
        for ax in range(3):
            sl_p = [slice(4, 4 + n0), slice(4, 4 + n1), slice(4, 4 + n2)]
            sl_m = list(sl_p)
            sl_p[ax] = slice(4 + m, 4 + m + u.shape[ax])
            sl_m[ax] = slice(4 - m, 4 - m + u.shape[ax])
            out = out + c[m] * (p[tuple(sl_p)] + p[tuple(sl_m)])
    return out


def test_iso_energy_conserved_without_absorbing_layer():
    """E^{n+1/2} = sum (1/v^2) ((u^{n+1}-u^n)/dt)^2 - sum u^{n+1} Lambda u^n / h^2 is constant
    once the source has died (eta = 0, zero-Dirichlet ghosts), random heterogeneous medium."""
    n = 20
    m = inputs.random_media((n, n, n))
    g = oracle.Grid(n, n, n, h=10.0, dt=6e-4)
    h, dt = float(np.float32(10.0)), float(np.float32(6e-4))
    c, _ = _c()
    fp = 40.0
    nt_src = int(3.2 / fp / dt) + 2
    w = inputs.source_series("iso", nt_src, dt, fp)
    st = oracle.iso_state(g)
    oracle.iso_run(g, m["vp"], st, 0, nt_src, [(7, 9, 11)], w[:, None])
    v2 = m["vp"].astype(np.float64) ** 2
    E = []
    for _ in range(6):
        oracle.iso_run(g, m["vp"], st, 0, 40)
        un, un1 = st["u_prev"], st["u_cur"]
        E.append(np.sum(((un1 - un) / dt) ** 2 / v2) - np.sum(un1 * _np_lap(un, c)) / h ** 2)
    E = np.asarray(E)
    assert E[0] > 0
    assert np.abs(E / E[0] - 1).max() < 1e-12


def _faces_b(rho, ax):
    r = rho.astype(np.float64)
    nxt = np.concatenate([np.take(r, range(1, r.shape[ax]), axis=ax),
                          np.take(r, [r.shape[ax] - 1], axis=ax)], axis=ax)
    return 2.0 / (r + nxt)


def test_acoustic_energy_conserved_without_absorbing_layer():
    """E^n = 1/2 sum p^2/K + 1/2 sum_d q_d^{n-1/2} q_d^{n+1/2} / b_d is constant after the source
    (O8; buoyancy 2/(rho_i + rho_i+1) on faces)."""
    n = 18
    m = inputs.random_media((n, n, n))
    g = oracle.Grid(n, n, n, h=10.0, dt=6e-4)
    dt = float(np.float32(6e-4))
    fp = 40.0
    nt_src = int(3.2 / fp / dt) + 2
    w = inputs.source_series("acoustic", nt_src, dt, fp)
    st = oracle.ac_state(g)
    oracle.ac_run(g, m["vp"], m["rho"], st, 0, nt_src, [(5, 8, 10)], w[:, None])
    K = m["rho"].astype(np.float64) * m["vp"].astype(np.float64) ** 2
    B = [_faces_b(m["rho"], 2), _faces_b(m["rho"], 1), _faces_b(m["rho"], 0)]  # x, y, z faces
    E = []
    for _ in range(5):
        oracle.ac_run(g, m["vp"], m["rho"], st, 0, 30)
        p_n = st["p"].copy()
        q_old = [st[k].copy() for k in ("qx", "qy", "qz")]
        st2 = {k: v.copy() for k, v in st.items()}
        oracle.ac_run(g, m["vp"], m["rho"], st2, 0, 1)
        e = 0.5 * np.sum(p_n ** 2 / K)
        for ax, key in enumerate(("qx", "qy", "qz")):
            e += 0.5 * np.sum(q_old[ax] * st2[key] / B[ax])
        E.append(e)
    E = np.asarray(E)
    assert E[0] > 0
    assert np.abs(E / E[0] - 1).max() < 1e-12


# ----------------------------------------------------------- reciprocity
@pytest.mark.parametrize("nb", [0, 4])
def test_iso_reciprocity(nb):
    """u_{A->B}(t) = u_{B->A}(t) with the v^2 f source scaling of Eq 1 (O3); also with the
    damping layer (the damping is diagonal, the weighted operator stays symmetric)."""
    n = 20
    m = inputs.random_media((n, n, n))
    g = oracle.Grid(n, n, n, h=10.0, dt=6e-4, nb=nb)
    w = inputs.source_series("iso", 120, 6e-4, 30.0)
    A, B = (4, 6, 9), (14, 11, 7)
    st = oracle.iso_state(g)
    ab = oracle.iso_run(g, m["vp"], st, 0, 120, [A], w[:, None], [B])
    st = oracle.iso_state(g)
    ba = oracle.iso_run(g, m["vp"], st, 0, 120, [B], w[:, None], [A])
    assert np.abs(ab).max() > 0
    assert np.abs(ab - ba).max() <= 1e-12 * np.abs(ab).max()


def test_acoustic_reciprocity():
    """p_{A->B}(t) = p_{B->A}(t) in a variable-density medium (O8), no C-PML."""
    n = 18
    m = inputs.random_media((n, n, n))
    g = oracle.Grid(n, n, n, h=10.0, dt=6e-4)
    w = inputs.source_series("acoustic", 120, 6e-4, 30.0)
    A, B = (3, 7, 8), (13, 10, 12)
    st = oracle.ac_state(g)
    ab = oracle.ac_run(g, m["vp"], m["rho"], st, 0, 120, [A], w[:, None], [B])
    st = oracle.ac_state(g)
    ba = oracle.ac_run(g, m["vp"], m["rho"], st, 0, 120, [B], w[:, None], [A])
    assert np.abs(ab).max() > 0
    assert np.abs(ab - ba).max() <= 1e-12 * np.abs(ab).max()


# --------------------------------------------------------- Green's function
def _green_setup(kind):
    n, h, dt, v, fp, nt = 64, 10.0, 1e-3, 2000.0, 15.0, 200
    c = n // 2
    recs = [(c + 5, c, c), (c + 10, c, c), (c + 15, c, c), (c + 6, c + 6, c + 6)]
    g = oracle.Grid(n, n, n, h=h, dt=dt)
    w = inputs.source_series(kind, nt, dt, fp)
    return g, n, h, dt, v, fp, nt, c, recs, w


def _rel(a, b):
    return np.linalg.norm(a - b) / np.linalg.norm(b)


@pytest.mark.slow
def test_iso_green_function_and_recording_convention():
    """u(r,t) = w(t - r/c)/(4 pi r) in a homogeneous medium (Eq 1 with f = w delta/h^3, O3);
    seis[n] = u^{n+1} is compared with the analytic value at (n+1) dt (O13): lag 0 matches
    to < 1e-2, a one-step lag does not."""
    g, n, h, dt, v, fp, nt, c, recs, w = _green_setup("iso")
    vp = np.full(g.shape, v, np.float32)
    st = oracle.iso_state(g)
    seis = oracle.iso_run(g, vp, st, 0, nt, [(c, c, c)], w[:, None], recs)
    hh, dd = float(np.float32(h)), float(np.float32(dt))
    t = (np.arange(nt) + 1) * dd
    for r_i, rp in enumerate(recs):
        r = hh * math.sqrt(sum((a - c) ** 2 for a in rp))
        ana = inputs.ricker(t - r / v, fp) / (4 * math.pi * r)
        assert _rel(seis[:, r_i], ana) < 1e-2, (rp, _rel(seis[:, r_i], ana))
        ana_lag = inputs.ricker(t - dd - r / v, fp) / (4 * math.pi * r)
        assert _rel(seis[:, r_i], ana_lag) > 5e-2


@pytest.mark.slow
def test_acoustic_green_function():
    """p(r,t) = rho w(t - r/c)/(4 pi r) for Eq 2 with the rho v^2 d_t^{-1} f source
    (s[n] = G((n+1/2) dt), O8/O11), homogeneous medium."""
    g, n, h, dt, v, fp, nt, c, recs, w = _green_setup("acoustic")
    rho = 1000.0
    vp = np.full(g.shape, v, np.float32)
    rr = np.full(g.shape, rho, np.float32)
    st = oracle.ac_state(g)
    seis = oracle.ac_run(g, vp, rr, st, 0, nt, [(c, c, c)], w[:, None], recs)
    hh, dd = float(np.float32(h)), float(np.float32(dt))
    t = (np.arange(nt) + 1) * dd
    for r_i, rp in enumerate(recs):
        r = hh * math.sqrt(sum((a - c) ** 2 for a in rp))
        ana = rho * inputs.ricker(t - r / v, fp) / (4 * math.pi * r)
        assert _rel(seis[:, r_i], ana) < 1e-2, (rp, _rel(seis[:, r_i], ana))


# ------------------------------------------------------------ fluid limit
@pytest.mark.parametrize("nb", [0, 4])
def test_elastic_fluid_limit_equals_acoustic(nb):
    """vs = 0: the elastic scheme reduces exactly to the acoustic one with
    sigma_xx = sigma_yy = sigma_zz = -p, v = -q (O9), C-PML included."""
    n = 16
    m = inputs.random_media((n, n, n))
    vs = np.zeros_like(m["vp"])
    g = oracle.Grid(n, n, n, h=10.0, dt=6e-4, nb=nb, pml_f=30.0)
    w = inputs.source_series("elastic", 60, 6e-4, 30.0)
    rec = [(3, 4, 5), (12, 9, 10), (8, 8, 8)]
    ea = oracle.el_state(g)
    se = oracle.el_run(g, m["vp"], vs, m["rho"], ea, 0, 60, [(8, 7, 6)], w[:, None], rec,
                       component=3)
    aa = oracle.ac_state(g)
    sa = oracle.ac_run(g, m["vp"], m["rho"], aa, 0, 60, [(8, 7, 6)], w[:, None], rec)
    scale = np.abs(aa["p"]).max()
    assert scale > 0
    for t in (3, 4, 5):
        assert np.abs(ea["f"][t] + aa["p"]).max() <= 1e-12 * scale
    for t, key in enumerate(("qx", "qy", "qz")):
        qs = np.abs(aa[key]).max()
        assert np.abs(ea["f"][t] + aa[key]).max() <= 1e-12 * qs
    for t in (6, 7, 8):
        assert np.abs(ea["f"][t]).max() == 0.0
    assert np.abs(se - sa).max() <= 1e-12 * np.abs(sa).max()


def test_elastic_energy_conserved_without_absorbing_layer():
    """E^n = 1/2 sum sigma_n^T C^{-1} sigma_n + 1/2 sum_shear sigma^2/mu_edge
    + 1/2 sum rho_face v^{n-1/2} v^{n+1/2} is constant after the source (O9, free surface off)."""
    n = 14
    m = inputs.random_media((n, n, n), elastic=True)
    g = oracle.Grid(n, n, n, h=10.0, dt=5e-4)
    dt = float(np.float32(5e-4))
    fp = 40.0
    nt_src = int(3.2 / fp / dt) + 2
    w = inputs.source_series("elastic", nt_src, dt, fp)
    st = oracle.el_state(g)
    oracle.el_run(g, m["vp"], m["vs"], m["rho"], st, 0, nt_src, [(6, 7, 8)], w[:, None])
    vp, vs, rho = (m[k].astype(np.float64) for k in ("vp", "vs", "rho"))
    mu = rho * vs ** 2
    lam = rho * (vp ** 2 - 2 * vs ** 2)

    def nxt(a, ax):
        return np.concatenate([np.take(a, range(1, a.shape[ax]), axis=ax),
                               np.take(a, [a.shape[ax] - 1], axis=ax)], axis=ax)

    def edge_mu(a1, a2):
        m1 = nxt(mu, a1)
        m2 = nxt(mu, a2)
        m12 = nxt(nxt(mu, a1), a2)
        return 4.0 / (1 / mu + 1 / m1 + 1 / m2 + 1 / m12)

    # numpy axes: z=0, y=1, x=2
    mu_xy, mu_xz, mu_yz = edge_mu(2, 1), edge_mu(2, 0), edge_mu(1, 0)
    rface = [(rho + nxt(rho, ax)) / 2.0 for ax in (2, 1, 0)]  # 1/b = (rho_i + rho_i+1)/2
    Cm = np.zeros(g.shape + (3, 3))
    for a in range(3):
        for b in range(3):
            Cm[..., a, b] = lam + (2 * mu if a == b else 0)
    Cinv = np.linalg.inv(Cm)
    E = []
    for _ in range(4):
        oracle.el_run(g, m["vp"], m["vs"], m["rho"], st, 0, 30)
        f_old = st["f"].copy()
        st2 = {k: v.copy() for k, v in st.items()}
        oracle.el_run(g, m["vp"], m["vs"], m["rho"], st2, 0, 1)
        sn = np.stack([f_old[3], f_old[4], f_old[5]], axis=-1)
        e = 0.5 * np.sum(np.einsum("...a,...ab,...b->...", sn, Cinv, sn))
        e += 0.5 * np.sum(f_old[6] ** 2 / mu_xy + f_old[7] ** 2 / mu_xz + f_old[8] ** 2 / mu_yz)
        for t in range(3):
            e += 0.5 * np.sum(rface[t] * f_old[t] * st2["f"][t])
        E.append(e)
    E = np.asarray(E)
    assert E[0] > 0
    assert np.abs(E / E[0] - 1).max() < 1e-11


# ----------------------------------------------------------- free surface (O16)
def test_free_surface_equals_mirrored_full_space():
    """Normal incidence on the stress-imaging free surface (O16): a laterally uniform
    P (vz, szz, sxx, syy) and S (vx, sxz) pulse in a half space with a free top must equal
    the full-space solution started from the odd/even mirror image of the initial data
    (szz, sxx, syy, sxz, syz odd; vx, vy, vz even about the surface plane), i.e. the surface
    reflects with R_sigma = -1 and doubles the surface velocity, exactly."""
    nh, h, dt = 80, 10.0, 1e-3
    vp_, vs_, r_ = 3000.0, 1700.0, 2200.0
    gh = oracle.Grid(4, 4, nh, h=h, dt=dt, free_surface=1, periodic=1)
    gf = oracle.Grid(4, 4, 2 * nh, h=h, dt=dt, periodic=1)
    k = np.arange(nh, dtype=np.float64)
    prof = np.exp(-((k - 10.0) / 3.0) ** 2)
    prof2 = np.exp(-((k - 14.0) / 2.5) ** 2) * np.sin(k / 3.0)
    half = oracle.el_state(gh)
    init = {2: prof, 5: prof2, 0: prof2, 7: prof}  # vz, szz, vx, sxz
    for f, pr in init.items():
        pr = pr.copy()
        if f == 5:
            pr[0] = 0.0  # an odd integer-z field vanishes on the surface plane
        half["f"][f] = pr[:, None, None] * np.ones((1, 4, 4))
    full = oracle.el_state(gf)
    odd = {3, 4, 5, 7, 8}
    halfz = {2, 7, 8}
    for f in range(9):
        s = -1.0 if f in odd else 1.0
        src = half["f"][f][:, 0, 0]
        col = np.zeros(2 * nh)
        col[nh:] = src
        if f in halfz:
            col[nh - 1 - np.arange(nh)] = s * src
        else:
            col[nh - np.arange(1, nh)] = s * src[1:]
        full["f"][f] = col[:, None, None] * np.ones((1, 4, 4))
    vp = lambda g: np.full(g.shape, vp_, np.float32)
    vs = lambda g: np.full(g.shape, vs_, np.float32)
    rr = lambda g: np.full(g.shape, r_, np.float32)
    nsteps = 100
    surf = oracle.el_run(gh, vp(gh), vs(gh), rr(gh), half, 0, nsteps, rec_pos=[(0, 0, 0)], component=2)
    oracle.el_run(gf, vp(gf), vs(gf), rr(gf), full, 0, nsteps)
    cmp = slice(0, 24)
    for f in range(9):
        a = half["f"][f][cmp, 0, 0]
        b = full["f"][f][nh:nh + 24, 0, 0]
        scale = max(np.abs(full["f"][f]).max(), 1e-30)
        assert np.abs(a - b).max() <= 1e-10 * scale, f
    # the pulse did reach the surface: surface vz peaks at about twice the incident amplitude
    assert np.abs(surf).max() > 0.5
