"""fp64 CPU oracle of the paper's hot path (ctypes wrapper around liboracle.so).

TEST INFRASTRUCTURE ONLY.  Only ``tests/``, ``__graft_entry__.smoke()`` and
``bench.py``'s ``cpu_baseline`` / ``--impl reference`` legs may import this
package.  It shares no code with the CUDA product path
(``paper_conf_ppopp_qawasmehchc15_b200``) and the product path never imports it.

Every function follows a passage of the paper (Qawasmeh et al., PMAM'15,
``/root/reference/PAPER.md``, cited ``P:<line>``) or a reading recorded in
DESIGN.md §3 (labels O1..O19):

* ``iso_run``      Eq 1, P:123-129 (+ O3 source scaling, O6 damping layer)
* ``ac_run``       Eq 2, P:131-142 in 3D (+ O7 C-PML, O8 grid/buoyancy)
* ``el_run``       Eq 3, P:146-159 (+ O7 C-PML, O9 grid, O16 free surface)
* ``migrate``      Algorithm 1, imaging condition P:111 (O14, O15)
* ``lap``/``dstag`` the 8th-order operators, P:175 (O1)

Parity status of every function: pinned by tests/test_oracle_*.py,
except the absorbing-layer formulas (O6, O7) and the free surface (O16), whose
form the paper does not state: "parity unpinned" beyond the physics checks
(reflection level, normal-incidence reflection) listed there.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")


def build(force: bool = False) -> str:
    """Compile liboracle.so with gcc (-O2, OpenMP, no fast-math)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < max(
        os.path.getmtime(_SRC), os.path.getmtime(os.path.join(_HERE, "oracle.h"))
    ):
        cmd = ["gcc", "-O2", "-fopenmp", "-fPIC", "-shared", "-std=c11", "-D_DEFAULT_SOURCE",
               "-Wall", "-o", _LIB + ".tmp", _SRC, "-lm"]
        subprocess.check_call(cmd)
        os.replace(_LIB + ".tmp", _LIB)
    return _LIB


class _Grid(C.Structure):
    _fields_ = [("nx", C.c_int32), ("ny", C.c_int32), ("nz", C.c_int32),
                ("h", C.c_double), ("dt", C.c_double), ("nb", C.c_int32),
                ("free_surface", C.c_int32), ("pml_R", C.c_double), ("pml_f", C.c_double),
                ("periodic", C.c_int32), ("iso_pml", C.c_int32)]


class _Inj(C.Structure):
    _fields_ = [("n", C.c_int32), ("pos", C.POINTER(C.c_int32)), ("amp", C.POINTER(C.c_double))]


class _Rec(C.Structure):
    _fields_ = [("n", C.c_int32), ("pos", C.POINTER(C.c_int32)), ("component", C.c_int32)]


_lib = None


def _L():
    global _lib
    if _lib is None:
        _lib = C.CDLL(build())
        d = C.POINTER(C.c_double)
        f = C.POINTER(C.c_float)
        i32 = C.POINTER(C.c_int32)
        g = C.POINTER(_Grid)
        _lib.or_coef.argtypes = [d, d]
        _lib.or_lap.argtypes = [g, d, d]
        _lib.or_dstag.argtypes = [g, C.c_int, C.c_int, d, d]
        _lib.or_iso_eta.argtypes = [C.c_int, C.c_int, C.c_double, C.c_double, C.c_double, d]
        _lib.or_cpml.argtypes = [C.c_int, C.c_int, C.c_int, C.c_int, C.c_double, C.c_double,
                                 C.c_double, C.c_double, C.c_double, d, d, d, d]
        _lib.or_iso_run.argtypes = [g, f, d, d, d, C.c_int, C.c_int, C.POINTER(_Inj),
                                    C.POINTER(_Rec), d]
        _lib.or_ac_run.argtypes = [g, f, f, d, d, d, d, d, C.c_int, C.c_int, C.POINTER(_Inj),
                                   C.POINTER(_Rec), d]
        _lib.or_el_run.argtypes = [g, f, f, f, d, d, C.c_int, C.c_int, C.POINTER(_Inj),
                                   C.POINTER(_Rec), d]
        _lib.or_migrate.argtypes = [g, C.c_int, f, f, f, i32, d, C.c_int, C.c_int, i32, d,
                                    C.c_int, d]
        for fn in ("or_iso_run", "or_ac_run", "or_el_run", "or_migrate"):
            getattr(_lib, fn).restype = C.c_int
    return _lib


@dataclass
class Grid:
    """Grid description (mirrors the product's seis_grid; h, dt are rounded to fp32)."""
    nx: int
    ny: int
    nz: int
    h: float
    dt: float
    nb: int = 0
    free_surface: int = 0
    pml_R: float = 1e-3
    pml_f: float = 10.0
    periodic: int = 0
    iso_pml: int = 0  # ISO layer: 0 = damped wave (O6), 1 = split-field PML (O6b)

    def c(self) -> _Grid:
        return _Grid(self.nx, self.ny, self.nz, float(np.float32(self.h)),
                     float(np.float32(self.dt)), self.nb, self.free_surface,
                     float(np.float32(self.pml_R)), float(np.float32(self.pml_f)), self.periodic,
                     self.iso_pml)

    @property
    def shape(self):
        return (self.nz, self.ny, self.nx)


def _dp(a):
    assert a.dtype == np.float64 and a.flags.c_contiguous
    return a.ctypes.data_as(C.POINTER(C.c_double))


def _fp(a):
    assert a.dtype == np.float32 and a.flags.c_contiguous
    return a.ctypes.data_as(C.POINTER(C.c_float))


def _ip(a):
    assert a.dtype == np.int32 and a.flags.c_contiguous
    return a.ctypes.data_as(C.POINTER(C.c_int32))


def _check(rc, what):
    if rc != 0:
        raise ValueError(f"oracle {what} failed with code {rc}")


def coef():
    c = np.zeros(5)
    d = np.zeros(4)
    _L().or_coef(_dp(c), _dp(d))
    return c, d


def lap(grid: Grid, u):
    u = np.ascontiguousarray(u, dtype=np.float64)
    out = np.empty_like(u)
    g = grid.c()
    _L().or_lap(C.byref(g), _dp(u), _dp(out))
    return out


def dstag(grid: Grid, axis: int, plus: bool, f):
    f = np.ascontiguousarray(f, dtype=np.float64)
    out = np.empty_like(f)
    g = grid.c()
    _L().or_dstag(C.byref(g), axis, int(bool(plus)), _dp(f), _dp(out))
    return out


def iso_eta(N, nb, h, vmax, R):
    e = np.zeros(N)
    _L().or_iso_eta(N, nb, float(np.float32(h)), float(vmax), float(np.float32(R)), _dp(e))
    return e


def cpml(N, nb, lo, hi, h, dt, vmax, R, f):
    a, b, ah, bh = (np.zeros(N) for _ in range(4))
    _L().or_cpml(N, nb, int(lo), int(hi), float(np.float32(h)), float(np.float32(dt)),
                 float(vmax), float(np.float32(R)), float(np.float32(f)),
                 _dp(a), _dp(b), _dp(ah), _dp(bh))
    return a, b, ah, bh


def _lists(inj_pos, inj_amp, rec_pos, component=2):
    keep = []
    inj = None
    if inj_pos is not None:
        ip = np.ascontiguousarray(np.asarray(inj_pos, dtype=np.int32).reshape(-1, 3))
        ia = np.ascontiguousarray(np.asarray(inj_amp, dtype=np.float64).reshape(-1, ip.shape[0]))
        keep += [ip, ia]
        inj = _Inj(ip.shape[0], _ip(ip), _dp(ia))
    rec = None
    nrec = 0
    if rec_pos is not None:
        rp = np.ascontiguousarray(np.asarray(rec_pos, dtype=np.int32).reshape(-1, 3))
        keep.append(rp)
        nrec = rp.shape[0]
        rec = _Rec(nrec, _ip(rp), component)
    return inj, rec, nrec, keep


def _ptr(x, T):
    return C.byref(x) if x is not None else C.POINTER(T)()


def iso_state(grid: Grid):
    # w: split-field PML components (O6b) [level n-1, n][x, y, z], used inside the layers
    return {"u_prev": np.zeros(grid.shape), "u_cur": np.zeros(grid.shape),
            "w": np.zeros((2, 3) + grid.shape)}


def ac_state(grid: Grid):
    s = {k: np.zeros(grid.shape) for k in ("p", "qx", "qy", "qz")}
    s["psi"] = np.zeros((6,) + grid.shape)
    return s


def el_state(grid: Grid):
    return {"f": np.zeros((9,) + grid.shape), "psi": np.zeros((18,) + grid.shape)}


def iso_run(grid, vp, state, n0, nsteps, inj_pos=None, inj_amp=None, rec_pos=None):
    """Advance an ISO state {u_prev, u_cur} in place; return seis[nsteps][nrec]."""
    vp = np.ascontiguousarray(vp, dtype=np.float32)
    inj, rec, nrec, keep = _lists(inj_pos, inj_amp, rec_pos)
    seis = np.zeros((nsteps, max(nrec, 1)))
    g = grid.c()
    w = state.get("w")
    if w is None:
        w = state["w"] = np.zeros((2, 3) + grid.shape)
    rc = _L().or_iso_run(C.byref(g), _fp(vp), _dp(state["u_prev"]), _dp(state["u_cur"]), _dp(w), n0,
                         nsteps, _ptr(inj, _Inj), _ptr(rec, _Rec), _dp(seis))
    _check(rc, "iso_run")
    return seis[:, :nrec]


def ac_run(grid, vp, rho, state, n0, nsteps, inj_pos=None, inj_amp=None, rec_pos=None):
    """Advance an ACOUSTIC state {p, qx, qy, qz, psi} in place; return seis."""
    vp = np.ascontiguousarray(vp, dtype=np.float32)
    rho = np.ascontiguousarray(rho, dtype=np.float32)
    inj, rec, nrec, keep = _lists(inj_pos, inj_amp, rec_pos)
    seis = np.zeros((nsteps, max(nrec, 1)))
    g = grid.c()
    rc = _L().or_ac_run(C.byref(g), _fp(vp), _fp(rho), _dp(state["p"]), _dp(state["qx"]),
                        _dp(state["qy"]), _dp(state["qz"]), _dp(state["psi"]), n0, nsteps,
                        _ptr(inj, _Inj), _ptr(rec, _Rec), _dp(seis))
    _check(rc, "ac_run")
    return seis[:, :nrec]


def el_run(grid, vp, vs, rho, state, n0, nsteps, inj_pos=None, inj_amp=None, rec_pos=None,
           component=2):
    """Advance an ELASTIC state {f[9], psi[18]} in place; return seis."""
    vp = np.ascontiguousarray(vp, dtype=np.float32)
    vs = np.ascontiguousarray(vs, dtype=np.float32)
    rho = np.ascontiguousarray(rho, dtype=np.float32)
    inj, rec, nrec, keep = _lists(inj_pos, inj_amp, rec_pos, component)
    seis = np.zeros((nsteps, max(nrec, 1)))
    g = grid.c()
    rc = _L().or_el_run(C.byref(g), _fp(vp), _fp(vs), _fp(rho), _dp(state["f"]),
                        _dp(state["psi"]), n0, nsteps, _ptr(inj, _Inj), _ptr(rec, _Rec),
                        _dp(seis))
    _check(rc, "el_run")
    return seis[:, :nrec]


KIND = {"iso": 0, "acoustic": 1, "elastic": 2}


def forward_model(grid, kind, vp, rho=None, vs=None, src=None, wavelet=None, rec=None,
                  component=2):
    """Seismic modeling (Alg 1 forward phase) from a zero state.
    Returns (seis[nt][nrec], final state dict)."""
    wavelet = np.asarray(wavelet, dtype=np.float64)
    nt = wavelet.shape[0]
    if kind == "iso":
        st = iso_state(grid)
        seis = iso_run(grid, vp, st, 0, nt, [src], wavelet[:, None], rec)
    elif kind == "acoustic":
        st = ac_state(grid)
        seis = ac_run(grid, vp, rho, st, 0, nt, [src], wavelet[:, None], rec)
    else:
        st = el_state(grid)
        seis = el_run(grid, vp, vs, rho, st, 0, nt, [src], wavelet[:, None], rec, component)
    return seis, st


def migrate(grid, kind, vp, rho, src, wavelet, rec, data, snap, image=None, vs=None):
    """RTM (Alg 1) of one shot; returns image (accumulated into `image` if given).
    ELASTIC images the pressure -(sxx+syy+szz)/3 with explosive receiver injection."""
    vp = np.ascontiguousarray(vp, dtype=np.float32)
    rho = np.ascontiguousarray(rho if rho is not None else np.ones_like(vp), dtype=np.float32)
    vs = np.ascontiguousarray(vs if vs is not None else np.zeros_like(vp), dtype=np.float32)
    sp = np.ascontiguousarray(np.asarray(src, dtype=np.int32).reshape(3))
    amp = np.ascontiguousarray(np.asarray(wavelet, dtype=np.float64))
    rp = np.ascontiguousarray(np.asarray(rec, dtype=np.int32).reshape(-1, 3))
    dd = np.ascontiguousarray(np.asarray(data, dtype=np.float64))
    nt = amp.shape[0]
    assert dd.shape == (nt, rp.shape[0])
    if image is None:
        image = np.zeros(grid.shape)
    g = grid.c()
    rc = _L().or_migrate(C.byref(g), KIND[kind], _fp(vp), _fp(vs), _fp(rho), _ip(sp), _dp(amp), nt,
                         rp.shape[0], _ip(rp), _dp(dd), int(snap), _dp(image))
    _check(rc, "migrate")
    return image
