"""Shared helpers of the GPU parity tests (CUDA path through the C ABI vs the fp64 oracle)."""
import numpy as np

import oracle
import paper_conf_ppopp_qawasmehchc15_b200 as seis
from paper_conf_ppopp_qawasmehchc15_b200 import inputs

# Tolerances (BASELINE.json north_star): relative L2 over the whole array
TOL_FIELD = 1e-4
TOL_IMAGE = 1e-3


def rel_l2(a, b):
    a = np.asarray(a, dtype=np.float64)
    b = np.asarray(b, dtype=np.float64)
    nb = np.linalg.norm(b)
    assert nb > 0, "reference is identically zero"
    return float(np.linalg.norm(a - b) / nb)


def grids(nx, ny, nz, h, dt, nb=0, free_surface=0, pml_f=10.0, slabs=1, pml_R=1e-3):
    return (seis.Grid(nx, ny, nz, h, dt, nb=nb, free_surface=free_surface, pml_R=pml_R,
                      pml_f=pml_f, slabs=slabs),
            oracle.Grid(nx, ny, nz, h, dt, nb=nb, free_surface=free_surface, pml_R=pml_R,
                        pml_f=pml_f))


def gpu_forward(kind, g, model, src, wavelet, rec, component=2, device=0):
    m = seis.Model(g, kind, model["vp"], vs=model.get("vs"), rho=model.get("rho"), device=device)
    shot = seis.Shot(src, wavelet, rec, rec_component=component)
    out = np.zeros((shot.nt, shot.nrec), np.float32)
    m.forward_model(shot, out)
    nf = {"iso": 2, "acoustic": 4, "elastic": 9}[kind]
    fields = [m.get_field(f) for f in range(nf)]
    m.close()
    return out, fields


def oracle_fields(kind, st):
    if kind == "iso":
        return [st["u_cur"], st["u_prev"]]
    if kind == "acoustic":
        return [st["p"], st["qx"], st["qy"], st["qz"]]
    return [st["f"][t] for t in range(9)]
