"""GPU-vs-oracle parity at the CONFIGURED step counts (BASELINE.json north_star: "relative
L2 <= 1e-4 on wavefields and seismograms after the configured steps, and <= 1e-3 on RTM
images"; SURVEY §4 T1 "full steps for the record").

The BASELINE configurations C1-C4 at their full step counts, on grids the fp64 oracle
finishes in about a minute (C1 exactly; C2 / C3 / C4 with their recipes -- layered /
salt models, source and receiver geometry, absorbing layers nb = 20, free surface --
scaled to 96^3, see inputs.c1 .. c4):

* C1  ISO 64^3, homogeneous, 200 steps (exactly BASELINE configs[0]);
* C2  acoustic layered, C-PML on 6 faces, receiver line, 2000 steps;
* C3  elastic layered, free surface + C-PML on 5 faces, surface v_z line, 1500 steps;
* C4  acoustic RTM on the smoothed salt model, data = the oracle's own forward modeling on
      the true model, receiver carpet, snapshots every 20 steps, 2000 steps.

Every comparison reports the whole-array relative L2 AND the relative L2 over the points
of the absorbing layers only (where the C-PML memory variables act and the field is
~1e-3 of its peak, so a wrong psi term would hide in the whole-array norm); both must
meet the bar.  Equations: Eq 1-3, C-PML P:179, Algorithm 1,
imaging P:111.
"""
import numpy as np
import pytest

import oracle
import paper_conf_ppopp_qawasmehchc15_b200 as seis
from paper_conf_ppopp_qawasmehchc15_b200 import inputs
from gpu_common import TOL_FIELD, TOL_IMAGE, oracle_fields, rel_l2

pytestmark = pytest.mark.gpu

N = 96


def layer_mask(shape, nb, free_surface=False):
    """Points inside an absorbing layer (C-PML slab width W = nb + 1 on each face; a free
    surface top has none)."""
    nz, ny, nx = shape
    W = nb + 1
    z = np.arange(nz)[:, None, None]
    y = np.arange(ny)[None, :, None]
    x = np.arange(nx)[None, None, :]
    m = (x < W) | (x >= nx - W) | (y < W) | (y >= ny - W) | (z >= nz - W)
    if not free_surface:
        m = m | (z < W)
    return np.broadcast_to(m, shape)


def both_l2(a, b, mask):
    return rel_l2(a, b), rel_l2(np.asarray(a)[mask], np.asarray(b)[mask])


def _check_fields(name, got, ref, mask, tol):
    for t, (a, b) in enumerate(zip(got, ref)):
        whole, lay = both_l2(a, b, mask)
        print(f"{name} field {t}: rel L2 whole {whole:.2e}, layers {lay:.2e}")
        assert whole <= tol, (name, t, whole)
        assert lay <= tol, (name, t, lay)


def test_c1_exact_parity():
    wl = inputs.c1()
    assert (wl.nx, wl.nt, wl.nb) == (64, 200, 0)
    g = seis.Grid(wl.nx, wl.ny, wl.nz, wl.h, wl.dt, nb=wl.nb)
    m = seis.Model(g, "iso", wl.model["vp"])
    shot = seis.Shot(wl.src, wl.wavelet, wl.rec)
    out = np.zeros((wl.nt, shot.nrec), np.float32)
    m.forward_model(shot, out)
    fields = [m.get_field(f) for f in range(2)]
    m.close()
    og = oracle.Grid(wl.nx, wl.ny, wl.nz, wl.h, wl.dt, nb=wl.nb)
    st = oracle.iso_state(og)
    ref = oracle.iso_run(og, wl.model["vp"], st, 0, wl.nt, [wl.src], wl.wavelet[:, None], wl.rec)
    e = rel_l2(out, ref)
    print(f"C1 seismogram rel L2 {e:.2e}")
    assert e <= TOL_FIELD
    for a, b in zip(fields, oracle_fields("iso", st)):
        assert rel_l2(a, b) <= TOL_FIELD


def test_c2_recipe_2000_steps():
    wl = inputs.c2(n=N, nt=2000, nb=20)
    g = seis.Grid(wl.nx, wl.ny, wl.nz, wl.h, wl.dt, nb=wl.nb, pml_R=wl.pml_R, pml_f=wl.fp)
    m = seis.Model(g, "acoustic", wl.model["vp"], rho=wl.model["rho"])
    shot = seis.Shot(wl.src, wl.wavelet, wl.rec)
    out = np.zeros((wl.nt, shot.nrec), np.float32)
    m.forward_model(shot, out)
    fields = [m.get_field(f) for f in range(4)]
    m.close()
    og = oracle.Grid(wl.nx, wl.ny, wl.nz, wl.h, wl.dt, nb=wl.nb, pml_R=wl.pml_R, pml_f=wl.fp)
    st = oracle.ac_state(og)
    ref = oracle.ac_run(og, wl.model["vp"], wl.model["rho"], st, 0, wl.nt, [wl.src], wl.wavelet[:, None],
                        wl.rec)
    e = rel_l2(out, ref)
    print(f"C2 seismogram rel L2 {e:.2e}")
    assert e <= TOL_FIELD
    _check_fields("C2", fields, oracle_fields("acoustic", st), layer_mask(og.shape, wl.nb), TOL_FIELD)


def test_c3_recipe_1500_steps():
    wl = inputs.c3(n=N, nt=1500, nb=20)
    g = seis.Grid(wl.nx, wl.ny, wl.nz, wl.h, wl.dt, nb=wl.nb, free_surface=1, pml_R=wl.pml_R, pml_f=wl.fp)
    m = seis.Model(g, "elastic", wl.model["vp"], vs=wl.model["vs"], rho=wl.model["rho"])
    shot = seis.Shot(wl.src, wl.wavelet, wl.rec, rec_component=2)
    out = np.zeros((wl.nt, shot.nrec), np.float32)
    m.forward_model(shot, out)
    fields = [m.get_field(f) for f in range(9)]
    m.close()
    og = oracle.Grid(wl.nx, wl.ny, wl.nz, wl.h, wl.dt, nb=wl.nb, free_surface=1, pml_R=wl.pml_R, pml_f=wl.fp)
    st = oracle.el_state(og)
    ref = oracle.el_run(og, wl.model["vp"], wl.model["vs"], wl.model["rho"], st, 0, wl.nt, [wl.src],
                        wl.wavelet[:, None], wl.rec, component=2)
    e = rel_l2(out, ref)
    print(f"C3 seismogram rel L2 {e:.2e}")
    assert e <= TOL_FIELD
    _check_fields("C3", fields, oracle_fields("elastic", st), layer_mask(og.shape, wl.nb, True), TOL_FIELD)


def test_c4_recipe_rtm_2000_steps():
    torch = pytest.importorskip("torch")
    wl = inputs.c4(n=N, nt=2000, nb=20, snap=20)
    og = oracle.Grid(wl.nx, wl.ny, wl.nz, wl.h, wl.dt, nb=wl.nb, pml_R=wl.pml_R, pml_f=wl.fp)
    # observed data: the ORACLE's forward modeling on the true model (no input from the CUDA path)
    data, _ = oracle.forward_model(og, "acoustic", wl.model["vp"], rho=wl.model["rho"], src=wl.src,
                                   wavelet=wl.wavelet, rec=wl.rec)
    data32 = data.astype(np.float32)
    mig = inputs.smooth(wl.model, 5.0 * N / 512.0)
    ref = oracle.migrate(og, "acoustic", mig["vp"], mig["rho"], wl.src, wl.wavelet, wl.rec,
                         data32.astype(np.float64), wl.snap)
    g = seis.Grid(wl.nx, wl.ny, wl.nz, wl.h, wl.dt, nb=wl.nb, pml_R=wl.pml_R, pml_f=wl.fp)
    m = seis.Model(g, "acoustic", mig["vp"], rho=mig["rho"])
    img = torch.zeros(og.shape, device="cuda:0")
    m.migrate(seis.Shot(wl.src, wl.wavelet, wl.rec, snap_period=wl.snap), torch.from_numpy(data32).cuda(), img)
    m.close()
    got = img.cpu().numpy()
    whole, lay = both_l2(got, ref, layer_mask(og.shape, wl.nb))
    print(f"C4 image ({wl.rec.shape[0]} receivers, {(wl.nt - 1) // wl.snap} snapshots): "
          f"rel L2 whole {whole:.2e}, layers {lay:.2e}")
    assert whole <= TOL_IMAGE
    assert lay <= TOL_IMAGE
