"""GPU edge cases through the C ABI against the fp64 oracle: degenerate and ragged grids
(a single point, one-point-thin axes, sizes below one tile), no receivers, one time step,
sources / receivers on the corners, absorbing layers as wide as allowed (3 nb = min dim),
RTM without any snapshot level, and zero data.

Bars as in test_parity_gpu.py (relative L2 <= 1e-4 fields / seismograms, <= 1e-3 images).
"""
import numpy as np
import pytest

import oracle
import paper_conf_ppopp_qawasmehchc15_b200 as seis
from paper_conf_ppopp_qawasmehchc15_b200 import inputs
from gpu_common import TOL_FIELD, TOL_IMAGE, oracle_fields, rel_l2

pytestmark = pytest.mark.gpu

H, DT, FP = 10.0, 5e-4, 35.0


def _run_oracle(kind, og, m, src, w, rec, comp=2):
    if kind == "iso":
        st = oracle.iso_state(og)
        s = oracle.iso_run(og, m["vp"], st, 0, w.shape[0], [src], w[:, None], rec)
    elif kind == "acoustic":
        st = oracle.ac_state(og)
        s = oracle.ac_run(og, m["vp"], m["rho"], st, 0, w.shape[0], [src], w[:, None], rec)
    else:
        st = oracle.el_state(og)
        s = oracle.el_run(og, m["vp"], m["vs"], m["rho"], st, 0, w.shape[0], [src], w[:, None], rec,
                          component=comp)
    return s, oracle_fields(kind, st)


def _compare(kind, shape, nb=0, fs=0, nt=30, src=None, rec=None, seed=31):
    nz, ny, nx = shape
    m = inputs.random_media(shape, seed=seed, elastic=(kind == "elastic"))
    w = inputs.source_series(kind, nt, DT, FP)
    src = src if src is not None else (nx // 2, ny // 2, nz // 2)
    rec = np.zeros((0, 3), np.int32) if rec is None else np.asarray(rec, np.int32).reshape(-1, 3)
    g = seis.Grid(nx, ny, nz, H, DT, nb=nb, free_surface=fs, pml_f=FP)
    mod = seis.Model(g, kind, m["vp"], vs=m.get("vs"), rho=m.get("rho"))
    shot = seis.Shot(src, w, rec, rec_component=2)
    out = np.zeros((nt, rec.shape[0]), np.float32)
    mod.forward_model(shot, out if rec.shape[0] else None)
    nf = {"iso": 2, "acoustic": 4, "elastic": 9}[kind]
    fields = [mod.get_field(f) for f in range(nf)]
    mod.close()
    og = oracle.Grid(nx, ny, nz, H, DT, nb=nb, free_surface=fs, pml_f=FP)
    s_o, f_o = _run_oracle(kind, og, m, src, w, rec)
    if rec.shape[0]:
        assert rel_l2(out, s_o) <= TOL_FIELD
    for a, b in zip(fields, f_o):
        if np.linalg.norm(b) > 0:
            assert rel_l2(a, b) <= TOL_FIELD
        else:
            assert np.all(a == 0)


@pytest.mark.parametrize("kind", ["iso", "acoustic", "elastic"])
@pytest.mark.parametrize("shape", [(1, 1, 1), (9, 3, 5), (17, 1, 65), (12, 70, 1), (3, 40, 67)])
def test_degenerate_and_ragged_grids(kind, shape):
    nz, ny, nx = shape
    rec = [[0, 0, 0], [nx - 1, ny - 1, nz - 1], [nx // 2, ny // 2, nz // 2]]
    _compare(kind, shape, rec=rec)


@pytest.mark.parametrize("kind", ["iso", "acoustic", "elastic"])
def test_no_receivers_one_step(kind):
    _compare(kind, (20, 18, 22), nt=1)
    _compare(kind, (20, 18, 22), nt=25)


@pytest.mark.parametrize("kind", ["iso", "acoustic", "elastic"])
def test_corner_source_widest_layer(kind):
    """Source on the grid corner inside a layer as wide as allowed (3 nb = min dim)."""
    shape = (24, 27, 30)
    rec = [[0, 0, 0], [29, 26, 23], [0, 26, 0], [15, 13, 12]]
    _compare(kind, shape, nb=8, fs=int(kind == "elastic"), src=(0, 0, 0), rec=rec)
    _compare(kind, shape, nb=8, src=(29, 26, 23), rec=rec)


@pytest.mark.parametrize("kind", ["iso", "acoustic", "elastic"])
def test_rtm_without_snapshot_levels_and_zero_data(kind):
    """snap_period >= nt: no level is imaged, the image is untouched; zero data leaves any
    image unchanged (the receiver wavefield stays zero)."""
    nz, ny, nx = 20, 22, 24
    m = inputs.random_media((nz, ny, nx), seed=33, elastic=(kind == "elastic"))
    nt = 16
    w = inputs.source_series(kind, nt, DT, FP)
    rec = np.asarray([[3, 4, 5], [10, 11, 2]], np.int32)
    g = seis.Grid(nx, ny, nz, H, DT, nb=4, pml_f=FP)
    mod = seis.Model(g, kind, m["vp"], vs=m.get("vs"), rho=m.get("rho"))
    rng = np.random.default_rng(5)
    img0 = rng.standard_normal((nz, ny, nx)).astype(np.float32)
    data = rng.standard_normal((nt, 2)).astype(np.float32)
    img = img0.copy()
    mod.migrate(seis.Shot((12, 11, 10), w, rec, snap_period=nt), data, img)
    assert np.array_equal(img, img0)
    img = img0.copy()
    mod.migrate(seis.Shot((12, 11, 10), w, rec, snap_period=3, ckpt_period=2), np.zeros_like(data), img)
    assert np.array_equal(img, img0)
    # and a real image on the same model matches the oracle
    img = np.zeros((nz, ny, nx), np.float32)
    mod.migrate(seis.Shot((12, 11, 10), w, rec, snap_period=3), data, img)
    mod.close()
    og = oracle.Grid(nx, ny, nz, H, DT, nb=4, pml_f=FP)
    I = oracle.migrate(og, kind, m["vp"], m.get("rho"), (12, 11, 10), w, rec, data.astype(np.float64), 3,
                       vs=m.get("vs"))
    assert rel_l2(img, I) <= TOL_IMAGE
