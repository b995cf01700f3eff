"""ISO split-field PML (O6b, seis_grid.iso_pml = 1; SURVEY §8f f4's "split-field 2nd-order
PML for ISO"): CUDA path vs the fp64 oracle, and decomposition / checkpoint invariance."""
import numpy as np
import pytest

import oracle
import paper_conf_ppopp_qawasmehchc15_b200 as seis
from paper_conf_ppopp_qawasmehchc15_b200 import inputs
from gpu_common import TOL_FIELD, TOL_IMAGE, rel_l2

pytestmark = pytest.mark.gpu

NX, NY, NZ, H, DT, FP, NB = 70, 37, 44, 10.0, 5e-4, 35.0, 6


def _grids(slabs=1):
    return (seis.Grid(NX, NY, NZ, H, DT, nb=NB, pml_f=FP, slabs=slabs, iso_pml=1),
            oracle.Grid(NX, NY, NZ, H, DT, nb=NB, pml_f=FP, iso_pml=1))


def _recs():
    # layer points on every face, edges and corners, interior points, a duplicate
    pts = [[1, NY // 2, NZ // 2], [NX - 2, 3, 20], [NX // 2, 0, 2], [NX // 2, NY - 1, NZ - 3],
           [2, 2, 2], [NX - 1, NY - 1, NZ - 1], [35, 18, 22], [20, 10, 30], [NX // 2, NY // 2, 5]]
    pts.append(pts[4])
    return np.asarray(pts, np.int32)


@pytest.mark.parametrize("src", [(3, NY // 2, NZ // 2), (NX // 2, NY // 2, NZ // 2)])
def test_iso_split_pml_forward_parity(src):
    nt = 120
    m = inputs.random_media((NZ, NY, NX), seed=41)
    w = inputs.source_series("iso", nt, DT, FP)
    rec = _recs()
    g, og = _grids()
    mod = seis.Model(g, "iso", m["vp"])
    sg = np.zeros((nt, rec.shape[0]), np.float32)
    mod.forward_model(seis.Shot(src, w, rec), sg)
    u_cur, u_prev = mod.get_field(0), mod.get_field(1)
    st = oracle.iso_state(og)
    ref = oracle.iso_run(og, m["vp"], st, 0, nt, [src], w[:, None], rec)
    assert rel_l2(sg, ref) <= TOL_FIELD
    assert rel_l2(u_cur, st["u_cur"]) <= TOL_FIELD
    assert rel_l2(u_prev, st["u_prev"]) <= TOL_FIELD
    if src[0] >= NB:
        return
    # (source inside the layer) the layer differs from the damped-wave layer (O6): the path
    # really changed
    g0 = seis.Grid(NX, NY, NZ, H, DT, nb=NB, pml_f=FP)
    sg0 = np.zeros_like(sg)
    seis.Model(g0, "iso", m["vp"]).forward_model(seis.Shot(src, w, rec), sg0)
    assert rel_l2(sg0, ref) > 10 * TOL_FIELD


def test_iso_split_pml_rtm_parity_and_invariance():
    nt, snap = 80, 4
    m = inputs.random_media((NZ, NY, NX), seed=42)
    w = inputs.source_series("iso", nt, DT, FP)
    rec = _recs()
    data = np.random.default_rng(5).standard_normal((nt, rec.shape[0])).astype(np.float32)
    src = (4, NY // 2, 3)
    _, og = _grids()
    I_o = oracle.migrate(og, "iso", m["vp"], None, src, w, rec, data.astype(np.float64), snap)
    imgs = []
    for P, ck in ((1, 0), (3, 0), (1, 5), (3, 4)):
        g, _ = _grids(P)
        mod = seis.Model(g, "iso", m["vp"])
        img = np.zeros((NZ, NY, NX), np.float32)
        mod.migrate(seis.Shot(src, w, rec, snap_period=snap, ckpt_period=ck), data, img)
        imgs.append(img)
        mod.close()
    assert rel_l2(imgs[0], I_o) <= TOL_IMAGE
    for img in imgs[1:]:
        assert np.array_equal(img, imgs[0])

