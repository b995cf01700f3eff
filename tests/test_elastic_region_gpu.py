"""Elastic kernel code paths (elastic kernels): the lean body without the C-PML
memory-variable code (the whole grid when there are no layers; by default, inside one launch,
the blocks whose tile and z-chunk hold no layer point; under SEIS_EL_REGION=1 a separate
launch over those blocks) computes the same points with the same arithmetic as the full body
(SEIS_EL_REGION=0 everywhere), so all three are BIT-identical --
seismogram, all 9 fields, and the RTM image (snapshot epilogue of el_s, imaging epilogue of
el_v).  Grids span several 64 x 15 tiles and z-chunks with ragged tails, C-PML on 5 or 6 faces.
Eq 3, C-PML."""
import numpy as np
import pytest

import paper_conf_ppopp_qawasmehchc15_b200 as seis
from paper_conf_ppopp_qawasmehchc15_b200 import inputs

pytestmark = pytest.mark.gpu


def _run(monkeypatch, flag, nx, ny, nz, nb, fs):
    if flag is None:
        monkeypatch.delenv("SEIS_EL_REGION", raising=False)
    else:
        monkeypatch.setenv("SEIS_EL_REGION", flag)
    m = inputs.random_media((nz, ny, nx), seed=71, elastic=True)
    h, dt, nt, snap = 10.0, 6e-4, 31, 3
    w = inputs.source_series("elastic", nt, dt, 30.0)
    src = (nx // 2, ny // 2, nz // 3)
    rec = np.asarray([[0, 0, 0], [nx - 1, ny - 1, nz - 1], [nx // 2, ny // 2, 0], [nb, nb, nb]], np.int32)
    g = seis.Grid(nx, ny, nz, h, dt, nb=nb, free_surface=fs, pml_f=30.0)
    mod = seis.Model(g, "elastic", m["vp"], vs=m["vs"], rho=m["rho"])
    sg = np.zeros((nt, rec.shape[0]), np.float32)
    mod.forward_model(seis.Shot(src, w, rec, snap_period=snap), sg)
    launches = seis.Model.launches()
    fields = [mod.get_field(f) for f in range(9)]
    data = np.random.default_rng(5).standard_normal((nt, rec.shape[0])).astype(np.float32)
    img = np.zeros((nz, ny, nx), np.float32)
    mod.migrate(seis.Shot(src, w, rec, snap_period=snap), data, img)
    mod.close()
    return sg, fields, img, launches, nt


@pytest.mark.parametrize("nx,ny,nz,nb,fs", [(200, 70, 90, 8, 1), (150, 50, 60, 5, 0)])
def test_region_split_bitwise(nx, ny, nz, nb, fs, monkeypatch):
    a = _run(monkeypatch, "0", nx, ny, nz, nb, fs)
    nt = a[4]
    assert a[3] == 3 * nt  # el_v + el_s + gather per step
    assert np.abs(a[0]).max() > 0 and np.abs(a[2]).max() > 0
    for flag, launches in ((None, 3 * nt), ("1", 5 * nt)):  # per-block choice; split: 2 more
        b = _run(monkeypatch, flag, nx, ny, nz, nb, fs)
        assert b[3] == launches, (flag, b[3])
        assert np.array_equal(a[0], b[0]), flag
        for t, (x, y) in enumerate(zip(a[1], b[1])):
            assert np.array_equal(x, y), (flag, t)
        assert np.array_equal(a[2], b[2]), flag
