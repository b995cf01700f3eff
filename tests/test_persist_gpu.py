"""Persistent small-grid ISO paths (one cooperative launch per shot): the
resident-brick kernel (each CTA owns a 64 x 8 x 4 brick, neighbour progress counters; the
default where the bricks fit) and the grid-stride kernel (grid-wide barrier between steps,
SEIS_ISO_RESIDENT=0) are both bitwise equal to the z-march kernel path (SEIS_NO_PERSIST=1) for
the seismogram and both stored levels, with and without the damping layer, source inside the
layer and in the interior, odd and even step counts, ragged bricks in x / y / z; and within the
parity bar of the oracle."""
import numpy as np
import pytest

import oracle
import paper_conf_ppopp_qawasmehchc15_b200 as seis
from paper_conf_ppopp_qawasmehchc15_b200 import inputs
from gpu_common import TOL_FIELD, rel_l2

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("shape,nb,src,nt", [((66, 61, 58), 0, (32, 30, 29), 120), ((66, 61, 58), 8, (3, 20, 40), 75),
                                             ((66, 61, 58), 8, (30, 31, 33), 200), ((64, 64, 64), 6, (31, 29, 27), 90)])
def test_persistent_iso_bitwise_equals_zmarch(shape, nb, src, nt, monkeypatch):
    (nx, ny, nz), h, dt = shape, 10.0, 5e-4  # 66 x 61 x 58: ragged bricks in x / y / z
    m = inputs.random_media((nz, ny, nx), seed=61)
    w = inputs.source_series("iso", nt, dt, 35.0)
    rec = np.asarray([[1, 2, 3], [nx - 1, ny - 1, nz - 1], [30, 30, 30], [30, 30, 30], [5, 50, 7]], np.int32)
    outs = []
    for off, res in (("0", "2"), ("1", "1"), ("0", "0")):  # resident (required), z-march, grid-stride
        monkeypatch.setenv("SEIS_NO_PERSIST", off)
        monkeypatch.setenv("SEIS_ISO_RESIDENT", res)
        mod = seis.Model(seis.Grid(nx, ny, nz, h, dt, nb=nb, pml_f=35.0), "iso", m["vp"])
        sg = np.zeros((nt, rec.shape[0]), np.float32)
        mod.forward_model(seis.Shot(src, w, rec), sg)
        outs.append((sg, mod.get_field(0), mod.get_field(1)))
        mod.close()
    for other in outs[1:]:
        for a, b in zip(outs[0], other):
            assert np.array_equal(a, b)
    og = oracle.Grid(nx, ny, nz, h, dt, nb=nb, pml_f=35.0)
    st = oracle.iso_state(og)
    ref = oracle.iso_run(og, m["vp"], st, 0, nt, [src], w[:, None], rec)
    assert rel_l2(outs[0][0], ref) <= TOL_FIELD
    assert rel_l2(outs[0][1], st["u_cur"]) <= TOL_FIELD


@pytest.mark.parametrize("nt", [1, 2, 3])
def test_resident_short_shots_and_reuse(nt, monkeypatch):
    """The resident kernel stores only the last two levels into the field arrays and keeps its
    exchange tags monotonic over shots: 1-, 2- and 3-step shots, run twice on one model (the
    second shot reuses the tags' buffers), equal the z-march path bit for bit."""
    nx, ny, nz, h, dt = 64, 24, 20, 10.0, 5e-4
    m = inputs.random_media((nz, ny, nx), seed=62)
    w = inputs.source_series("iso", nt, dt, 35.0) * 1e3
    rec = np.asarray([[31, 12, 10], [0, 0, 0], [63, 23, 19]], np.int32)
    res = []
    for off, r in (("0", "2"), ("1", "1")):
        monkeypatch.setenv("SEIS_NO_PERSIST", off)
        monkeypatch.setenv("SEIS_ISO_RESIDENT", r)
        mod = seis.Model(seis.Grid(nx, ny, nz, h, dt, nb=4, pml_f=35.0), "iso", m["vp"])
        outs = []
        for _ in range(2):
            sg = np.zeros((nt, rec.shape[0]), np.float32)
            mod.forward_model(seis.Shot((31, 12, 10), w, rec), sg)
            outs.append((sg, mod.get_field(0), mod.get_field(1)))
        mod.close()
        res.append(outs)
    for shot in range(2):
        for a, b in zip(res[0][shot], res[1][shot]):
            assert np.array_equal(a, b), shot
    assert np.abs(res[0][0][0]).max() > 0
