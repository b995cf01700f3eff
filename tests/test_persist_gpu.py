"""Persistent small-grid ISO path (one cooperative launch per shot, grid-wide barrier between
steps): bitwise equal to the z-march kernel path (SEIS_NO_PERSIST=1) for the
seismogram and both stored levels, with and without the damping layer, source inside the
layer and in the interior, odd and even step counts; and within the parity bar of the oracle."""
import numpy as np
import pytest

import oracle
import paper_conf_ppopp_qawasmehchc15_b200 as seis
from paper_conf_ppopp_qawasmehchc15_b200 import inputs
from gpu_common import TOL_FIELD, rel_l2

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("nb,src,nt", [(0, (32, 30, 29), 120), (8, (3, 20, 40), 75), (8, (30, 31, 33), 200)])
def test_persistent_iso_bitwise_equals_zmarch(nb, src, nt, monkeypatch):
    nx, ny, nz, h, dt = 66, 61, 58, 10.0, 5e-4  # ragged x / y tails
    m = inputs.random_media((nz, ny, nx), seed=61)
    w = inputs.source_series("iso", nt, dt, 35.0)
    rec = np.asarray([[1, 2, 3], [nx - 1, ny - 1, nz - 1], [30, 30, 30], [30, 30, 30], [5, 50, 7]], np.int32)
    outs = []
    for off in ("0", "1"):
        monkeypatch.setenv("SEIS_NO_PERSIST", off)
        mod = seis.Model(seis.Grid(nx, ny, nz, h, dt, nb=nb, pml_f=35.0), "iso", m["vp"])
        sg = np.zeros((nt, rec.shape[0]), np.float32)
        mod.forward_model(seis.Shot(src, w, rec), sg)
        outs.append((sg, mod.get_field(0), mod.get_field(1)))
        mod.close()
    for a, b in zip(outs[0], outs[1]):
        assert np.array_equal(a, b)
    og = oracle.Grid(nx, ny, nz, h, dt, nb=nb, pml_f=35.0)
    st = oracle.iso_state(og)
    ref = oracle.iso_run(og, m["vp"], st, 0, nt, [src], w[:, None], rec)
    assert rel_l2(outs[0][0], ref) <= TOL_FIELD
    assert rel_l2(outs[0][1], st["u_cur"]) <= TOL_FIELD
