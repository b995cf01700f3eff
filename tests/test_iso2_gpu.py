"""f1 ("2-step temporal blocking for ISO"): the ISO 2-step kernel
(kernels_iso2.cuh -- time steps n and n + 1 in ONE persistent launch, tiles exchanging their
u^{n+1} halos through L2 as a wavefront, in-place state) reproduces the one-step z-march
kernel BIT FOR BIT: seismogram (both rows of every pair, receivers on tile edges, corners, a
duplicate) and both time levels, with and without the damped-wave layer (O6), for even and
odd step counts (a trailing single step), on grids with one tile, many tiles, ragged x / y
tails and fewer planes than the step-2 lag.  Eq 1, Alg 1.

SEIS_ISO2=1 / 0 selects the path at model creation; SEIS_NO_PERSIST=1 keeps these small
grids off the one-launch small-grid kernels.  The launch count of a shot (one 2-step kernel
+ 2 gathers per pair, against 2 steps + 2 gathers) proves which path ran; one case is also
checked against the fp64 oracle."""
import numpy as np
import pytest

import oracle
import paper_conf_ppopp_qawasmehchc15_b200 as seis
from paper_conf_ppopp_qawasmehchc15_b200 import inputs
from gpu_common import TOL_FIELD, rel_l2

pytestmark = pytest.mark.gpu

CASES = [  # (nx, ny, nz, nb, nt) -- tiles are 128 x 14
    (150, 45, 60, 7, 37),    # 2 x 4 tiles, ragged x and y, damped layer, odd step count
    (128, 14, 30, 0, 24),    # exactly one tile, no layer, even step count
    (300, 97, 40, 9, 30),    # 3 x 7 tiles, ragged
    (9, 5, 3, 0, 11),        # smaller than a tile, fewer planes than the step-2 lag
    (260, 30, 20, 4, 2),     # one pair only
]


def _recs(nx, ny, nz):
    pts = [[0, 0, 0], [nx - 1, ny - 1, nz - 1], [min(127, nx - 1), min(13, ny - 1), nz // 2],
           [min(128, nx - 1), min(14, ny - 1), nz // 2], [nx // 2, ny // 2, 0], [nx // 2, ny // 2, nz - 1],
           [nx // 2, ny // 2, 0]]
    return np.asarray(pts, np.int32)


def _run(monkeypatch, flag, nx, ny, nz, nb, nt):
    monkeypatch.setenv("SEIS_ISO2", flag)
    monkeypatch.setenv("SEIS_NO_PERSIST", "1")
    m = inputs.random_media((nz, ny, nx), seed=67)
    h, dt = 10.0, 6e-4
    w = inputs.source_series("iso", nt, dt, 30.0)
    src = (min(128, nx - 1), min(14, ny - 1), nz // 2)
    rec = _recs(nx, ny, nz)
    g = seis.Grid(nx, ny, nz, h, dt, nb=nb, pml_f=30.0)
    mod = seis.Model(g, "iso", m["vp"])
    sg = np.zeros((nt, rec.shape[0]), np.float32)
    mod.forward_model(seis.Shot(src, w, rec), sg)
    out = {"launches": seis.Model.launches(), "seis": sg, "fields": [mod.get_field(f) for f in range(2)]}
    # a second shot on the same model (counters and in-place state reused)
    sg2 = np.zeros_like(sg)
    mod.forward_model(seis.Shot(src, w, rec), sg2)
    out["seis2"] = sg2
    mod.close()
    return out, m, (h, dt, w, src, rec)


@pytest.mark.parametrize("nx,ny,nz,nb,nt", CASES)
def test_iso2_bitwise_equals_one_step(monkeypatch, nx, ny, nz, nb, nt):
    two, _, _ = _run(monkeypatch, "1", nx, ny, nz, nb, nt)
    one, _, _ = _run(monkeypatch, "0", nx, ny, nz, nb, nt)
    # one step: 1 kernel + 1 gather; a pair: 1 kernel + 2 gathers
    assert one["launches"] == 2 * nt
    assert two["launches"] == (nt // 2) * 3 + (nt % 2) * 2
    assert np.array_equal(two["seis"], one["seis"])
    assert np.array_equal(two["seis2"], two["seis"])
    for a, b in zip(two["fields"], one["fields"]):
        assert np.array_equal(a, b)


def test_iso2_against_oracle(monkeypatch):
    nx, ny, nz, nb, nt = 150, 45, 60, 7, 37
    two, m, (h, dt, w, src, rec) = _run(monkeypatch, "1", nx, ny, nz, nb, nt)
    og = oracle.Grid(nx, ny, nz, h, dt, nb=nb, pml_f=30.0)
    st = oracle.iso_state(og)
    s_o = oracle.iso_run(og, m["vp"], st, 0, nt, [src], w[:, None], rec)
    assert rel_l2(two["seis"], s_o) <= TOL_FIELD
