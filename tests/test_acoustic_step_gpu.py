"""f1: the fused acoustic step (kernels_acoustic_step.cuh -- V and P of a time
step in ONE persistent launch, tiles exchanging their q^{n+1/2} halos through L2 as a
wavefront, in-place state) reproduces the split V / P kernels BIT FOR BIT: forward modeling
(seismogram + every field), RTM (imaging epilogue, snapshots fp32 and 24-bit, checkpointing),
with and without C-PML, on grids with one tile, many tiles, ragged x / y tails, a source
and receivers on tile edges, and fewer than L = 4 planes.  Eq 2, Alg 1.

SEIS_AC_STEP=1 / 0 forces the fused step on / off at model creation; the launch count of a
shot (1 step kernel + 1 gather per time step, against 2 + 1) proves which path ran."""
import numpy as np
import pytest

import oracle
import paper_conf_ppopp_qawasmehchc15_b200 as seis
from paper_conf_ppopp_qawasmehchc15_b200 import inputs
from gpu_common import TOL_FIELD, TOL_IMAGE, rel_l2

pytestmark = pytest.mark.gpu

CASES = [  # (nx, ny, nz, nb) -- tiles are 128 x 14
    (150, 45, 120, 7),   # 2 x 4 tiles, ragged x and y
    (128, 14, 50, 0),    # exactly one tile, zero walls
    (300, 97, 40, 9),    # 3 x 7 tiles, ragged
    (9, 5, 3, 0),        # smaller than a tile, fewer planes than the P lag
]


def _recs(nx, ny, nz):
    pts = [[0, 0, 0], [nx - 1, ny - 1, nz - 1], [min(127, nx - 1), min(13, ny - 1), nz // 2],
           [min(128, nx - 1), min(14, ny - 1), nz // 2], [nx // 2, ny // 2, 0], [nx // 2, ny // 2, nz - 1],
           [nx // 2, ny // 2, 0]]  # corners, both sides of the first tile edges, a duplicate
    return np.asarray(pts, np.int32)


def _run(monkeypatch, flag, nx, ny, nz, nb, kind_runs):
    monkeypatch.setenv("SEIS_AC_STEP", flag)
    m = inputs.random_media((nz, ny, nx), seed=61)
    h, dt, nt, snap = 10.0, 5e-4, 37, 4
    w = inputs.source_series("acoustic", nt, dt, 35.0)
    src = (min(128, nx - 1), min(14, ny - 1), nz // 2)
    rec = _recs(nx, ny, nz)
    g = seis.Grid(nx, ny, nz, h, dt, nb=nb, pml_f=35.0)
    mod = seis.Model(g, "acoustic", m["vp"], rho=m["rho"])
    out = {}
    shot = seis.Shot(src, w, rec, snap_period=snap)
    sg = np.zeros((nt, rec.shape[0]), np.float32)
    mod.forward_model(shot, sg)
    out["launches"] = seis.Model.launches()
    out["seis"] = sg
    out["fields"] = [mod.get_field(f) for f in range(4)]
    data = np.random.default_rng(4).standard_normal((nt, rec.shape[0])).astype(np.float32)
    for name, kw in kind_runs:
        img = np.zeros((nz, ny, nx), np.float32)
        mod.migrate(seis.Shot(src, w, rec, snap_period=snap, **kw), data, img)
        out[name] = img
    mod.close()
    return out, m, (h, dt, nt, snap, w, src, rec, data)


@pytest.mark.parametrize("nx,ny,nz,nb", CASES)
def test_fused_step_bitwise_equals_split(nx, ny, nz, nb, monkeypatch):
    runs = [("img", {}), ("img_ck", {"ckpt_period": 3}), ("img24", {"snap_bits": 24})]
    a, m, (h, dt, nt, snap, w, src, rec, data) = _run(monkeypatch, "0", nx, ny, nz, nb, runs)
    b, _, _ = _run(monkeypatch, "1", nx, ny, nz, nb, runs)
    assert a["launches"] == 3 * nt and b["launches"] == 2 * nt, (a["launches"], b["launches"])
    assert np.abs(a["seis"]).max() > 0
    assert np.array_equal(a["seis"], b["seis"])
    for t, (x, y) in enumerate(zip(a["fields"], b["fields"])):
        assert np.array_equal(x, y), t
    for name, _ in runs:
        assert np.array_equal(a[name], b[name]), name
    assert np.array_equal(b["img_ck"], b["img"])
    # and against the fp64 oracle (forward + image)
    og = oracle.Grid(nx, ny, nz, h, dt, nb=nb, pml_f=35.0)
    st = oracle.ac_state(og)
    ref = oracle.ac_run(og, m["vp"], m["rho"], st, 0, nt, [src], w[:, None], rec)
    assert rel_l2(b["seis"], ref) <= TOL_FIELD
    I = oracle.migrate(og, "acoustic", m["vp"], m["rho"], src, w, rec, data.astype(np.float64), snap)
    assert rel_l2(b["img"], I) <= TOL_IMAGE


def test_fused_step_default_selection():
    """A 512 x 512 plane is 4 x 37 tiles: without absorbing layers the fused step is selected
    without any override; with C-PML the split pair is."""
    torch = pytest.importorskip("torch")
    import os

    assert "SEIS_AC_STEP" not in os.environ
    n, nz, nt = 512, 40, 3
    wl = inputs.c2(n=n, nt=nt, nb=20, model=False)
    vp = np.full((nz, n, n), 2000.0, np.float32)
    for nb, launches in ((0, 2 * nt), (10, 3 * nt)):
        g = seis.Grid(n, n, nz, wl.h, wl.dt, nb=nb, pml_f=wl.fp)
        mod = seis.Model(g, "acoustic", vp, rho=vp * 0 + 1000.0)
        out = torch.zeros((nt, 3), device="cuda:0")
        mod.forward_model(seis.Shot((256, 256, 20), wl.wavelet[:nt], np.asarray([[250, 256, 20]] * 3, np.int32)), out)
        assert seis.Model.launches() == launches, nb
        mod.close()
