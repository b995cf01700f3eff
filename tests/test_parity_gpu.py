"""GPU parity: the CUDA path (through the C ABI) against the fp64 oracle, on the
same seeded inputs, at sizes the oracle finishes in seconds that span several
32 x 16 tiles, several z-chunks and a ragged tail in x and y.

Bars (BASELINE.json north_star): relative L2 <= 1e-4 on wavefields and
seismograms, <= 1e-3 on RTM images.  Equations: Eq 1-3,
Algorithm 1, imaging P:111.
"""
import numpy as np
import pytest

import oracle
import paper_conf_ppopp_qawasmehchc15_b200 as seis
from paper_conf_ppopp_qawasmehchc15_b200 import inputs
from gpu_common import TOL_FIELD, TOL_IMAGE, grids, gpu_forward, oracle_fields, rel_l2

pytestmark = pytest.mark.gpu

NX, NY, NZ = 72, 40, 44   # 3 ragged x-tiles, 3 ragged y-tiles


def _recs(nx, ny, nz, z):
    xs = np.arange(2, nx - 2, 3)
    line = np.stack([xs, np.full_like(xs, ny // 2), np.full_like(xs, z)], axis=1)
    extra = np.asarray([[nx // 3, ny // 4, nz // 2], [nx - 1, ny - 1, nz - 1], [0, 0, 0],
                        [nx // 3, ny // 4, nz // 2]])  # corners + a duplicate
    return np.concatenate([line, extra]).astype(np.int32)


@pytest.mark.parametrize("nb", [0, 6])
def test_iso_forward_parity(nb):
    m = inputs.random_media((NZ, NY, NX), seed=11)
    h, dt, nt, fp = 10.0, 6e-4, 140, 35.0
    g, og = grids(NX, NY, NZ, h, dt, nb=nb)
    w = inputs.source_series("iso", nt, dt, fp)
    src = (NX // 2 + 1, NY // 2 - 3, NZ // 2)
    rec = _recs(NX, NY, NZ, 9)
    seis_g, fields_g = gpu_forward("iso", g, m, src, w, rec)
    st = oracle.iso_state(og)
    seis_o = oracle.iso_run(og, m["vp"], st, 0, nt, [src], w[:, None], rec)
    assert rel_l2(seis_g, seis_o) <= TOL_FIELD
    for a, b in zip(fields_g, oracle_fields("iso", st)):
        assert rel_l2(a, b) <= TOL_FIELD


@pytest.mark.parametrize("nb", [0, 7])
def test_acoustic_forward_parity(nb):
    m = inputs.random_media((NZ, NY, NX), seed=12)
    h, dt, nt, fp = 10.0, 6e-4, 150, 30.0
    g, og = grids(NX, NY, NZ, h, dt, nb=nb, pml_f=fp)
    w = inputs.source_series("acoustic", nt, dt, fp)
    src = (NX // 2 - 2, NY // 2 + 1, NZ // 2 + 3)
    rec = _recs(NX, NY, NZ, 10)
    seis_g, fields_g = gpu_forward("acoustic", g, m, src, w, rec)
    st = oracle.ac_state(og)
    seis_o = oracle.ac_run(og, m["vp"], m["rho"], st, 0, nt, [src], w[:, None], rec)
    assert rel_l2(seis_g, seis_o) <= TOL_FIELD
    for a, b in zip(fields_g, oracle_fields("acoustic", st)):
        assert rel_l2(a, b) <= TOL_FIELD


def test_acoustic_layered_c2_recipe_parity():
    """The C2 workload recipe (layered model, line of receivers, C-PML), scaled to 96x64x72."""
    nx, ny, nz = 96, 64, 72
    wl = inputs.c2(n=nz, nt=220, nb=8)
    m = inputs.layered_acoustic(nx, ny, nz)
    g, og = grids(nx, ny, nz, wl.h, wl.dt, nb=8, pml_f=wl.fp)
    src = (nx // 2, ny // 2, 12)
    rec = np.stack([np.arange(4, nx - 4), np.full(nx - 8, ny // 2), np.full(nx - 8, 12)], 1).astype(np.int32)
    w = inputs.source_series("acoustic", wl.nt, wl.dt, 25.0)
    seis_g, fields_g = gpu_forward("acoustic", g, m, src, w, rec)
    st = oracle.ac_state(og)
    seis_o = oracle.ac_run(og, m["vp"], m["rho"], st, 0, wl.nt, [src], w[:, None], rec)
    assert rel_l2(seis_g, seis_o) <= TOL_FIELD
    assert rel_l2(fields_g[0], st["p"]) <= TOL_FIELD


@pytest.mark.parametrize("fs,nb,comp", [(0, 0, 2), (1, 6, 2), (1, 6, 3), (0, 5, 0)])
def test_elastic_forward_parity(fs, nb, comp):
    nx, ny, nz = 68, 36, 40
    m = inputs.random_media((nz, ny, nx), seed=13, elastic=True)
    h, dt, nt, fp = 10.0, 5e-4, 110, 35.0
    g, og = grids(nx, ny, nz, h, dt, nb=nb, free_surface=fs, pml_f=fp)
    w = inputs.source_series("elastic", nt, dt, fp)
    src = (nx // 2, ny // 2, 5 if fs else nz // 2)
    rec = _recs(nx, ny, nz, 0 if fs else 7)
    seis_g, fields_g = gpu_forward("elastic", g, m, src, w, rec, component=comp)
    st = oracle.el_state(og)
    seis_o = oracle.el_run(og, m["vp"], m["vs"], m["rho"], st, 0, nt, [src], w[:, None], rec,
                           component=comp)
    assert rel_l2(seis_g, seis_o) <= TOL_FIELD
    for t, (a, b) in enumerate(zip(fields_g, oracle_fields("elastic", st))):
        assert rel_l2(a, b) <= TOL_FIELD, t


@pytest.mark.parametrize("kind", ["iso", "acoustic"])
def test_rtm_image_parity(kind):
    nx, ny, nz = 56, 40, 36
    m = inputs.random_media((nz, ny, nx), seed=14)
    h, dt, nt, fp, snap = 10.0, 6e-4, 120, 30.0, 5
    g, og = grids(nx, ny, nz, h, dt, nb=5, pml_f=fp)
    w = inputs.source_series(kind, nt, dt, fp)
    src = (nx // 2, ny // 2, 8)
    rec = _recs(nx, ny, nz, 8)
    rng = np.random.default_rng(5)
    data = rng.standard_normal((nt, rec.shape[0])).astype(np.float32)
    I_o = oracle.migrate(og, kind, m["vp"], m.get("rho") if kind == "acoustic" else None, src, w,
                         rec, data.astype(np.float64), snap)
    model = seis.Model(g, kind, m["vp"], rho=m["rho"] if kind == "acoustic" else None)
    img = np.zeros((nz, ny, nx), np.float32)
    model.migrate(seis.Shot(src, w, rec, snap_period=snap), data, img)
    assert rel_l2(img, I_o) <= TOL_IMAGE
    # accumulation over shots (P:111 sum_s): a second call adds the same image again
    model.migrate(seis.Shot(src, w, rec, snap_period=snap), data, img)
    assert rel_l2(img, 2 * I_o) <= TOL_IMAGE


@pytest.mark.parametrize("fs", [0, 1])
def test_elastic_rtm_image_parity(fs):
    """Elastic RTM: pressure imaging, explosive receiver injection, free surface."""
    nx, ny, nz = 52, 36, 40
    m = inputs.random_media((nz, ny, nx), seed=18, elastic=True)
    h, dt, nt, fp, snap = 10.0, 5e-4, 100, 35.0, 4
    g, og = grids(nx, ny, nz, h, dt, nb=5, free_surface=fs, pml_f=fp)
    w = inputs.source_series("elastic", nt, dt, fp)
    src = (nx // 2, ny // 2, 6)
    rec = _recs(nx, ny, nz, 0 if fs else 5)
    data = np.random.default_rng(6).standard_normal((nt, rec.shape[0])).astype(np.float32)
    I_o = oracle.migrate(og, "elastic", m["vp"], m["rho"], src, w, rec, data.astype(np.float64), snap,
                         vs=m["vs"])
    model = seis.Model(g, "elastic", m["vp"], vs=m["vs"], rho=m["rho"])
    img = np.zeros((nz, ny, nx), np.float32)
    model.migrate(seis.Shot(src, w, rec, snap_period=snap), data, img)
    assert rel_l2(img, I_o) <= TOL_IMAGE


@pytest.mark.parametrize("kind", ["iso", "acoustic", "elastic"])
def test_decomposition_bitwise_invariance(kind):
    """P z-slabs (halo planes copied between slabs) give bitwise-identical results (§8e)."""
    nx, ny, nz = 40, 34, 64
    m = inputs.random_media((nz, ny, nx), seed=15, elastic=(kind == "elastic"))
    h, dt, nt = 10.0, 5e-4, 60
    w = inputs.source_series(kind, nt, dt, 35.0)
    src = (nx // 2, ny // 2, nz // 2 + 4)
    rec = _recs(nx, ny, nz, 20)
    outs = []
    for P in (1, 2, 3, 4):
        g = seis.Grid(nx, ny, nz, h, dt, nb=5, free_surface=int(kind == "elastic"), pml_f=35.0,
                      slabs=P)
        outs.append(gpu_forward(kind, g, m, src, w, rec))
    for s, f in outs[1:]:
        assert np.array_equal(s, outs[0][0])
        for a, b in zip(f, outs[0][1]):
            assert np.array_equal(a, b)


def test_rtm_decomposition_bitwise_invariance():
    nx, ny, nz = 40, 34, 64
    m = inputs.random_media((nz, ny, nx), seed=16)
    nt, snap = 60, 4
    w = inputs.source_series("acoustic", nt, 5e-4, 35.0)
    rec = _recs(nx, ny, nz, 6)
    data = np.random.default_rng(1).standard_normal((nt, rec.shape[0])).astype(np.float32)
    imgs = []
    for P in (1, 4):
        g = seis.Grid(nx, ny, nz, 10.0, 5e-4, nb=5, pml_f=35.0, slabs=P)
        mod = seis.Model(g, "acoustic", m["vp"], rho=m["rho"])
        img = np.zeros((nz, ny, nx), np.float32)
        mod.migrate(seis.Shot((nx // 2, ny // 2, 6), w, rec, snap_period=snap), data, img)
        imgs.append(img)
    assert np.array_equal(imgs[0], imgs[1])


def test_device_and_host_buffers_agree():
    import torch

    nx, ny, nz = 40, 33, 30
    m = inputs.random_media((nz, ny, nx), seed=17)
    g = seis.Grid(nx, ny, nz, 10.0, 5e-4, nb=4, pml_f=30.0)
    w = inputs.source_series("acoustic", 50, 5e-4, 30.0)
    rec = _recs(nx, ny, nz, 5)
    mod = seis.Model(g, "acoustic", m["vp"], rho=m["rho"])
    shot = seis.Shot((20, 16, 15), w, rec)
    host = np.zeros((50, rec.shape[0]), np.float32)
    mod.forward_model(shot, host)
    dev = mod.forward_model(shot)
    torch.cuda.synchronize()
    assert np.array_equal(host, dev.cpu().numpy())


def test_error_codes():
    nx = 24
    vp = np.full((nx, nx, nx), 2000.0, np.float32)
    with pytest.raises(seis.SeisError) as e:  # Courant 2000*1e-2/10 = 2 > 0.45
        seis.Model(seis.Grid(nx, nx, nx, 10.0, 1e-2), "iso", vp)
    assert e.value.name == "SEIS_ECFL"
    with pytest.raises(seis.SeisError) as e:
        seis.Model(seis.Grid(nx, nx, nx, 10.0, 1e-3), "elastic", vp, rho=vp)
    assert e.value.name == "SEIS_EINVAL"
    mod = seis.Model(seis.Grid(nx, nx, nx, 10.0, 1e-3), "iso", vp)
    w = np.zeros(10, np.float32)
    with pytest.raises(seis.SeisError) as e:
        mod.forward_model(seis.Shot((nx, 0, 0), w, np.zeros((1, 3), np.int32)),
                          np.zeros((10, 1), np.float32))
    assert e.value.name == "SEIS_EINVAL"
    with pytest.raises(seis.SeisError) as e:
        mod.forward_model(seis.Shot((1, 1, 1), w, np.asarray([[0, 0, nx]], np.int32)),
                          np.zeros((10, 1), np.float32))
    assert e.value.name == "SEIS_EINVAL"
    with pytest.raises(seis.SeisError) as e:  # snapshot cadence must be >= 1
        mod.migrate(seis.Shot((1, 1, 1), w, np.zeros((1, 3), np.int32), snap_period=0),
                    np.zeros((10, 1), np.float32), np.zeros((nx, nx, nx), np.float32))
    assert e.value.name == "SEIS_EINVAL"


def _deep_recs(nx, ny, nz):
    """Receivers at every depth band, so the injection tables of both the boundary chunks
    and the interior chunks of every slab are exercised (a duplicate included)."""
    pts = [[(7 * t) % nx, (5 * t) % ny, (11 * t) % nz] for t in range(40)]
    pts.append(pts[3])
    return np.asarray(pts, np.int32)


@pytest.mark.parametrize("kind", ["iso", "acoustic", "elastic"])
def test_overlapped_exchange_bitwise(kind, monkeypatch):
    """§8(e) pipeline: with z-slabs the first / last z-chunk of every slab runs first, the
    ghost exchange overlaps the interior chunks on a second stream.  Grids deep enough for
    many chunks per slab; forward modeling and RTM (receivers injected in boundary and
    interior chunks) are bitwise identical to one slab, and to the serial exchange
    (SEIS_NO_OVERLAP=1); one slab matches the oracle."""
    nx, ny, nz = 64, 40, 168
    el = kind == "elastic"
    m = inputs.random_media((nz, ny, nx), seed=21, elastic=el)
    h, dt, nt, snap = 10.0, 5e-4, 40, 4
    w = inputs.source_series(kind, nt, dt, 35.0)
    src = (nx // 2, ny // 2, 84)
    rec = _deep_recs(nx, ny, nz)
    data = np.random.default_rng(2).standard_normal((nt, rec.shape[0])).astype(np.float32)
    runs = []
    for P, serial in ((1, False), (2, False), (3, False), (3, True)):
        monkeypatch.setenv("SEIS_NO_OVERLAP", "1" if serial else "0")
        g = seis.Grid(nx, ny, nz, h, dt, nb=6, free_surface=int(el), pml_f=35.0, slabs=P)
        mod = seis.Model(g, kind, m["vp"], vs=m.get("vs"), rho=m.get("rho"))
        shot = seis.Shot(src, w, rec, rec_component=2, snap_period=snap)
        sg = np.zeros((nt, rec.shape[0]), np.float32)
        mod.forward_model(shot, sg)
        img = np.zeros((nz, ny, nx), np.float32)
        mod.migrate(shot, data, img)
        runs.append((sg, img))
        mod.close()
    for sg, img in runs[1:]:
        assert np.array_equal(sg, runs[0][0])
        assert np.array_equal(img, runs[0][1])
    og = oracle.Grid(nx, ny, nz, h, dt, nb=6, free_surface=int(el), pml_f=35.0)
    if kind == "iso":
        ref = oracle.iso_run(og, m["vp"], oracle.iso_state(og), 0, nt, [src], w[:, None], rec)
    elif kind == "acoustic":
        ref = oracle.ac_run(og, m["vp"], m["rho"], oracle.ac_state(og), 0, nt, [src], w[:, None], rec)
    else:
        ref = oracle.el_run(og, m["vp"], m["vs"], m["rho"], oracle.el_state(og), 0, nt, [src],
                            w[:, None], rec, component=2)
    assert rel_l2(runs[0][0], ref) <= TOL_FIELD


@pytest.mark.parametrize("kind,P", [("iso", 1), ("acoustic", 1), ("acoustic", 3), ("elastic", 1)])
def test_checkpointed_rtm_bitwise(kind, P):
    """f2: RTM with source-state checkpoints (segments of c snapshots recomputed in the
    backward phase) gives the image of the all-snapshots pool bit for bit, for segment
    lengths that divide the snapshot count, leave a ragged last segment, or are 1; and the
    image matches the oracle."""
    nx, ny, nz = 48, 40, 72
    el = kind == "elastic"
    m = inputs.random_media((nz, ny, nx), seed=23, elastic=el)
    h, dt, nt, snap = 10.0, 5e-4, 61, 4   # 15 snapshots
    w = inputs.source_series(kind, nt, dt, 35.0)
    src = (nx // 2, ny // 2, 8)
    rec = _deep_recs(nx, ny, nz)
    data = np.random.default_rng(3).standard_normal((nt, rec.shape[0])).astype(np.float32)
    g = seis.Grid(nx, ny, nz, h, dt, nb=6, free_surface=int(el), pml_f=35.0, slabs=P)
    mod = seis.Model(g, kind, m["vp"], vs=m.get("vs"), rho=m.get("rho"))
    imgs = {}
    for c in (0, 1, 4, 5, 7, 15):
        img = np.zeros((nz, ny, nx), np.float32)
        mod.migrate(seis.Shot(src, w, rec, snap_period=snap, ckpt_period=c), data, img)
        imgs[c] = img
    mod.close()
    for c, img in imgs.items():
        assert np.array_equal(img, imgs[0]), c
    og = oracle.Grid(nx, ny, nz, h, dt, nb=6, free_surface=int(el), pml_f=35.0)
    I = oracle.migrate(og, kind, m["vp"], m.get("rho"), src, w, rec, data.astype(np.float64), snap,
                       vs=m.get("vs"))
    assert rel_l2(imgs[0], I) <= TOL_IMAGE


