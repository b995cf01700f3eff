"""GPU runtime state across calls on ONE model (C ABI): the CUDA graph of forward_model
(captured once per shot geometry / wavelet / output buffer, replayed afterwards) must stay
valid when a migrate in between rebuilds the receiver tables, and the host bookkeeping of
the current time level must follow the replay (stale gather-table pointers and
S.cur after a replay).

Every call of a model is the same computation from a zero state, so a repeated
forward_model must return bitwise the first seismogram and final fields.
"""
import numpy as np
import pytest

import paper_conf_ppopp_qawasmehchc15_b200 as seis
from paper_conf_ppopp_qawasmehchc15_b200 import inputs

pytestmark = pytest.mark.gpu

NX, NY, NZ = 72, 40, 44
H, DT, FP = 10.0, 6e-4, 30.0


def _line(z, x0=3, x1=NX - 3, step=2):
    xs = np.arange(x0, x1, step)
    return np.stack([xs, np.full_like(xs, NY // 2), np.full_like(xs, z)], 1).astype(np.int32)


@pytest.mark.parametrize("kind", ["iso", "acoustic", "elastic"])
@pytest.mark.parametrize("other_geometry", [False, True])
def test_forward_migrate_forward_replay(kind, other_geometry, monkeypatch):
    torch = pytest.importorskip("torch")
    monkeypatch.setenv("SEIS_NO_PERSIST", "1")  # small ISO grids: use the graph path too
    m = inputs.random_media((NZ, NY, NX), seed=41, elastic=(kind == "elastic"))
    g = seis.Grid(NX, NY, NZ, H, DT, nb=6, pml_f=FP)
    model = seis.Model(g, kind, m["vp"], vs=m.get("vs"), rho=m.get("rho"))
    nt = 40  # even
    shot = seis.Shot((NX // 2, NY // 2, NZ // 2), inputs.source_series(kind, nt, DT, FP), _line(8))
    out = torch.zeros((nt, shot.nrec), device="cuda:0")
    nf = {"iso": 2, "acoustic": 4, "elastic": 9}[kind]
    model.forward_model(shot, out)  # captures the graph
    ref = out.clone()
    ref_f = [model.get_field(f) for f in range(nf)]
    model.forward_model(shot, out)  # replays it
    assert torch.equal(out, ref)
    for f in range(nf):
        assert np.array_equal(model.get_field(f), ref_f[f]), f
    # a migrate with an ODD step count (other final level) and, optionally, another geometry
    nt2 = 33
    rec2 = _line(12, 5, NX - 5, 3) if other_geometry else shot.rec
    src2 = (NX // 3, NY // 3, NZ // 3) if other_geometry else shot.src
    shot2 = seis.Shot(src2, inputs.source_series(kind, nt2, DT, FP), rec2, snap_period=4)
    data = torch.from_numpy(np.random.default_rng(3).standard_normal((nt2, shot2.nrec)).astype(np.float32)).cuda()
    img = torch.zeros((NZ, NY, NX), device="cuda:0")
    model.migrate(shot2, data, img)
    # a few allocations in between so that freed table addresses are not simply reused
    junk = [torch.empty(1 << 20, device="cuda:0") for _ in range(4)]
    out.zero_()
    model.forward_model(shot, out)  # must not replay freed tables or keep the migrate's level
    assert torch.equal(out, ref)
    for f in range(nf):
        assert np.array_equal(model.get_field(f), ref_f[f]), f
    del junk
    model.close()


def test_host_staging_buffers_regrow():
    """forward_model into a host seismogram, then a migrate with a host image and data, then a
    larger host seismogram: the staging buffer grows (the old one is freed) and results stay
    those of device buffers."""
    torch = pytest.importorskip("torch")
    m = inputs.random_media((NZ, NY, NX), seed=42)
    g = seis.Grid(NX, NY, NZ, H, DT, nb=6, pml_f=FP)
    model = seis.Model(g, "acoustic", m["vp"], rho=m["rho"])
    nt = 30
    shot = seis.Shot((NX // 2, NY // 2, 10), inputs.source_series("acoustic", nt, DT, FP), _line(8))
    dev = torch.zeros((nt, shot.nrec), device="cuda:0")
    model.forward_model(shot, dev)
    host = np.zeros((nt, shot.nrec), np.float32)
    model.forward_model(shot, host)
    assert np.array_equal(host, dev.cpu().numpy())
    data = np.random.default_rng(1).standard_normal((nt, shot.nrec)).astype(np.float32)
    img_h = np.zeros((NZ, NY, NX), np.float32)
    model.migrate(seis.Shot(shot.src, shot.wavelet, shot.rec, snap_period=3), data, img_h)
    img_d = torch.zeros((NZ, NY, NX), device="cuda:0")
    model.migrate(seis.Shot(shot.src, shot.wavelet, shot.rec, snap_period=3), torch.from_numpy(data).cuda(), img_d)
    assert np.array_equal(img_h, img_d.cpu().numpy())
    nt3 = 4 * nt  # a larger host buffer than any before
    shot3 = seis.Shot(shot.src, inputs.source_series("acoustic", nt3, DT, FP), np.tile(shot.rec, (4, 1)))
    big_h = np.zeros((nt3, shot3.nrec), np.float32)
    model.forward_model(shot3, big_h)
    big_d = torch.zeros((nt3, shot3.nrec), device="cuda:0")
    model.forward_model(shot3, big_d)
    assert np.array_equal(big_h, big_d.cpu().numpy())
    model.close()


def test_graph_sampled_profiling():
    """seis_profile(S > 1) keeps the shot graph and times the launches of every S-th step by
    event nodes inside it (bench.py's timed region): the seismogram is bitwise the unprofiled
    one, every sampled kernel has ceil(nt / S) launches per replay with positive times, the
    counters accumulate over replays and a repeated seis_profile(S) zeroes them only."""
    nx, ny, nz, nt, S = 100, 40, 48, 23, 5
    m = inputs.random_media((nz, ny, nx), seed=81)
    w = inputs.source_series("acoustic", nt, 5e-4, 30.0)
    rec = np.asarray([[10, 10, 10], [50, 20, 30]], np.int32)
    mod = seis.Model(seis.Grid(nx, ny, nz, 10.0, 5e-4, nb=5, pml_f=30.0), "acoustic", m["vp"], rho=m["rho"])
    shot = seis.Shot((50, 20, 24), w, rec)
    ref = np.zeros((nt, 2), np.float32)
    mod.forward_model(shot, ref)
    try:
        seis.profile(True, sample=S)
        out = np.zeros((nt, 2), np.float32)
        mod.forward_model(shot, out)  # (captures the graph with its event nodes)
        assert np.array_equal(out, ref)
        seis.profile(True, sample=S)  # same mode: counters zeroed, graph kept
        for _ in range(2):
            mod.forward_model(shot, out)
        kp = seis.profile_read()
        per = -(-nt // S)
        for k in ("ac_v", "ac_p", "gather"):
            assert kp[k][1] == 2 * per, (k, kp[k])
            assert kp[k][0] > 0
        assert np.array_equal(out, ref)
    finally:
        seis.profile(False)
    mod.forward_model(shot, out)
    assert np.array_equal(out, ref)
    mod.close()
