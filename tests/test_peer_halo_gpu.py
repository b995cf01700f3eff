"""f4: direct ghost-plane stores.

* In-process z-slabs: the kernel producing an exchanged field writes its boundary planes
  straight into the neighbouring slab's ghost planes (default), bitwise equal to the copy
  exchange (SEIS_GHOST_COPY=1) and to one slab, for modeling, RTM and checkpointed RTM.
* Ranks: P processes, one z-slab each, all on cuda:0 (NCCL refuses two ranks on one GPU, so
  the communicator is peer-only), the rank faces written through CUDA IPC mappings and
  ordered by stream-memory-operation flags -- the same code path as NVLink peers between
  GPUs.  Seismogram, every field and the RTM image are bitwise equal to one process.
"""
import os
import socket

import numpy as np
import pytest

import paper_conf_ppopp_qawasmehchc15_b200 as seis
from paper_conf_ppopp_qawasmehchc15_b200 import inputs

pytestmark = pytest.mark.gpu

NF = {"iso": 2, "acoustic": 4, "elastic": 9}


def _case(kind):
    nx, ny, nz = 48, 36, 96
    el = kind == "elastic"
    m = inputs.random_media((nz, ny, nx), seed=31, elastic=el)
    h, dt, nt, snap = 10.0, 5e-4, 36, 4
    w = inputs.source_series(kind, nt, dt, 35.0)
    # receivers in every depth band (boundary planes of the slabs included) + a duplicate
    pts = [[(7 * t) % nx, (5 * t) % ny, (3 * t) % nz] for t in range(48)]
    pts.append(pts[5])
    rec = np.asarray(pts, np.int32)
    data = np.random.default_rng(4).standard_normal((nt, rec.shape[0])).astype(np.float32)
    return dict(nx=nx, ny=ny, nz=nz, el=el, m=m, h=h, dt=dt, nt=nt, snap=snap, w=w, rec=rec, data=data,
                src=(nx // 2, ny // 2, nz // 2 + 1))


def _grid(c, slabs=1):
    return seis.Grid(c["nx"], c["ny"], c["nz"], c["h"], c["dt"], nb=5, free_surface=int(c["el"]),
                     pml_f=35.0, slabs=slabs)


def _run(kind, c, model, ckpt=0):
    shot = seis.Shot(c["src"], c["w"], c["rec"], rec_component=2, snap_period=c["snap"])
    sg = np.zeros((c["nt"], c["rec"].shape[0]), np.float32)
    model.forward_model(shot, sg)
    fields = [model.get_field(f) for f in range(NF[kind])]
    img = np.zeros(model.local_shape, np.float32)
    model.migrate(shot, c["data"], img)
    shot.ckpt_period = ckpt or 3
    img2 = np.zeros(model.local_shape, np.float32)
    model.migrate(shot, c["data"], img2)
    return sg, fields, img, img2


@pytest.mark.parametrize("kind", ["iso", "acoustic", "elastic"])
def test_direct_ghost_stores_bitwise(kind, monkeypatch):
    c = _case(kind)
    m = c["m"]
    runs = []
    for P, copy in ((1, "0"), (3, "1"), (3, "0"), (5, "0")):
        monkeypatch.setenv("SEIS_GHOST_COPY", copy)
        mod = seis.Model(_grid(c, P), kind, m["vp"], vs=m.get("vs"), rho=m.get("rho"))
        runs.append(_run(kind, c, mod))
        mod.close()
    ref = runs[0]
    assert np.abs(ref[0]).max() > 0 and np.abs(ref[2]).max() > 0
    for r in runs[1:]:
        assert np.array_equal(r[0], ref[0])
        for a, b in zip(r[1], ref[1]):
            assert np.array_equal(a, b)
        assert np.array_equal(r[2], ref[2])
        assert np.array_equal(r[3], ref[3])
    assert np.array_equal(ref[3], ref[2])  # checkpointed RTM = all-snapshot RTM


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _rank_worker(rank, world, port, kind, q):
    try:
        import torch.distributed as dist

        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        c = _case(kind)
        m = c["m"]
        z0, n = seis.slab_bounds(c["nz"], world, rank)
        sl = {k: (None if v is None else np.ascontiguousarray(v[z0:z0 + n])) for k, v in m.items()}
        comm = seis.Comm.peer(world, rank, 0, float(m["vp"].max()))
        mod = seis.Model(_grid(c), kind, sl["vp"], vs=sl.get("vs"), rho=sl.get("rho"), comm=comm)
        assert (mod.z0, mod.nz_local) == (z0, n)
        mod.enable_peer_halo()
        out = _run(kind, c, mod)
        # second shot on the same model: the flag counters carry on across calls
        out2 = _run(kind, c, mod)
        mod.close()
        dist.barrier()
        comm.close()
        q.put((rank, z0, out, out2))
        dist.destroy_process_group()
    except Exception as e:  # report instead of hanging the parent
        import traceback

        q.put((rank, None, traceback.format_exc(), str(e)))


@pytest.mark.parametrize("kind,P", [("acoustic", 2), ("iso", 3), ("elastic", 2), ("acoustic", 3)])
def test_peer_ranks_on_one_gpu_bitwise(kind, P):
    import torch.multiprocessing as mp

    c = _case(kind)
    m = c["m"]
    mod = seis.Model(_grid(c), kind, m["vp"], vs=m.get("vs"), rho=m.get("rho"))
    ref = _run(kind, c, mod)
    mod.close()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_rank_worker, args=(r, P, port, kind, q)) for r in range(P)]
    for p in procs:
        p.start()
    res = {}
    try:
        for _ in range(P):
            r, z0, out, out2 = q.get(timeout=600)
            assert z0 is not None, out
            res[r] = (z0, out, out2)
    finally:
        for p in procs:
            p.join(timeout=60)
            if p.is_alive():
                p.kill()
    for r in range(P):
        z0, out, out2 = res[r]
        for o in (out, out2):
            sg, fields, img, img2 = o
            n = img.shape[0]
            assert np.array_equal(sg, ref[0])  # the binding sums the rank-owned columns
            for a, b in zip(fields, ref[1]):
                assert np.array_equal(a, b[z0:z0 + n])
            assert np.array_equal(img, ref[2][z0:z0 + n])
            assert np.array_equal(img2, ref[3][z0:z0 + n])


@pytest.mark.parametrize("kind", ["iso", "acoustic", "elastic"])
def test_short_tail_chunk_decomposition_bitwise(kind, monkeypatch):
    """Slabs of 65 planes: an even split into >= 8-plane chunks would leave a 2-plane last
    chunk, so the planes a neighbour needs would straddle an interior chunk.  The chunking
    keeps >= 4 planes in the first and last chunk of every slab; receivers injected right at
    the slab face, copy exchange and direct stores, forward + RTM == one slab bitwise."""
    nx, ny, nz = 48, 36, 130
    el = kind == "elastic"
    m = inputs.random_media((nz, ny, nx), seed=33, elastic=el)
    h, dt, nt, snap = 10.0, 5e-4, 30, 3
    w = inputs.source_series(kind, nt, dt, 35.0)
    rec = np.asarray([[10 + t, 7 + (t % 5), 59 + t] for t in range(12)], np.int32)
    data = np.random.default_rng(6).standard_normal((nt, rec.shape[0])).astype(np.float32)
    runs = []
    for P, copy in ((1, "0"), (2, "1"), (2, "0")):
        monkeypatch.setenv("SEIS_GHOST_COPY", copy)
        g = seis.Grid(nx, ny, nz, h, dt, nb=5, free_surface=int(el), pml_f=35.0, slabs=P)
        mod = seis.Model(g, kind, m["vp"], vs=m.get("vs"), rho=m.get("rho"))
        shot = seis.Shot((nx // 2, ny // 2, 64), w, rec, rec_component=2, snap_period=snap)
        sg = np.zeros((nt, rec.shape[0]), np.float32)
        mod.forward_model(shot, sg)
        img = np.zeros((nz, ny, nx), np.float32)
        mod.migrate(shot, data, img)
        runs.append((sg, img))
        mod.close()
    for sg, img in runs[1:]:
        assert np.array_equal(sg, runs[0][0])
        assert np.array_equal(img, runs[0][1])
