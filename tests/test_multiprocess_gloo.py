"""World-size-2 checks of the multi-process (one process per GPU) host logic on CPU with
the gloo backend -- every check runs product code, not a re-typed copy of it:

1. ``Comm.broadcast_unique_id`` (the NCCL-id broadcast ``Comm.from_torch_distributed`` uses)
   gives every rank the id rank 0 drew with ``seis_comm_unique_id``;
2. the z-slab partition of the C ABI (``seis_slab_bounds``, P:175 sub-domains) tiles [0, nz)
   identically on every rank, with sizes differing by at most one;
3. the per-rank model generation of ``bench.py --gpus N`` (``inputs.layered_acoustic`` with
   ``z0 / nzl``: each rank builds only its slab) concatenates over the ranks to exactly the
   whole-grid model;
4. the receivers of a shot have exactly one owning rank (the slab holding their z), the rule
   that makes the library's seismogram all-reduce exact.
"""
import os
import socket

import numpy as np
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    import torch
    import torch.distributed as dist

    import paper_conf_ppopp_qawasmehchc15_b200 as seis
    from paper_conf_ppopp_qawasmehchc15_b200 import inputs

    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        # 1. NCCL unique id broadcast
        got = seis.Comm.broadcast_unique_id()
        ids = [None] * world
        dist.all_gather_object(ids, got)
        assert all(x == ids[0] for x in ids) and len(ids[0]) == 128
        assert any(ids[0]), "rank 0 must have drawn a non-zero NCCL id"
        # 2. slab partition (C ABI) agrees across ranks and tiles [0, nz)
        for nz in (512, 1024, 45, 9):
            z0, n = seis.slab_bounds(nz, world, rank)
            allb = [None] * world
            dist.all_gather_object(allb, (z0, n))
            assert allb[0][0] == 0 and sum(b[1] for b in allb) == nz
            assert all(allb[r][0] + allb[r][1] == allb[r + 1][0] for r in range(world - 1))
            assert max(b[1] for b in allb) - min(b[1] for b in allb) <= 1
        # 3. per-rank model slabs (bench.py weak / strong scaling) == the whole model
        nx, ny, nz = 40, 24, 70
        z0, n = seis.slab_bounds(nz, world, rank)
        mine = inputs.layered_acoustic(nx, ny, nz, z0=z0, nzl=n)
        for key in ("vp", "rho"):
            parts = [None] * world
            dist.all_gather_object(parts, mine[key])
            whole = inputs.layered_acoustic(nx, ny, nz)[key]
            assert np.array_equal(np.concatenate(parts, axis=0), whole), key
        # 4. receiver ownership: each receiver's z lies in exactly one rank's slab
        rng = np.random.default_rng(7)
        recz = rng.integers(0, nz, 200)
        owned = torch.from_numpy(((recz >= z0) & (recz < z0 + n)).astype(np.int64))
        dist.all_reduce(owned)
        assert np.all(owned.numpy() == 1)
        q.put((rank, "ok"))
    except Exception as e:  # pragma: no cover - reported to the parent
        q.put((rank, repr(e)))
    finally:
        dist.destroy_process_group()


def test_world_size_2_host_logic():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(120)
    res = dict(q.get(timeout=5) for _ in range(2))
    assert res == {0: "ok", 1: "ok"}, res
