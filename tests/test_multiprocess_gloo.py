"""World-size-2 checks of the multi-process (one process per GPU) host logic on CPU
with the gloo backend: NCCL-id broadcast, slab partition agreement with the C ABI,
and the exact seismogram assembly rule (every receiver column has one owner)."""
import os
import socket

import numpy as np
import pytest
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
    from paper_conf_ppopp_qawasmehchc15_b200 import dist as sd

    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        # 1. NCCL unique id broadcast (rank 0 draws it; deterministic fake id on hosts
        #    where NCCL cannot bootstrap)
        def uid():
            try:
                return seis.Comm.unique_id()
            except Exception:
                return bytes(range(128))

        got = sd.broadcast_unique_id(uid)
        ids = [None] * world
        dist.all_gather_object(ids, got)
        assert all(x == ids[0] for x in ids) and len(ids[0]) == 128
        # 2. slab partition: Python helper == C ABI, slabs tile [0, nz)
        for nz in (512, 1024, 45):
            z0, n = sd.slab_of(nz, world, rank)
            assert (z0, n) == seis.slab_bounds(nz, world, rank)
            allb = [None] * world
            dist.all_gather_object(allb, (z0, n))
            assert allb[0][0] == 0 and sum(b[1] for b in allb) == nz
            assert all(allb[r][0] + allb[r][1] == allb[r + 1][0] for r in range(world - 1))
        # 3. seismogram assembly: sum over ranks of owned columns == full seismogram, bitwise
        rng = np.random.default_rng(7)
        nz, nt = 64, 20
        rec = np.stack([rng.integers(0, 32, 50), rng.integers(0, 32, 50), rng.integers(0, nz, 50)], 1)
        full = rng.standard_normal((nt, 50)).astype(np.float32)
        part = torch.from_numpy(sd.assemble_seismogram(full, rec, nz, world, rank))
        dist.all_reduce(part)
        assert np.array_equal(part.numpy(), full)
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
