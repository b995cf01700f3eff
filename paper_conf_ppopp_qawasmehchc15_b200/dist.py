"""Host-side helpers of the z-slab decomposition across processes (one per GPU).

The data path (halo planes, seismogram all-reduce) runs inside libseis through
NCCL; these helpers are the process-group plumbing around it: broadcasting the
NCCL unique id over a torch.distributed group (any backend, gloo included) and
the slab / receiver-ownership arithmetic every rank must agree on (P:175:
"each domain may be divided into sub-domains mapped onto several hosts").
"""
from __future__ import annotations

import numpy as np


def slab_of(nz: int, world: int, rank: int):
    """(z0, nz_local) of `rank`: contiguous z-slabs, sizes differing by at most one
    (the same arithmetic as seis_slab_bounds)."""
    base, rem = divmod(nz, world)
    n = base + (1 if rank < rem else 0)
    return rank * base + min(rank, rem), n


def owner_of(z, nz: int, world: int):
    """Rank owning global plane(s) z (vectorised)."""
    z = np.asarray(z)
    bounds = np.asarray([slab_of(nz, world, r)[0] for r in range(world)] + [nz])
    return np.searchsorted(bounds, z, side="right") - 1


def broadcast_unique_id(uid_fn, group=None) -> bytes:
    """Rank 0 draws the 128-byte NCCL unique id with uid_fn(); every rank returns it."""
    import torch
    import torch.distributed as dist

    rank = dist.get_rank(group)
    uid = uid_fn() if rank == 0 else bytes(128)
    dev = "cpu"
    if dist.get_backend(group) == "nccl":
        dev = f"cuda:{torch.cuda.current_device()}"
    t = torch.tensor(list(uid), dtype=torch.uint8, device=dev)
    dist.broadcast(t, 0, group=group)
    return bytes(t.cpu().tolist())


def assemble_seismogram(local: np.ndarray, rec: np.ndarray, nz: int, world: int, rank: int):
    """Reference of the library's seismogram assembly: each rank fills the columns of the
    receivers its slab owns, zeros elsewhere; the all-reduce(sum) of these is exact
    because every column has exactly one owner.  Returns this rank's contribution."""
    own = owner_of(np.asarray(rec)[:, 2], nz, world) == rank
    out = np.zeros_like(local)
    out[:, own] = local[:, own]
    return out
