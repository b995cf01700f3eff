"""B200-native seismic modeling and RTM hot path (Qawasmeh et al., PMAM'15).

Thin ctypes binding over the C ABI in ``include/seis.h`` (``libseis.so``, built
in-tree for sm_100a by ``build.py``).  Argument marshalling only: every step of
the path runs in the library's CUDA kernels.  There is no CPU fallback: if
the library or a CUDA device is missing the calls raise.

torch is used only for device memory (tensors whose ``data_ptr()`` is passed),
streams (``torch.cuda.current_stream().cuda_stream``) and process groups (the
NCCL unique id broadcast in ``Comm.from_torch_distributed``).
"""
from __future__ import annotations

import ctypes as C
import os
from dataclasses import dataclass
from typing import Optional

import numpy as np

__all__ = ["Grid", "Shot", "Model", "Comm", "SeisError", "lib", "slab_bounds", "ISO", "ACOUSTIC",
           "ELASTIC", "KINDS"]

_HERE = os.path.dirname(os.path.abspath(__file__))
# SEIS_LIBPATH selects an alternative build of the same library (tools/sweep.py tuning runs)
_LIBPATH = os.environ.get("SEIS_LIBPATH", os.path.join(_HERE, "libseis.so"))

ISO, ACOUSTIC, ELASTIC = 0, 1, 2
KINDS = {"iso": ISO, "acoustic": ACOUSTIC, "elastic": ELASTIC}
STATUS = {0: "SEIS_OK", 1: "SEIS_EINVAL", 2: "SEIS_ECFL", 3: "SEIS_ENOMEM", 4: "SEIS_ECUDA",
          5: "SEIS_ENCCL", 6: "SEIS_EUNSUPPORTED"}

# every symbol include/seis.h declares
SYMBOLS = ["seis_comm_unique_id", "seis_comm_create", "seis_comm_destroy", "seis_image_reduce",
           "seis_comm_create_peer", "seis_model_peer_export", "seis_model_peer_import",
           "seis_model_create",
           "seis_slab_bounds", "seis_model_slab", "seis_model_destroy", "seis_forward_model",
           "seis_migrate", "seis_get_field", "seis_memory_required", "seis_profile",
           "seis_profile_read", "seis_last_launch_count",
           "seis_version", "seis_last_error"]


class SeisError(RuntimeError):
    def __init__(self, status: int, msg: str):
        self.status = status
        self.name = STATUS.get(status, str(status))
        super().__init__(f"{self.name}: {msg}")


class _CGrid(C.Structure):
    _fields_ = [("nx", C.c_int32), ("ny", C.c_int32), ("nz", C.c_int32), ("h", C.c_float),
                ("dt", C.c_float), ("nb", C.c_int32), ("free_surface", C.c_int32),
                ("pml_R", C.c_float), ("pml_f", C.c_float), ("slabs", C.c_int32),
                ("iso_pml", C.c_int32)]


class _CShot(C.Structure):
    _fields_ = [("sx", C.c_int32), ("sy", C.c_int32), ("sz", C.c_int32),
                ("wavelet", C.POINTER(C.c_float)), ("nt", C.c_int32), ("nrec", C.c_int32),
                ("rec", C.POINTER(C.c_int32)), ("rec_component", C.c_int32),
                ("snap_period", C.c_int32), ("ckpt_period", C.c_int32), ("snap_bits", C.c_int32)]


_lib = None


def lib():
    """Load libseis.so (raises if it was not built: there is no fallback)."""
    global _lib
    if _lib is None:
        if not os.path.exists(_LIBPATH):
            raise RuntimeError(f"{_LIBPATH} is missing: run `python -m "
                               "paper_conf_ppopp_qawasmehchc15_b200.build` (no CPU fallback)")
        L = C.CDLL(_LIBPATH)
        vp = C.c_void_p
        L.seis_comm_unique_id.argtypes = [C.POINTER(C.c_uint8)]
        L.seis_comm_create.argtypes = [C.c_int32, C.c_int32, C.POINTER(C.c_uint8), C.c_int32,
                                       C.POINTER(vp)]
        L.seis_comm_destroy.argtypes = [vp]
        L.seis_image_reduce.argtypes = [vp, vp, C.c_uint64, vp]
        L.seis_comm_create_peer.argtypes = [C.c_int32, C.c_int32, C.c_int32, C.c_double, C.POINTER(vp)]
        L.seis_model_peer_export.argtypes = [vp, vp, C.c_uint64, C.POINTER(C.c_uint64)]
        L.seis_model_peer_import.argtypes = [vp, vp, C.c_uint64, vp, C.c_uint64]
        L.seis_model_create.argtypes = [C.POINTER(_CGrid), C.c_int, vp, vp, vp, vp, C.c_int32,
                                        C.POINTER(vp)]
        L.seis_slab_bounds.argtypes = [C.c_int32, C.c_int32, C.c_int32, C.POINTER(C.c_int32),
                                       C.POINTER(C.c_int32)]
        L.seis_model_slab.argtypes = [vp, C.POINTER(C.c_int32), C.POINTER(C.c_int32)]
        L.seis_model_destroy.argtypes = [vp]
        L.seis_forward_model.argtypes = [vp, C.POINTER(_CShot), vp, vp]
        L.seis_migrate.argtypes = [vp, C.POINTER(_CShot), vp, vp, vp]
        L.seis_get_field.argtypes = [vp, C.c_int32, vp, vp]
        L.seis_memory_required.argtypes = [C.POINTER(_CGrid), C.c_int, C.POINTER(_CShot),
                                           C.c_int32, C.POINTER(C.c_uint64)]
        L.seis_profile.argtypes = [C.c_int32]
        L.seis_profile_read.argtypes = [C.c_int32, C.POINTER(C.c_double), C.POINTER(C.c_int64)]
        L.seis_last_launch_count.restype = C.c_int64
        L.seis_version.restype = C.c_char_p
        L.seis_last_error.restype = C.c_char_p
        for name in SYMBOLS:
            if name not in ("seis_last_launch_count", "seis_version", "seis_last_error"):
                getattr(L, name).restype = C.c_int
        _lib = L
    return _lib


def _check(rc: int):
    if rc != 0:
        raise SeisError(rc, lib().seis_last_error().decode(errors="replace"))


@dataclass
class Grid:
    nx: int
    ny: int
    nz: int
    h: float
    dt: float
    nb: int = 0
    free_surface: int = 0
    pml_R: float = 1e-3
    pml_f: float = 10.0
    slabs: int = 1
    iso_pml: int = 0  # ISO layer: 0 = damped wave (O6), 1 = split-field PML (O6b)

    def c(self) -> _CGrid:
        return _CGrid(self.nx, self.ny, self.nz, self.h, self.dt, self.nb, self.free_surface,
                      self.pml_R, self.pml_f, self.slabs, self.iso_pml)


@dataclass
class Shot:
    src: tuple
    wavelet: np.ndarray          # host fp32 [nt] (injected samples s[n], O11)
    rec: np.ndarray              # host int32 [nrec][3] (x, y, z)
    rec_component: int = 2
    snap_period: int = 1
    ckpt_period: int = 0         # RTM: 0 = all snapshots in HBM; c >= 1 = checkpointed segments of c
    snap_bits: int = 32          # RTM snapshot precision: 32 (fp32) or 24 (3/4 of the pool, 2^-16 rounding)

    def c(self):
        w = np.ascontiguousarray(self.wavelet, dtype=np.float32)
        r = np.ascontiguousarray(np.asarray(self.rec, dtype=np.int32).reshape(-1, 3))
        cs = _CShot(int(self.src[0]), int(self.src[1]), int(self.src[2]),
                    w.ctypes.data_as(C.POINTER(C.c_float)), w.shape[0], r.shape[0],
                    r.ctypes.data_as(C.POINTER(C.c_int32)), self.rec_component, self.snap_period,
                    self.ckpt_period, self.snap_bits)
        return cs, (w, r)

    @property
    def nt(self):
        return int(np.asarray(self.wavelet).shape[0])

    @property
    def nrec(self):
        return int(np.asarray(self.rec).reshape(-1, 3).shape[0])


def _ptr(a):
    """Raw pointer of a torch tensor (device or host) or numpy array (host)."""
    if a is None:
        return None
    if isinstance(a, np.ndarray):
        assert a.flags.c_contiguous and a.dtype == np.float32, "need C-contiguous float32"
        return a.ctypes.data
    assert a.is_contiguous() and str(a.dtype) == "torch.float32", "need contiguous float32"
    return a.data_ptr()


def _stream(stream):
    if stream is None:
        try:
            import torch

            if torch.cuda.is_available():
                return torch.cuda.current_stream().cuda_stream
        except Exception:
            pass
        return None
    if isinstance(stream, int):
        return stream
    return stream.cuda_stream


def slab_bounds(nz: int, nranks: int, rank: int):
    z0, n = C.c_int32(), C.c_int32()
    _check(lib().seis_slab_bounds(nz, nranks, rank, C.byref(z0), C.byref(n)))
    return z0.value, n.value


class Comm:
    """NCCL communicator for the z-slab decomposition (one process per GPU)."""

    peer_only = False

    def __init__(self, nranks: int, rank: int, uid: bytes, device: int):
        buf = (C.c_uint8 * 128).from_buffer_copy(uid)
        h = C.c_void_p()
        _check(lib().seis_comm_create(nranks, rank, buf, device, C.byref(h)))
        self.h, self.nranks, self.rank, self.device = h, nranks, rank, device

    @classmethod
    def peer(cls, nranks: int, rank: int, device: int, vmax: float):
        """Peer-only communicator (no NCCL; seis_comm_create_peer): the halo planes travel by
        direct peer stores once every rank's model ran enable_peer_halo().  vmax = global max vp."""
        self = cls.__new__(cls)
        h = C.c_void_p()
        _check(lib().seis_comm_create_peer(nranks, rank, device, float(vmax), C.byref(h)))
        self.h, self.nranks, self.rank, self.device, self.peer_only = h, nranks, rank, device, True
        return self

    @staticmethod
    def unique_id() -> bytes:
        buf = (C.c_uint8 * 128)()
        _check(lib().seis_comm_unique_id(buf))
        return bytes(buf)

    @classmethod
    def broadcast_unique_id(cls, group=None, device: Optional[int] = None) -> bytes:
        """Rank 0 of the torch.distributed group draws the 128-byte NCCL unique id
        (seis_comm_unique_id); every rank returns it (broadcast over the group's backend:
        a CUDA tensor on `device` for nccl, a CPU tensor for gloo)."""
        import torch
        import torch.distributed as dist

        rank = dist.get_rank(group)
        uid = cls.unique_id() if rank == 0 else bytes(128)
        on_gpu = dist.get_backend(group) == "nccl"
        t = torch.tensor(list(uid), dtype=torch.uint8,
                         device=f"cuda:{device if device is not None else torch.cuda.current_device()}"
                         if on_gpu else "cpu")
        dist.broadcast(t, 0, group=group)
        return bytes(t.cpu().tolist())

    @classmethod
    def from_torch_distributed(cls, device: int, group=None):
        """Create from an initialised torch.distributed group (broadcasts the NCCL id)."""
        import torch.distributed as dist

        uid = cls.broadcast_unique_id(group, device)
        return cls(dist.get_world_size(group), dist.get_rank(group), uid, device)

    def reduce_image(self, image, stream=None):
        """Sum a device image over all ranks in place (shot-parallel RTM, sum_s of P:111)."""
        n = image.numel() if hasattr(image, "numel") else int(np.asarray(image).size)
        _check(lib().seis_image_reduce(self.h, _ptr(image), n, _stream(stream)))
        return image

    def close(self):
        if getattr(self, "h", None):
            lib().seis_comm_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class Model:
    """A velocity model resident on one GPU (this process's z-slab)."""

    def __init__(self, grid: Grid, kind, vp, vs=None, rho=None, comm: Optional[Comm] = None,
                 device: int = 0):
        self.grid = grid
        self.kind = KINDS[kind] if isinstance(kind, str) else int(kind)
        arrs = [None if a is None else np.ascontiguousarray(a, dtype=np.float32)
                for a in (vp, vs, rho)]
        g = grid.c()
        h = C.c_void_p()
        _check(lib().seis_model_create(C.byref(g), self.kind, *[_ptr(a) for a in arrs],
                                       comm.h if comm is not None else None, device, C.byref(h)))
        self.h = h
        self.device = device
        self.comm = comm
        z0, n = C.c_int32(), C.c_int32()
        _check(lib().seis_model_slab(h, C.byref(z0), C.byref(n)))
        self.z0, self.nz_local = z0.value, n.value

    @property
    def local_shape(self):
        return (self.nz_local, self.grid.ny, self.grid.nx)

    def forward_model(self, shot: Shot, seis=None, stream=None):
        """Seismic modeling of one shot; returns seis [nt][nrec] (the given buffer, or a new
        device tensor)."""
        if seis is None:
            import torch

            seis = torch.empty((shot.nt, shot.nrec), dtype=torch.float32,
                               device=f"cuda:{self.device}")
        cs, keep = shot.c()
        _check(lib().seis_forward_model(self.h, C.byref(cs), _ptr(seis), _stream(stream)))
        if self.comm is not None and self.comm.peer_only and getattr(self, "_group", None) is not None:
            # the library leaves each rank its own receivers' columns (no NCCL): sum them here
            import torch
            import torch.distributed as dist

            t = torch.as_tensor(seis)
            if dist.get_backend(self._group) == "gloo" and t.is_cuda:
                c = t.cpu()
                dist.all_reduce(c, group=self._group)
                t.copy_(c)
            else:
                dist.all_reduce(t, group=self._group)
        return seis

    def enable_peer_halo(self, group=None):
        """Switch the rank faces to direct ghost-plane stores over peer memory (f4): export
        this rank's CUDA IPC blob, all-gather the blobs over the torch.distributed group,
        map the neighbours'.  Collective over the group (one rank per z-slab, rank order)."""
        import torch.distributed as dist

        n = C.c_uint64()
        _check(lib().seis_model_peer_export(self.h, None, 0, C.byref(n)))
        buf = (C.c_uint8 * n.value)()
        _check(lib().seis_model_peer_export(self.h, buf, n.value, C.byref(n)))
        blobs = [None] * dist.get_world_size(group)
        dist.all_gather_object(blobs, bytes(buf), group=group)
        r = dist.get_rank(group)
        lo = blobs[r - 1] if r > 0 else None
        hi = blobs[r + 1] if r + 1 < len(blobs) else None
        lob = (C.c_uint8 * len(lo)).from_buffer_copy(lo) if lo else None
        hib = (C.c_uint8 * len(hi)).from_buffer_copy(hi) if hi else None
        _check(lib().seis_model_peer_import(self.h, lob, len(lo) if lo else 0, hib, len(hi) if hi else 0))
        self._group = group if group is not None else dist.group.WORLD
        return self

    def migrate(self, shot: Shot, data, image, stream=None):
        """RTM of one shot; image [nz_local][ny][nx] is accumulated (+=)."""
        cs, keep = shot.c()
        _check(lib().seis_migrate(self.h, C.byref(cs), _ptr(data), _ptr(image), _stream(stream)))
        return image

    def get_field(self, which: int, out=None, stream=None):
        if out is None:
            out = np.empty(self.local_shape, dtype=np.float32)
        _check(lib().seis_get_field(self.h, which, _ptr(out), _stream(stream)))
        return out

    @staticmethod
    def launches() -> int:
        return int(lib().seis_last_launch_count())

    def close(self):
        if getattr(self, "h", None):
            lib().seis_model_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


KERNEL_IDS = {"iso_step": 0, "ac_v": 1, "ac_p": 2, "el_v": 3, "el_s": 4, "inject": 5,
              "gather": 6, "exchange": 7, "fs_mirror": 8, "ac_step": 9, "iso2": 10}


def profile(enable, sample: int = 1):
    """Start (resetting the counters) / stop per-kernel CUDA-event timing in the library.
    sample > 1: keep the forward shot's CUDA graph and time the launches of every sample-th
    time step through event nodes inside it (seis.h seis_profile)."""
    _check(lib().seis_profile((sample if sample > 1 else 1) if enable else 0))


def profile_read():
    """{kernel: (total_ms, launches)} for every kernel id with launches since profile(True)."""
    out = {}
    for name, k in KERNEL_IDS.items():
        ms, n = C.c_double(), C.c_int64()
        _check(lib().seis_profile_read(k, C.byref(ms), C.byref(n)))
        if n.value:
            out[name] = (ms.value, n.value)
    return out


def memory_required(grid: Grid, kind, shot: Optional[Shot] = None, nranks: int = 1) -> int:
    g = grid.c()
    out = C.c_uint64()
    if shot is not None:
        cs, keep = shot.c()
        _check(lib().seis_memory_required(C.byref(g), KINDS.get(kind, kind), C.byref(cs), nranks,
                                          C.byref(out)))
    else:
        _check(lib().seis_memory_required(C.byref(g), KINDS.get(kind, kind), None, nranks,
                                          C.byref(out)))
    return out.value
