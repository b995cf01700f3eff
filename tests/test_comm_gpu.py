"""NCCL code paths of the library on ONE GPU (the only multi-GPU evidence a 1-GPU box can
give): a 1-rank NCCL communicator (seis_comm_create with nranks = 1).

* forward_model with the communicator runs the seismogram ncclAllReduce (P:222 results
  assembled across sub-domains; an identity for one rank) inside the shot's CUDA graph,
  and must return bitwise the communicator-less result, on capture and on replay;
* seis_image_reduce (shot-parallel RTM, the sum over shots of P:111 across ranks) must
  leave a 1-rank image bitwise unchanged, and a migrate with the communicator must equal
  the one without.
"""
import numpy as np
import pytest

import paper_conf_ppopp_qawasmehchc15_b200 as seis
from paper_conf_ppopp_qawasmehchc15_b200 import inputs

pytestmark = pytest.mark.gpu

NX, NY, NZ = 64, 40, 48
H, DT, FP = 10.0, 6e-4, 30.0


@pytest.fixture(scope="module")
def comm1():
    c = seis.Comm(1, 0, seis.Comm.unique_id(), 0)
    yield c
    c.close()


@pytest.mark.parametrize("kind", ["iso", "acoustic", "elastic"])
def test_one_rank_nccl_forward_bitwise(kind, comm1):
    torch = pytest.importorskip("torch")
    m = inputs.random_media((NZ, NY, NX), seed=51, elastic=(kind == "elastic"))
    g = seis.Grid(NX, NY, NZ, H, DT, nb=6, pml_f=FP)
    nt = 50
    xs = np.arange(2, NX - 2, 3)
    rec = np.stack([xs, np.full_like(xs, NY // 2), np.full_like(xs, 9)], 1).astype(np.int32)
    shot = seis.Shot((NX // 2, NY // 2, NZ // 2), inputs.source_series(kind, nt, DT, FP), rec)
    a = seis.Model(g, kind, m["vp"], vs=m.get("vs"), rho=m.get("rho"))
    ref = a.forward_model(shot)
    a.close()
    b = seis.Model(g, kind, m["vp"], vs=m.get("vs"), rho=m.get("rho"), comm=comm1, device=0)
    out = torch.zeros_like(ref)
    b.forward_model(shot, out)  # capture (graph incl. the all-reduce)
    assert torch.equal(out, ref)
    out.zero_()
    b.forward_model(shot, out)  # replay
    assert torch.equal(out, ref)
    b.close()


def test_one_rank_image_reduce_and_migrate(comm1):
    torch = pytest.importorskip("torch")
    m = inputs.random_media((NZ, NY, NX), seed=52)
    g = seis.Grid(NX, NY, NZ, H, DT, nb=6, pml_f=FP)
    nt = 40
    xs = np.arange(2, NX - 2, 3)
    rec = np.stack([xs, np.full_like(xs, NY // 2), np.full_like(xs, 9)], 1).astype(np.int32)
    shot = seis.Shot((NX // 2, NY // 2, 10), inputs.source_series("acoustic", nt, DT, FP), rec, snap_period=4)
    data = torch.from_numpy(np.random.default_rng(2).standard_normal((nt, rec.shape[0])).astype(np.float32)).cuda()
    a = seis.Model(g, "acoustic", m["vp"], rho=m["rho"])
    ref = torch.zeros((NZ, NY, NX), device="cuda:0")
    a.migrate(shot, data, ref)
    a.close()
    b = seis.Model(g, "acoustic", m["vp"], rho=m["rho"], comm=comm1, device=0)
    img = torch.zeros_like(ref)
    b.migrate(shot, data, img)
    assert torch.equal(img, ref)
    comm1.reduce_image(img)  # sum over one rank: identity
    torch.cuda.synchronize()
    assert torch.equal(img, ref)
    b.close()
    # a host image is refused (the reduction works on device buffers)
    with pytest.raises(seis.SeisError):
        comm1.reduce_image(np.zeros(8, np.float32))
