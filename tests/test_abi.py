"""C-ABI checks that need no GPU: the library loads, exports every symbol that
include/seis.h declares, and its pure host logic (slab bounds, validation order,
memory estimate) behaves; compute calls are not made here."""
import ctypes as C
import os
import re

import pytest

import paper_conf_ppopp_qawasmehchc15_b200 as seis

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared():
    src = open(os.path.join(ROOT, "include", "seis.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(seis_[a-z_]+)\s*\(", src)))


def test_header_symbols_match_binding_list():
    assert _declared() == sorted(seis.SYMBOLS)


def test_library_exports_every_declared_symbol():
    L = seis.lib()
    for name in _declared():
        assert hasattr(L, name), name
    out = os.popen(f"nm -D --defined-only {seis._LIBPATH}").read()
    for name in _declared():
        assert re.search(rf"\bT {name}\b", out), name


def test_version_and_error_strings():
    assert b"sm_100a" in seis.lib().seis_version()
    assert isinstance(seis.lib().seis_last_error(), bytes)


@pytest.mark.parametrize("nz,P", [(512, 1), (512, 3), (1024, 8), (10, 4), (7, 7)])
def test_slab_bounds_partition(nz, P):
    prev = 0
    sizes = []
    for r in range(P):
        z0, n = seis.slab_bounds(nz, P, r)
        assert z0 == prev
        prev = z0 + n
        sizes.append(n)
    assert prev == nz
    assert max(sizes) - min(sizes) <= 1


def test_slab_bounds_rejects_bad_rank():
    with pytest.raises(seis.SeisError) as e:
        seis.slab_bounds(64, 2, 2)
    assert e.value.name == "SEIS_EINVAL"


def test_memory_required_counts_snapshots():
    g = seis.Grid(128, 96, 64, 10.0, 8e-4, nb=10)
    import numpy as np

    sh = seis.Shot((1, 1, 1), np.zeros(201, np.float32), np.zeros((1, 3), np.int32), snap_period=20)
    m0 = seis.memory_required(g, "acoustic")
    m1 = seis.memory_required(g, "acoustic", sh)
    assert m1 - m0 == 10 * 128 * 96 * 64 * 4


def test_invalid_grid_is_rejected_before_touching_the_device():
    import numpy as np

    g = seis.Grid(16, 16, 16, 10.0, 1e-3, nb=7)  # 3 nb > 16
    with pytest.raises(seis.SeisError) as e:
        seis.Model(g, "iso", np.full((16, 16, 16), 2000.0, np.float32))
    assert e.value.name == "SEIS_EINVAL"
    g = seis.Grid(16, 16, 16, 10.0, 1e-3, free_surface=1)
    with pytest.raises(seis.SeisError) as e:
        seis.Model(g, "acoustic", np.full((16, 16, 16), 2000.0, np.float32),
                   rho=np.ones((16, 16, 16), np.float32))
    assert e.value.name == "SEIS_EUNSUPPORTED"


def test_no_cpu_fallback_without_a_device():
    """On a GPU-less host the product path must fail loudly, never compute on the CPU."""
    import numpy as np
    import torch

    if torch.cuda.is_available():
        pytest.skip("a CUDA device is present")
    g = seis.Grid(16, 16, 16, 10.0, 1e-3)
    with pytest.raises(seis.SeisError) as e:
        seis.Model(g, "iso", np.full((16, 16, 16), 2000.0, np.float32))
    assert e.value.name == "SEIS_ECUDA"


def test_memory_required_checkpointing():
    """f2: checkpointed RTM keeps c snapshots + ceil(nsnap/c)-1 state checkpoints; the
    C5 1024^3 single-GPU RTM (49 snapshots) only fits in 180 GB with checkpointing."""
    import numpy as np

    g = seis.Grid(128, 96, 64, 10.0, 8e-4, nb=10)
    pts = 128 * 96 * 64 * 4
    w = np.zeros(201, np.float32)
    rec = np.zeros((1, 3), np.int32)
    m0 = seis.memory_required(g, "acoustic")
    full = seis.memory_required(g, "acoustic", seis.Shot((1, 1, 1), w, rec, snap_period=20))
    c3 = seis.memory_required(g, "acoustic", seis.Shot((1, 1, 1), w, rec, snap_period=20, ckpt_period=3))
    c10 = seis.memory_required(g, "acoustic", seis.Shot((1, 1, 1), w, rec, snap_period=20, ckpt_period=10))
    assert c10 == full  # one segment = no checkpoint
    # 10 snapshots in segments of 3 -> 3 snapshots in the pool + 3 checkpoints of the state
    ck = (c3 - m0 - 3 * pts) / 3
    assert ck > 4 * pts  # 4 padded fields + C-PML slabs
    g5 = seis.Grid(1024, 1024, 1024, 10.0, 8e-4, nb=20)
    w5 = np.zeros(1000, np.float32)
    allsnap = seis.memory_required(g5, "acoustic", seis.Shot((1, 1, 1), w5, rec, snap_period=20))
    ckpt = seis.memory_required(g5, "acoustic", seis.Shot((1, 1, 1), w5, rec, snap_period=20, ckpt_period=10))
    assert allsnap > 180e9 > ckpt


def test_peer_mode_entry_points_validate_before_touching_the_device():
    """f4 peer halo ABI: argument errors are reported without a device; a NULL model is
    rejected by export / import."""
    import ctypes as C

    L = seis.lib()
    h = C.c_void_p()
    for args in ((0, 0, 0, 3000.0), (2, 2, 0, 3000.0), (2, -1, 0, 3000.0), (2, 0, 0, 0.0), (2, 0, 0, float("nan"))):
        assert L.seis_comm_create_peer(*args, C.byref(h)) == 1  # SEIS_EINVAL
    n = C.c_uint64()
    assert L.seis_model_peer_export(None, None, 0, C.byref(n)) == 1
    assert L.seis_model_peer_import(None, None, 0, None, 0) == 1


def test_iso_split_pml_rejected_for_other_kinds():
    import numpy as np

    vp = np.full((16, 16, 16), 2000.0, np.float32)
    with pytest.raises(seis.SeisError) as e:
        seis.Model(seis.Grid(16, 16, 16, 10.0, 1e-3, nb=4, iso_pml=1), "acoustic", vp, rho=vp)
    assert e.value.name == "SEIS_EUNSUPPORTED"


def test_memory_required_24bit_snapshots():
    import numpy as np

    g = seis.Grid(128, 96, 64, 10.0, 8e-4, nb=10)
    sh = seis.Shot((1, 1, 1), np.zeros(201, np.float32), np.zeros((1, 3), np.int32), snap_period=20)
    sh24 = seis.Shot((1, 1, 1), np.zeros(201, np.float32), np.zeros((1, 3), np.int32), snap_period=20,
                     snap_bits=24)
    m0 = seis.memory_required(g, "acoustic")
    assert seis.memory_required(g, "acoustic", sh24) - m0 == 10 * 128 * 96 * 64 * 3
    assert seis.memory_required(g, "acoustic", sh) - m0 == 10 * 128 * 96 * 64 * 4


def test_product_path_fails_loudly_without_the_library():
    """No CPU fallback: with the CUDA library missing, the binding raises (fresh process)."""
    import subprocess
    import sys

    code = ("import os; os.environ['SEIS_LIBPATH'] = '/nonexistent/libseis.so'\n"
            "import paper_conf_ppopp_qawasmehchc15_b200 as s\n"
            "try:\n    s.lib()\nexcept RuntimeError as e:\n    print('RAISED', e)\n")
    r = subprocess.run([sys.executable, "-c", code], capture_output=True, text=True, cwd=ROOT, timeout=120)
    assert "RAISED" in r.stdout and "no CPU fallback" in r.stdout


def test_product_package_never_touches_the_oracle():
    """The oracle is test infrastructure: nothing in the product package or its CUDA sources
    imports, includes or links it."""
    pkg = os.path.join(ROOT, "paper_conf_ppopp_qawasmehchc15_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h")):
                src = open(os.path.join(dirpath, f)).read()
                assert not re.search(r"^\s*(import|from)\s+oracle\b", src, re.M), f
                assert "oracle.h" not in src and "liboracle" not in src, f
