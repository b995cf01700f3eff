"""Small-grid cases that launch every kernel variant of libseis, for compute-sanitizer
(memcheck / racecheck / synccheck on 32^3 - 64^3 grids):

    compute-sanitizer --tool memcheck  python tools/sanitize_cases.py
    compute-sanitizer --tool racecheck python tools/sanitize_cases.py --quick
    compute-sanitizer --tool synccheck python tools/sanitize_cases.py

Variants: ISO z-march (damped layer, split-field PML, 1 / 3 slabs, the resident-brick and
grid-stride persistent small-grid kernels), acoustic split V / P (1 and 3 slabs: direct ghost stores, the copy exchange, the
serial order), the fused acoustic step (cooperative, counters), elastic V / S (free surface,
C-PML), RTM of every kind (imaging + snapshot epilogues, fp32 and 24-bit snapshots,
checkpointing), receiver injection / gather, host staging buffers.  Each case only checks
that results are finite; parity lives in tests/.
"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402

import paper_conf_ppopp_qawasmehchc15_b200 as seis  # noqa: E402
from paper_conf_ppopp_qawasmehchc15_b200 import inputs  # noqa: E402


def case(kind, shape, nb=4, fs=0, slabs=1, iso_pml=0, nt=6, rtm=True, env=None, ck=0, bits=32):
    env = env or {}
    old = {k: os.environ.get(k) for k in env}
    os.environ.update(env)
    try:
        nz, ny, nx = shape
        m = inputs.random_media(shape, seed=9, elastic=(kind == "elastic"))
        g = seis.Grid(nx, ny, nz, 10.0, 4e-4, nb=nb, free_surface=fs, pml_f=30.0, slabs=slabs, iso_pml=iso_pml)
        mod = seis.Model(g, kind, m["vp"], vs=m.get("vs"), rho=m.get("rho"))
        rec = np.asarray([[1, 2, 0], [nx - 1, ny - 1, nz - 1], [nx // 2, ny // 2, nz // 2], [nx // 2, ny // 2, nz // 2]],
                         np.int32)
        w = inputs.source_series(kind, nt, 4e-4, 30.0)
        shot = seis.Shot((nx // 2, ny // 2, max(1, nz // 3)), w, rec, snap_period=2, ckpt_period=ck, snap_bits=bits)
        out = np.zeros((nt, rec.shape[0]), np.float32)
        mod.forward_model(shot, out)
        assert np.all(np.isfinite(out))
        if rtm:
            img = np.zeros(shape, np.float32)
            data = np.random.default_rng(1).standard_normal((nt, rec.shape[0])).astype(np.float32)
            mod.migrate(shot, data, img)
            assert np.all(np.isfinite(img))
        mod.close()
        print(f"ok {kind} {shape} nb={nb} fs={fs} slabs={slabs} iso_pml={iso_pml} ck={ck} bits={bits} {env}",
              flush=True)
    finally:
        for k, v in old.items():
            if v is None:
                os.environ.pop(k, None)
            else:
                os.environ[k] = v


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--quick", action="store_true", help="fewer, smaller cases (racecheck)")
    a = ap.parse_args()
    s = (24, 20, 36) if a.quick else (40, 36, 70)
    # ISO
    case("iso", s, nb=4, env={"SEIS_NO_PERSIST": "1"})
    case("iso", s, nb=4)  # resident-brick small-grid kernel
    case("iso", s, nb=4, env={"SEIS_ISO_RESIDENT": "0"})  # grid-stride small-grid kernel
    case("iso", s, nb=4, iso_pml=1)
    case("iso", s, nb=4, slabs=3, env={"SEIS_NO_PERSIST": "1"})
    # acoustic: split pair, decompositions, fused step
    case("acoustic", s, nb=4)
    case("acoustic", s, nb=4, slabs=3)
    case("acoustic", s, nb=4, slabs=3, env={"SEIS_GHOST_COPY": "1"})
    case("acoustic", s, nb=4, slabs=3, env={"SEIS_NO_OVERLAP": "1"})
    case("acoustic", s, nb=4, env={"SEIS_AC_STEP": "1"})
    case("acoustic", s, nb=0, env={"SEIS_AC_STEP": "1"}, ck=2, bits=24)
    case("acoustic", s, nb=4, ck=2)
    case("acoustic", s, nb=4, bits=24)
    # elastic (warp-specialized producer)
    case("elastic", s, nb=4, fs=1)
    case("elastic", s, nb=4, fs=0, slabs=3)
    case("elastic", s, nb=4, fs=1, bits=24, ck=2)
    if not a.quick:
        case("iso", s, nb=4, iso_pml=1, slabs=2, ck=2)
        case("elastic", s, nb=0, fs=1, env={"SEIS_NO_OVERLAP": "1"}, slabs=2)
    print("all cases ok")


if __name__ == "__main__":
    main()
