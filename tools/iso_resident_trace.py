"""Per-step phase times of the resident small-grid ISO kernel (iso_resident_kernel, C1 64^3) from
a -DSEIS_AS_TRACE=1 build: thread 0's clock64 at step start, compute done, halo done, and after
the closing barrier; medians over bricks and the middle steps, in SM cycles.
    python tools/iso_resident_trace.py [--defines A=1,B=2]"""
import argparse
import ctypes as C
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--defines", default="")
    a = ap.parse_args()
    from paper_conf_ppopp_qawasmehchc15_b200 import build

    lib = build.build(force=True, defines=["SEIS_AS_TRACE=1"] + [d for d in a.defines.split(",") if d],
                      out="/tmp/libseis_trace.so")
    os.environ["SEIS_LIBPATH"] = lib
    import numpy as np
    import torch

    import paper_conf_ppopp_qawasmehchc15_b200 as seis
    from paper_conf_ppopp_qawasmehchc15_b200 import inputs

    seis._LIBPATH = lib
    wl = inputs.c1()
    m = seis.Model(seis.Grid(wl.nx, wl.ny, wl.nz, wl.h, wl.dt, nb=wl.nb), "iso", wl.model["vp"])
    shot = seis.Shot(wl.src, wl.wavelet, wl.rec)
    out = torch.zeros((wl.nt, shot.nrec), device="cuda:0")
    for _ in range(2):
        m.forward_model(shot, out)
    torch.cuda.synchronize()
    L = seis.lib()
    L.seis_debug_trace.restype = C.c_void_p
    L.seis_debug_trace.argtypes = [C.POINTER(C.c_uint64)]
    n = C.c_uint64()
    p = L.seis_debug_trace(C.byref(n))
    buf = np.ctypeslib.as_array((C.c_uint64 * n.value).from_address(p)).copy().astype(np.float64)
    t = buf.reshape(-1, wl.nt, 4)[:, 20:wl.nt - 20]
    res = {
        "bricks": t.shape[0],
        "step_cycles": float(np.median(np.diff(t[:, :, 0], axis=1))),
        "compute": float(np.median(t[:, :, 1] - t[:, :, 0])),
        "sync1_centre_halo": float(np.median(t[:, :, 2] - t[:, :, 1])),
        "sync2": float(np.median(t[:, :, 3] - t[:, :, 2])),
        "tail_to_next": float(np.median(t[:, 1:, 0] - t[:, :-1, 3])),
        "halo_p90": float(np.percentile(t[:, :, 2] - t[:, :, 1], 90)),
        "sync2_p90": float(np.percentile(t[:, :, 3] - t[:, :, 2], 90)),
    }
    print(json.dumps(res))


if __name__ == "__main__":
    main()
