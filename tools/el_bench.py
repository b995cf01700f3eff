"""C3-size timing of the elastic kernels on one B200 (per-kernel CUDA-event times and the
algorithmic-byte roofline fraction): python tools/el_bench.py [--n 384] [--nt 100]
Alternative builds via SEIS_LIBPATH (sweeps)."""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import paper_conf_ppopp_qawasmehchc15_b200 as seis  # noqa: E402
from paper_conf_ppopp_qawasmehchc15_b200 import inputs  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=384)
    ap.add_argument("--nt", type=int, default=100)
    ap.add_argument("--nb", type=int, default=20)
    a = ap.parse_args()
    wl = inputs.c3(n=a.n, nt=a.nt, nb=a.nb)
    g = seis.Grid(wl.nx, wl.ny, wl.nz, wl.h, wl.dt, nb=wl.nb, free_surface=1, pml_f=wl.fp)
    m = seis.Model(g, "elastic", wl.model["vp"], vs=wl.model["vs"], rho=wl.model["rho"])
    shot = seis.Shot(wl.src, wl.wavelet, wl.rec, rec_component=2)
    out = torch.zeros((a.nt, shot.nrec), device="cuda:0")
    stream = torch.cuda.current_stream()
    m.forward_model(shot, out, stream)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    for _ in range(3):
        m.forward_model(shot, out, stream)
    e1.record(stream)
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / 3
    seis.profile(True)
    m.forward_model(shot, out, stream)
    torch.cuda.synchronize()
    seis.profile(False)
    kp = seis.profile_read()
    W = wl.nb + 1
    psi = 8.0 * (2 * W / wl.nx + 2 * W / wl.ny + W / wl.nz) * 9 / 3.0 if wl.nb else 0.0
    hbm = 6538.3
    res = {"n": a.n, "nt": a.nt, "nb": a.nb, "ms_per_step": round(ms / a.nt, 4), "gpts_s": round(wl.npts * a.nt / (ms * 1e-3) / 1e9, 2),
           "seis_norm": float(out.norm().item())}
    for k, b in (("el_v", 52.0), ("el_s", 68.0)):
        t = kp[k][0] / kp[k][1]
        res[k] = {"ms": round(t, 4), "frac": round(wl.npts * (b + psi) / (t * 1e-3) / 1e9 / hbm, 4)}
    print(json.dumps(res))


if __name__ == "__main__":
    main()
