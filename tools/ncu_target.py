"""Small driver for ncu captures: one C2-shaped (default 512^3) forward shot of a few steps,
or one ISO / elastic / RTM shot.  Not a benchmark (numbers under ncu are never bench values).

    python tools/ncu_target.py [--kind acoustic|iso|elastic|rtm] [--n 512] [--nt 4]
"""
import argparse
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ppopp_qawasmehchc15_b200 as seis  # noqa: E402
from paper_conf_ppopp_qawasmehchc15_b200 import inputs  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--kind", default="acoustic")
ap.add_argument("--n", type=int, default=512)
ap.add_argument("--nt", type=int, default=4)
a = ap.parse_args()
dev = torch.device("cuda", 0)
if a.kind in ("acoustic", "rtm"):
    wl = inputs.c2(n=a.n, nt=a.nt) if a.kind == "acoustic" else inputs.c4(n=a.n, nt=a.nt, snap=2)
    g = seis.Grid(wl.nx, wl.ny, wl.nz, wl.h, wl.dt, nb=wl.nb, pml_f=wl.fp)
    m = seis.Model(g, "acoustic", wl.model["vp"], rho=wl.model["rho"])
elif a.kind == "iso":
    wl = inputs.c1(n=a.n, nt=a.nt, nb=20)
    g = seis.Grid(wl.nx, wl.ny, wl.nz, wl.h, wl.dt, nb=wl.nb)
    m = seis.Model(g, "iso", wl.model["vp"])
else:
    wl = inputs.c3(n=a.n, nt=a.nt)
    g = seis.Grid(wl.nx, wl.ny, wl.nz, wl.h, wl.dt, nb=wl.nb, free_surface=1, pml_f=wl.fp)
    m = seis.Model(g, "elastic", wl.model["vp"], vs=wl.model["vs"], rho=wl.model["rho"])
shot = seis.Shot(wl.src, wl.wavelet, wl.rec, snap_period=getattr(wl, "snap", 1))
buf = torch.empty((wl.nt, shot.nrec), device=dev)
if a.kind == "rtm":
    img = torch.zeros((wl.nz, wl.ny, wl.nx), device=dev)
    m.migrate(shot, buf, img)
else:
    m.forward_model(shot, buf)
torch.cuda.synchronize()
print("ok", a.kind, a.n, a.nt, "launches", seis.Model.launches())
