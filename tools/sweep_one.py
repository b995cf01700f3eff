"""Time one library build (selected by SEIS_LIBPATH) on short ISO / acoustic / elastic runs."""
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ppopp_qawasmehchc15_b200 as seis  # noqa: E402
from paper_conf_ppopp_qawasmehchc15_b200 import inputs  # noqa: E402

name = sys.argv[1]
dev = torch.device("cuda", 0)
res = {"variant": name, "lib": os.environ.get("SEIS_LIBPATH")}


def timed(model, shot, nrep=2):
    buf = torch.empty((shot.nt, shot.nrec), device=dev)
    model.forward_model(shot, buf)
    torch.cuda.synchronize()
    seis.profile(True)
    for _ in range(nrep):
        model.forward_model(shot, buf)
    torch.cuda.synchronize()
    seis.profile(False)
    return {k: round(v[0] / v[1], 4) for k, v in seis.profile_read().items()}


n = 512
vp = np.full((n, n, n), 2000.0, np.float32)
vp[n // 3:] = 3000.0
m = seis.Model(seis.Grid(n, n, n, 10.0, 1e-3, nb=20), "iso", vp)
w = inputs.source_series("iso", 60, 1e-3, 15.0)
res["iso_512"] = timed(m, seis.Shot((n // 2, n // 2, 24), w, np.asarray([[10, 10, 24]], np.int32)))
m.close()
try:  # split-field PML (O6b) variant of the same run
    m = seis.Model(seis.Grid(n, n, n, 10.0, 1e-3, nb=20, iso_pml=1), "iso", vp)
    res["iso_512_spml"] = timed(m, seis.Shot((n // 2, n // 2, 24), w, np.asarray([[10, 10, 24]], np.int32)))
    m.close()
except Exception as e:  # older builds without iso_pml
    res["iso_512_spml"] = str(e)[:100]
del vp
wl = inputs.c2(n=512, nt=60)
m = seis.Model(seis.Grid(wl.nx, wl.ny, wl.nz, wl.h, wl.dt, nb=wl.nb, pml_f=wl.fp), "acoustic",
               wl.model["vp"], rho=wl.model["rho"])
res["c2_512"] = timed(m, seis.Shot(wl.src, wl.wavelet, wl.rec))
m.close()
wl = inputs.c3(nt=40)
m = seis.Model(seis.Grid(wl.nx, wl.ny, wl.nz, wl.h, wl.dt, nb=wl.nb, free_surface=1, pml_f=wl.fp),
               "elastic", wl.model["vp"], vs=wl.model["vs"], rho=wl.model["rho"])
res["c3_384"] = timed(m, seis.Shot(wl.src, wl.wavelet, wl.rec))
m.close()
if os.environ.get("SWEEP_NOPML"):  # the same without absorbing layers (cost of the C-PML paths)
    m = seis.Model(seis.Grid(wl.nx, wl.ny, wl.nz, wl.h, wl.dt, nb=0, free_surface=1, pml_f=wl.fp),
                   "elastic", wl.model["vp"], vs=wl.model["vs"], rho=wl.model["rho"])
    res["c3_384_nopml"] = timed(m, seis.Shot(wl.src, wl.wavelet, wl.rec))
    m.close()
    wl = inputs.c2(n=512, nt=60)
    m = seis.Model(seis.Grid(wl.nx, wl.ny, wl.nz, wl.h, wl.dt, nb=0, pml_f=wl.fp), "acoustic",
                   wl.model["vp"], rho=wl.model["rho"])
    res["c2_512_nopml"] = timed(m, seis.Shot(wl.src, wl.wavelet, wl.rec))
    m.close()
print(json.dumps(res))
