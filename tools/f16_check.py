"""fp16 vs fp32 RTM snapshots on the C4 salt model at 128^3 and 256^3 (image relative L2);
forward-modeled data, migration on the true model.  On a B200: python tools/f16_check.py"""
import os, sys, json, numpy as np, torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ppopp_qawasmehchc15_b200 as seis
from paper_conf_ppopp_qawasmehchc15_b200 import inputs
res = {}
for n in (128, 256):
    wl = inputs.c4(n=n, nt=800 if n == 128 else 1000, snap=20)
    g = seis.Grid(wl.nx, wl.ny, wl.nz, wl.h, wl.dt, nb=wl.nb, pml_f=wl.fp)
    true = seis.Model(g, "acoustic", wl.model["vp"], rho=wl.model["rho"])
    shot = seis.Shot(wl.src, wl.wavelet, wl.rec, snap_period=wl.snap)
    data = true.forward_model(shot); torch.cuda.synchronize(); true.close()
    mig = seis.Model(g, "acoustic", wl.migration_model["vp"] if hasattr(wl, "migration_model") else wl.model["vp"],
                     rho=wl.migration_model["rho"] if hasattr(wl, "migration_model") else wl.model["rho"])
    out = {}
    for f16 in (0, 1):
        img = torch.zeros((wl.nz, wl.ny, wl.nx), device="cuda")
        shot.snap_fp16 = f16
        mig.migrate(shot, data, img); torch.cuda.synchronize()
        out[f16] = img.cpu().numpy().astype(np.float64)
    d = np.linalg.norm(out[1] - out[0]) / np.linalg.norm(out[0])
    res[n] = d
    print(n, "fp16 vs fp32 image rel L2", d, flush=True)
