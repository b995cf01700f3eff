"""C1 (ISO 64^3, 200 steps; L2-resident, launch-bound): z-march path vs the persistent kernels.

    python tools/c1_sweep.py        # on a B200: one line per SEIS_ZCHUNK_MIN value
"""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
ONE = r'''
import json, sys, torch
sys.path.insert(0, sys.argv[1])
import paper_conf_ppopp_qawasmehchc15_b200 as seis
from paper_conf_ppopp_qawasmehchc15_b200 import inputs
wl = inputs.c1()
m = seis.Model(seis.Grid(wl.nx, wl.ny, wl.nz, wl.h, wl.dt, nb=wl.nb), "iso", wl.model["vp"])
shot = seis.Shot(wl.src, wl.wavelet, wl.rec)
buf = torch.empty((wl.nt, shot.nrec), device="cuda")
for _ in range(3): m.forward_model(shot, buf)
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(20): m.forward_model(shot, buf)
e1.record(); torch.cuda.synchronize()
ms = e0.elapsed_time(e1) / 20
print(json.dumps({"ms_per_shot": round(ms, 4), "gpts_s": round(wl.npts * wl.nt / (ms * 1e-3) / 1e9, 2)}))
'''

# pers: 0 z-march kernels (graph), 1 grid-stride persistent kernel (grid barriers),
# 2 resident bricks (neighbour counters, the default)
for zmin, bpsm, pers in ((2, 0, 0), (2, 0, 1), (2, 0, 2)):
    env = dict(os.environ, SEIS_ZCHUNK_MIN=str(zmin), SEIS_NO_PERSIST="0" if pers else "1",
               SEIS_ISO_RESIDENT="1" if pers == 2 else "0")
    if bpsm:
        env["SEIS_PERSIST_BPSM"] = str(bpsm)
    r = subprocess.run([sys.executable, "-c", ONE, ROOT], env=env, capture_output=True, text=True, timeout=600)
    out = r.stdout.strip().splitlines()[-1] if r.stdout.strip() else json.dumps({"error": r.stderr[-300:]})
    print(json.dumps({"zchunk_min": zmin, "persistent": pers, "blocks_per_sm": bpsm or "max", **json.loads(out)}),
          flush=True)
