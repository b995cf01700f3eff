"""Acoustic-step variant sweep: the split pair's z-chunking vs the fused persistent step (f1).

    python tools/sweep_ac.py build      # here: compile the variants into sweep_out/
    python tools/sweep_ac.py run        # on a B200: C2 512^3, 60 steps, per-kernel CUDA-event ms
"""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
OUT = os.path.join(ROOT, "sweep_out")
sys.path.insert(0, ROOT)

VARIANTS = {  # name: (defines, env)
    "split": ([], {"SEIS_AC_STEP": "0"}),
    "step": ([], {"SEIS_AC_STEP": "1"}),
    "step_pf8": (["SEIS_AS_PF=8"], {"SEIS_AC_STEP": "1"}),
    "split_z128": ([], {"SEIS_AC_STEP": "0", "SEIS_ZCHUNK_MAX": "128"}),
    "split_z64": ([], {"SEIS_AC_STEP": "0", "SEIS_ZCHUNK_MAX": "64"}),
    "split_z32": ([], {"SEIS_AC_STEP": "0", "SEIS_ZCHUNK_MAX": "32"}),
}
if os.environ.get("SWEEP_ONLY"):
    VARIANTS = {k: v for k, v in VARIANTS.items() if k in os.environ["SWEEP_ONLY"].split(",")}

ONE = r'''
import json, os, sys, numpy as np, torch
sys.path.insert(0, sys.argv[2])
import paper_conf_ppopp_qawasmehchc15_b200 as seis
from paper_conf_ppopp_qawasmehchc15_b200 import inputs
n = int(os.environ.get("SWEEP_N", "512"))
wl = inputs.c2(n=n, nt=60)
m = seis.Model(seis.Grid(wl.nx, wl.ny, wl.nz, wl.h, wl.dt, nb=wl.nb, pml_f=wl.fp), "acoustic",
               wl.model["vp"], rho=wl.model["rho"])
shot = seis.Shot(wl.src, wl.wavelet, wl.rec)
buf = torch.empty((shot.nt, shot.nrec), device="cuda")
m.forward_model(shot, buf); torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(3): m.forward_model(shot, buf)
e1.record(); torch.cuda.synchronize()
ms_step = e0.elapsed_time(e1) / (3 * shot.nt)
seis.profile(True)
m.forward_model(shot, buf); torch.cuda.synchronize()
seis.profile(False)
prof = {k: round(v[0] / v[1], 4) for k, v in seis.profile_read().items()}
print(json.dumps({"variant": sys.argv[1], "n": n, "ms_per_step": round(ms_step, 4),
                  "gpts_s": round(n ** 3 / (ms_step * 1e-3) / 1e9, 2), "kernels_ms": prof}))
'''


def build():
    from paper_conf_ppopp_qawasmehchc15_b200 import build as b

    os.makedirs(OUT, exist_ok=True)
    for name, (defs, _) in VARIANTS.items():
        path = os.path.join(OUT, f"libseis_ac_{name}.so")
        b.build(force=True, defines=defs, out=path)
        print("built", path)


def run():
    for name, (_, env) in VARIANTS.items():
        path = os.path.join(OUT, f"libseis_ac_{name}.so")
        e = dict(os.environ, SEIS_LIBPATH=path, **env)
        r = subprocess.run([sys.executable, "-c", ONE, name, ROOT], env=e, capture_output=True, text=True,
                           timeout=600)
        line = r.stdout.strip().splitlines()[-1] if r.stdout.strip() else json.dumps(
            {"variant": name, "error": r.stderr[-800:]})
        print(line, flush=True)


if __name__ == "__main__":
    {"build": build, "run": run}[sys.argv[1]]()
