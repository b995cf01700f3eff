"""Tile / ring-depth tuning sweep of the stencil kernels (not part of the product path).

    python tools/sweep.py build          # here: compile the variants into sweep_out/*.so
    python tools/sweep.py run            # on a B200 (gpurun): time every variant

Each variant is the same libseis source compiled with different -D macros
(SEIS_BY, SEIS_BYE and the TMA ring depths); the runner loads it through
SEIS_LIBPATH in a fresh process and reports the per-kernel CUDA-event times of
short ISO 512^3, acoustic C2 512^3 and elastic C3 384^3 runs.
"""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
OUT = os.path.join(ROOT, "sweep_out")
sys.path.insert(0, ROOT)

VARIANTS = {
    "base": [],
    "byv16": ["SEIS_BYV=16"],
    "byv16_vns2": ["SEIS_BYV=16", "SEIS_AC_VNS=2"],
    "byv12": ["SEIS_BYV=12"],
    "base2": [],
    "byv16b": ["SEIS_BYV=16"],
}
if os.environ.get("SWEEP_ONLY"):
    VARIANTS = {k: v for k, v in VARIANTS.items() if k in os.environ["SWEEP_ONLY"].split(",")}


def build():
    from paper_conf_ppopp_qawasmehchc15_b200 import build as b

    os.makedirs(OUT, exist_ok=True)
    for name, defs in VARIANTS.items():
        if defs is None:
            continue
        path = os.path.join(OUT, f"libseis_{name}.so")
        b.build(force=True, defines=defs, out=path)
        print("built", path)


def run():
    for name in VARIANTS:
        path = os.path.join(OUT, f"libseis_{name}.so")
        env = dict(os.environ, SEIS_LIBPATH=path)
        r = subprocess.run([sys.executable, os.path.join(ROOT, "tools", "sweep_one.py"), name],
                           env=env, capture_output=True, text=True, timeout=900)
        line = r.stdout.strip().splitlines()[-1] if r.stdout.strip() else json.dumps(
            {"variant": name, "error": r.stderr[-500:]})
        print(line, flush=True)


if __name__ == "__main__":
    {"build": build, "run": run}[sys.argv[1]]()
