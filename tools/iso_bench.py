"""ISO 512^3 timing (the bench's iso_512 / iso_512_split_pml extras) with per-kernel CUDA-event
times: python tools/iso_bench.py [--n 512] [--nt 100] [--pml 0|1].  SEIS_LIBPATH selects a build."""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ppopp_qawasmehchc15_b200 as seis  # noqa: E402
from paper_conf_ppopp_qawasmehchc15_b200 import inputs  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=512)
    ap.add_argument("--nt", type=int, default=100)
    ap.add_argument("--pml", type=int, default=1)
    a = ap.parse_args()
    n = a.n
    vp = np.full((n, n, n), 2000.0, np.float32)
    vp[n // 3:] = 3000.0
    g = seis.Grid(n, n, n, 10.0, 1e-3, nb=20, iso_pml=a.pml)
    m = seis.Model(g, "iso", vp)
    w = inputs.source_series("iso", a.nt, 1e-3, 15.0)
    shot = seis.Shot((n // 2, n // 2, 24), w, np.asarray([[n // 2, n // 2, 24]], np.int32))
    out = torch.zeros((a.nt, 1), device="cuda:0")
    m.forward_model(shot, out)
    seis.profile(True)
    m.forward_model(shot, out)
    torch.cuda.synchronize()
    seis.profile(False)
    kp = seis.profile_read()["iso_step"]
    t = kp[0] / kp[1]
    lay = 1.0 - ((n - 40) / n) ** 3
    bpp = 16.0 + (36.0 * lay if a.pml else 0.0)
    print(json.dumps({"n": n, "pml": a.pml, "iso_step_ms": round(t, 4), "alg_B_per_pt": round(bpp, 2),
                      "frac": round(float(n) ** 3 * bpp / (t * 1e-3) / 1e9 / 6538.3, 4),
                      "seis": float(out.abs().sum().item())}))


if __name__ == "__main__":
    main()
