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
    prof = seis.profile_read()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    m.forward_model(shot, out)
    e1.record()
    torch.cuda.synchronize()
    shot_ms = e0.elapsed_time(e1)
    res = {"n": n, "pml": a.pml, "ms_per_step": round(shot_ms / a.nt, 4),
           "gpts_s": round(float(n) ** 3 * a.nt / (shot_ms * 1e-3) / 1e9, 2)}
    if "iso2" in prof:  # the 2-step kernel (f1): 20 B per point per launch of two steps
        kp = prof["iso2"]
        t = kp[0] / kp[1]
        res.update({"iso2_ms": round(t, 4), "alg_B_per_pt": 20.0,
                    "frac": round(float(n) ** 3 * 20.0 / (t * 1e-3) / 1e9 / 6538.3, 4)})
    if "iso_step" in prof:
        kp = prof["iso_step"]
        t = kp[0] / kp[1]
        lay = 1.0 - ((n - 40) / n) ** 3
        bpp = 16.0 + (36.0 * lay if a.pml else 0.0)
        res.update({"iso_step_ms": round(t, 4), "alg_B_per_pt_step": round(bpp, 2),
                    "frac_step": round(float(n) ** 3 * bpp / (t * 1e-3) / 1e9 / 6538.3, 4)})
    res["seis"] = float(out.abs().sum().item())
    print(json.dumps(res))


if __name__ == "__main__":
    main()
