"""C2-size timing of the acoustic step paths on one B200: the split V / P pair vs the fused
persistent step (SEIS_AC_STEP=0 / 1), per-kernel CUDA-event times (library profiler) and
whole-shot time.  python tools/ac_step_bench.py [--n 512] [--nt 200]"""
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
    ap.add_argument("--n", type=int, default=512)
    ap.add_argument("--nt", type=int, default=200)
    ap.add_argument("--modes", default="0,1")
    ap.add_argument("--nb", type=int, default=20)
    a = ap.parse_args()
    wl = inputs.c2(n=a.n, nt=a.nt, nb=a.nb)
    stream = torch.cuda.current_stream()
    res = {"n": a.n, "nt": a.nt, "nb": a.nb}
    outs = {}
    for mode in a.modes.split(","):
        os.environ["SEIS_AC_STEP"] = mode
        g = seis.Grid(wl.nx, wl.ny, wl.nz, wl.h, wl.dt, nb=wl.nb, pml_f=wl.fp)
        m = seis.Model(g, "acoustic", wl.model["vp"], rho=wl.model["rho"])
        shot = seis.Shot(wl.src, wl.wavelet, wl.rec)
        out = torch.zeros((a.nt, shot.nrec), device="cuda:0")
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
        kp = {k: round(v[0] / v[1], 4) for k, v in seis.profile_read().items()}
        outs[mode] = out.clone()
        res[f"mode{mode}"] = {"ms_per_shot": round(ms, 2), "ms_per_step": round(ms / a.nt, 4),
                              "gpts_s": round(wl.npts * a.nt / (ms * 1e-3) / 1e9, 2), "kernel_ms": kp}
        m.close()
        del m
        torch.cuda.empty_cache()
    if len(outs) == 2:
        res["bitwise_equal"] = bool(torch.equal(outs["0"], outs["1"]))
    print(json.dumps(res))


if __name__ == "__main__":
    main()
