"""C5 on ONE B200 (BASELINE.json configs[4]): acoustic RTM 1024^3.

The driver's scaling run covers N > 1 (bench.py under torchrun); on a single GPU this tool
measures what C5 needs there:
  1. forward modeling 1024^3 (the strong-scaling propagation base, P = 1),
  2. one full checkpointed RTM shot 1024^3, nt = 1000, snap 20 (49 snapshots = 196 GiB do
     not fit in 180 GB: source-state checkpoints, f2), shots/hour,
  3. the z-slab decomposition path on one GPU (slabs = 8, halo copies between slabs) with
     the overlapped exchange and with the serial one (SEIS_NO_OVERLAP=1), against slabs = 1.
Prints one JSON line.  Timing: CUDA events on the launching stream after a warm-up.

    python tools/c5_bench.py [--n 1024] [--nt 1000] [--short 100] [--out gpurun_out/c5.json]
"""
import argparse
import json
import os
import sys
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_ppopp_qawasmehchc15_b200 as seis  # noqa: E402
from paper_conf_ppopp_qawasmehchc15_b200 import inputs  # noqa: E402


def timed(fn, stream, reps=1, warm=1):
    for _ in range(warm):
        fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    for _ in range(reps):
        fn()
    e1.record(stream)
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=1024)
    ap.add_argument("--nt", type=int, default=1000)
    ap.add_argument("--short", type=int, default=100, help="steps of the decomposition runs")
    ap.add_argument("--out", default=None)
    ap.add_argument("--no-24", action="store_true", help="skip the 24-bit-snapshot RTM run")
    a = ap.parse_args()
    dev = torch.device("cuda", 0)
    stream = torch.cuda.current_stream()
    res = {"workload": f"C5 acoustic RTM {a.n}^3 salt model, nt={a.nt}, snap 20, carpet step 8, 1 GPU"}
    t0 = time.time()
    wl = inputs.c5(n=a.n, nt=a.nt)
    res["model_build_s"] = round(time.time() - t0, 1)
    npts = float(wl.npts)
    g = seis.Grid(wl.nx, wl.ny, wl.nz, wl.h, wl.dt, nb=wl.nb, pml_f=wl.fp)
    shot = seis.Shot(wl.src, wl.wavelet, wl.rec, snap_period=wl.snap)

    # 1. forward modeling on the true model = the observed data of the RTM
    m = seis.Model(g, "acoustic", wl.model["vp"], rho=wl.model["rho"], device=0)
    data = torch.empty((wl.nt, shot.nrec), device=dev)
    ms = timed(lambda: m.forward_model(shot, data, stream), stream, reps=1, warm=1)
    res["forward"] = {"gpts_s": round(npts * wl.nt / (ms * 1e-3) / 1e9, 2), "ms_per_shot": round(ms, 1),
                      "receivers": shot.nrec}
    m.close()
    del m
    torch.cuda.empty_cache()

    # 2. checkpointed RTM on the smoothed model
    t0 = time.time()
    sm = inputs.smooth_torch(wl.model, 5.0, dev)
    res["smooth_s"] = round(time.time() - t0, 1)
    del wl.model
    free, total = torch.cuda.mem_get_info(dev)
    nsnap = (wl.nt - 1) // wl.snap
    need_all = seis.memory_required(g, "acoustic", shot)
    img_bytes = npts * 4 + data.numel() * 4

    def choose_c(bits):
        """0 if every snapshot fits, else the largest checkpoint segment length that fits."""
        if seis.memory_required(g, "acoustic", seis.Shot(wl.src, wl.wavelet, wl.rec, snap_period=wl.snap,
                                                         snap_bits=bits)) + img_bytes <= 0.95 * free:
            return 0
        fits = [cc for cc in range(1, nsnap + 1)
                if seis.memory_required(g, "acoustic", seis.Shot(wl.src, wl.wavelet, wl.rec, snap_period=wl.snap,
                                                                 ckpt_period=cc, snap_bits=bits)) + img_bytes
                <= 0.95 * free]
        if not fits:
            raise SystemExit("C5 RTM does not fit even with checkpointing")
        # fewest recomputed steps: every segment but the last is recomputed once, (nseg - 1) c
        return min(fits, key=lambda cc: ((nsnap + cc - 1) // cc - 1) * cc)

    def recomputed(c):
        if not c:
            return 0, 1
        nseg = (nsnap + c - 1) // c
        return sum(min((s + 1) * c, nsnap) * wl.snap - s * c * wl.snap for s in range(nseg - 1)), nseg

    c = choose_c(32)
    rshot = seis.Shot(wl.src, wl.wavelet, wl.rec, snap_period=wl.snap, ckpt_period=c)
    mig = seis.Model(g, "acoustic", sm["vp"], rho=sm["rho"], device=0)
    img = torch.zeros((wl.nz, wl.ny, wl.nx), device=dev)
    ms = timed(lambda: mig.migrate(rshot, data, img, stream), stream, reps=1, warm=1)
    recompute_steps, nseg = recomputed(c)
    res["rtm"] = {"shots_per_hour": round(3600.0 / (ms * 1e-3), 1), "ms_per_shot": round(ms, 1),
                  "gpts_s_both_phases": round(2 * npts * wl.nt / (ms * 1e-3) / 1e9, 2),
                  "gpts_s_all_steps": round(npts * (2 * wl.nt + recompute_steps) / (ms * 1e-3) / 1e9, 2),
                  "snapshots": nsnap, "ckpt_period": c, "segments": nseg, "recomputed_steps": recompute_steps,
                  "pool_bytes": int(seis.memory_required(g, "acoustic", rshot) - seis.memory_required(g, "acoustic")),
                  "all_snapshots_would_need_bytes": int(need_all), "free_bytes_before": int(free),
                  "image_norm": float(img.norm().item())}
    # 2b. 24-bit snapshots (seis_shot.snap_bits = 24, opt-in): 3/4 of the pool, so fewer (or no)
    # recomputed segments; bitwise decomposition-invariant, ~1e-5 from the fp32-snapshot image
    if not a.no_24:
        c24 = choose_c(24)
        sh24 = seis.Shot(wl.src, wl.wavelet, wl.rec, snap_period=wl.snap, ckpt_period=c24, snap_bits=24)
        img24 = torch.zeros_like(img)
        ms24 = timed(lambda: (img24.zero_(), mig.migrate(sh24, data, img24, stream)), stream, reps=1, warm=0)
        num = den = 0.0
        # (img holds the sum of 2a's warm-up and timed calls = 2 I exactly; img24 one call)
        for z0 in range(0, wl.nz, 64):  # slab-wise norms (no 4 GiB temporary)
            ref = 0.5 * img[z0:z0 + 64]
            num += float(torch.linalg.vector_norm(img24[z0:z0 + 64] - ref).item()) ** 2
            den += float(torch.linalg.vector_norm(ref).item()) ** 2
        r24, nseg24 = recomputed(c24)
        res["rtm_24bit_snapshots"] = {
            "shots_per_hour": round(3600.0 / (ms24 * 1e-3), 1), "ms_per_shot": round(ms24, 1),
            "gpts_s_both_phases": round(2 * npts * wl.nt / (ms24 * 1e-3) / 1e9, 2),
            "ckpt_period": c24, "segments": nseg24, "recomputed_steps": r24,
            "pool_bytes": int(seis.memory_required(g, "acoustic", sh24) - seis.memory_required(g, "acoustic")),
            "image_rel_l2_vs_fp32": round((num / den) ** 0.5, 7)}
        del img24
    mig.close()
    del mig, img
    torch.cuda.empty_cache()

    # 3. decomposition path on one GPU: slabs = 1 / 8 (overlapped) / 8 (serial)
    K = a.short
    w = wl.wavelet[:K]
    fshot = seis.Shot(wl.src, w, wl.rec)
    buf = torch.empty((K, fshot.nrec), device=dev)
    dec = {}
    for name, P, serial, copy in (("slabs1", 1, False, False), ("slabs8_overlap", 8, False, False),
                                  ("slabs8_serial", 8, True, False), ("slabs8_overlap_copy", 8, False, True),
                                  ("slabs8_serial_copy", 8, True, True)):
        # direct ghost stores (f4, default) vs the copy exchange (SEIS_GHOST_COPY=1)
        os.environ["SEIS_NO_OVERLAP"] = "1" if serial else "0"
        os.environ["SEIS_GHOST_COPY"] = "1" if copy else "0"
        gg = seis.Grid(g.nx, g.ny, g.nz, g.h, g.dt, nb=g.nb, pml_f=g.pml_f, slabs=P)
        mm = seis.Model(gg, "acoustic", sm["vp"], rho=sm["rho"], device=0)
        ms = timed(lambda: mm.forward_model(fshot, buf, stream), stream, reps=2, warm=1)
        dec[name] = {"gpts_s": round(npts * K / (ms * 1e-3) / 1e9, 2), "ms_per_step": round(ms / K, 3)}
        mm.close()
        del mm
        torch.cuda.empty_cache()
    os.environ.pop("SEIS_NO_OVERLAP", None)
    os.environ.pop("SEIS_GHOST_COPY", None)
    res["decomposition_1gpu"] = dec
    line = json.dumps(res)
    print(line)
    if a.out:
        with open(a.out, "w") as f:
            f.write(line + "\n")


if __name__ == "__main__":
    main()
