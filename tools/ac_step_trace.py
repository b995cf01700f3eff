"""Event timeline of the fused acoustic step (kernels_acoustic_step.cuh) on one B200: builds a
-DSEIS_AS_TRACE=1 copy of the library, runs a few C2-size steps and prints, for a few tiles,
per-plane latencies: V-load issue -> consumer V wait done, publish, P-load issue, P wait.
    python tools/ac_step_trace.py [--n 512] [--nt 3]"""
import argparse
import ctypes as C
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=512)
    ap.add_argument("--nt", type=int, default=3)
    ap.add_argument("--defines", default="")
    a = ap.parse_args()
    from paper_conf_ppopp_qawasmehchc15_b200 import build

    lib = build.build(force=True, defines=["SEIS_AS_TRACE=1"] + [d for d in a.defines.split(",") if d],
                      out="/tmp/libseis_trace.so")
    os.environ["SEIS_LIBPATH"] = lib
    os.environ["SEIS_AC_STEP"] = "1"
    import numpy as np
    import torch

    import paper_conf_ppopp_qawasmehchc15_b200 as seis
    from paper_conf_ppopp_qawasmehchc15_b200 import inputs

    seis._LIBPATH = lib  # (the package fixed its default path at import)

    wl = inputs.c2(n=a.n, nt=a.nt, nb=20)
    g = seis.Grid(wl.nx, wl.ny, wl.nz, wl.h, wl.dt, nb=wl.nb, pml_f=wl.fp)
    m = seis.Model(g, "acoustic", wl.model["vp"], rho=wl.model["rho"])
    shot = seis.Shot(wl.src, wl.wavelet, wl.rec)
    out = torch.zeros((a.nt, shot.nrec), device="cuda:0")
    os.environ["SEIS_NO_GRAPH"] = "1"
    m.forward_model(shot, out)
    L = seis.lib()
    L.seis_debug_trace.restype = C.c_void_p
    L.seis_debug_trace.argtypes = [C.POINTER(C.c_uint64)]
    n = C.c_uint64()
    p = L.seis_debug_trace(C.byref(n))
    buf = np.ctypeslib.as_array((C.c_uint64 * n.value).from_address(p)).copy()
    nz = wl.nz
    ntiles = n.value // (nz * 48)
    t = buf.reshape(ntiles, nz, 48).astype(np.float64)
    t0 = t[t > 0].min()
    t = np.where(t > 0, t - t0, np.nan) / 1000.0  # us
    names = ["vload", "publish", "pload", "p_ready", "v_ready", "v_done", "p_start", "v_done_lastwarp"]
    res = {"tiles": ntiles, "nz": nz, "kernel_us": float(np.nanmax(t))}
    mid = slice(40, nz - 40)
    for tile in (0, ntiles // 2 + 3, ntiles - 1):
        T = t[tile, mid]
        res[f"tile{tile}"] = {
            "us_per_plane": float(np.nanmean(np.diff(T[:, 5]))),
            "vload_to_vready": float(np.nanmedian(T[:, 4] - T[:, 0])),
            "vdone_to_publish": float(np.nanmedian(T[:, 1] - T[:, 7])),
            "publish_to_pload": float(np.nanmedian(T[:, 2] - T[:, 1])),
            "pload_to_pready": float(np.nanmedian(T[:, 3] - T[:, 2])),
            "p_wait": float(np.nanmedian(T[:, 3] - T[:, 6])),
            "iter_pwait": float(np.nanmedian(t[tile, 40:nz - 44, 3] - t[tile, 40:nz - 44, 6])),
            "iter_pcompute_plus_vwait": float(np.nanmedian(t[tile, 44:nz - 40, 4] - t[tile, 40:nz - 44, 3])),
            "iter_vcompute": float(np.nanmedian(t[tile, 44:nz - 40, 5] - t[tile, 44:nz - 40, 4])),
            "iter_tail": float(np.nanmedian(t[tile, 41:nz - 43, 6] - t[tile, 44:nz - 40, 5])),
            "vready_to_vdone": float(np.nanmedian(T[:, 5] - T[:, 4])),
            "warp_skew_vdone": float(np.nanmedian(T[:, 7] - T[:, 5])),
            "lastwarp_vdone_to_emptyv_seen": float(np.nanmedian(T[:, 8] - T[:, 7])),
            "fence_proxy": float(np.nanmedian(T[:, 9] - T[:, 8])),
            "red_release": float(np.nanmedian(T[:, 1] - T[:, 9])),
            "publish_to_pslot_free": float(np.nanmedian(T[:, 10] - T[:, 1])),
            "pslot_to_neighbours_ok": float(np.nanmedian(T[:, 11] - T[:, 10])),
            "neighbours_ok_to_pload": float(np.nanmedian(T[:, 2] - T[:, 11])),
        }
    # per-tile busy / wait breakdown over the middle planes (consumer warp 0)
    lo, hi = 40, nz - 44
    pw = np.nanmean(t[:, lo:hi, 3] - t[:, lo:hi, 6], axis=1)                # P-stage wait
    vc = np.nanmean(t[:, lo + 4:hi + 4, 5] - t[:, lo + 4:hi + 4, 4], axis=1)  # V wait-done -> V done
    per = (t[:, hi, 1] - t[:, lo, 1]) / (hi - lo)                           # publish period
    order = np.argsort(pw)
    res["p_wait_least_tiles"] = [(int(i), round(float(pw[i]), 2), round(float(vc[i]), 2)) for i in order[:8]]
    res["p_wait_most_tiles"] = [(int(i), round(float(pw[i]), 2), round(float(vc[i]), 2)) for i in order[-5:]]
    res["publish_period_us"] = [round(float(np.nanmin(per)), 3), round(float(np.nanmedian(per)), 3),
                                round(float(np.nanmax(per)), 3)]
    res["p_wait_grid"] = [[round(float(pw[r * 4 + c]), 1) for c in range(4)] for r in range(ntiles // 4)]
    # per-warp V start / done relative to the tile's earliest warp, middle planes, median
    for tile in (0, 1, 77):
        vs = t[tile, lo:hi, 32:46]
        vd = t[tile, lo:hi, 16:30]
        res[f"warps_tile{tile}_vstart_rel"] = [round(float(x), 2) for x in np.nanmedian(vs - np.nanmin(vs, axis=1, keepdims=True), axis=0)]
        res[f"warps_tile{tile}_vdur"] = [round(float(x), 2) for x in np.nanmedian(vd - vs, axis=0)]
    # lateness of the P-load relative to the time the consumers need it
    k = np.arange(nz)
    res["pload_minus_pstart_median"] = float(np.nanmedian(t[:, mid, 2] - t[:, mid, 6]))
    print(json.dumps(res, indent=1))


if __name__ == "__main__":
    main()
