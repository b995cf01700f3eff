#!/usr/bin/env python
"""Benchmark of the seismic modeling / RTM hot path (driver contract: one JSON line).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl reference] [--no-extras]

Headline (BASELINE.json configs[1], "C2"): acoustic 3D, 512^3 layered model,
2000 time steps, C-PML (nb = 20) on 6 faces, 472-receiver surface line, one
Ricker shot.  One bench "step" = one seismic-modeling shot (seis_forward_model:
every time step's V and P kernels (source injection fused into P) and the receiver gather).  metric =
Gpts/s = grid points x time steps / second (whole job over all ranks).

* value:  device-timed (CUDA events on the launching stream, barrier + synchronize on
          both sides, max over ranks), inputs resident in HBM, seismogram to a device buffer.
* e2e:    the same shots through the C ABI with HOST buffers (pinned): the wavelet and
          receiver table are copied in and the seismogram copied out inside the timed region.
* roofline: dominant kernel's algorithmic bytes per launch / its average CUDA-event launch
          time (library event pairs on the launching stream, recorded over the timed region),
          against MEASURED_PEAKS.json hbm_gbs.
* cpu_baseline: the fp64 oracle (oracle/, test infrastructure) timed on the host cores on a
          bounded sample of the same workload (2 time steps of the full 512^3 grid).
* extras (N = 1, unless --no-extras): Gpts/s of the other propagators (C1 ISO 64^3, an ISO 512^3
          sweep, C3 elastic 384^3) and RTM shots/hour (C4, 512^3 salt model, 2000 steps,
          snapshots every 20 steps in HBM).
N > 1 (torchrun): weak scaling, z-slab decomposition with NCCL halo exchange; each rank
holds 512^3 points (global nz = 512 N).  --scaling strong splits one 512^3 grid instead;
--halo peer replaces the NCCL send/recv by direct ghost-plane stores over NVLink (f4).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "Gpts/s per propagator and RTM shots/hour; % of B200 HBM roofline at 1/2/4/8"

# algorithmic bytes per grid point per launch: each state field read once and
# written once, model coefficients read once, C-PML memory variables RMW only inside layers
ALG_BYTES = {"iso_step": 16.0, "ac_v": 32.0, "ac_p": 24.0, "el_v": 52.0, "el_s": 68.0}
PSI_AXES = {"ac_v": 3, "ac_p": 3, "el_v": 9, "el_s": 9}


def peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            p = json.load(f)
        return float(p["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


class Clocks:
    """nvidia-smi sampling of SM clocks and throttle reasons DURING the timed region."""

    FIELDS = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,"
              "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
              "clocks_event_reasons.sw_power_cap")

    def __init__(self, device):
        self.device = device
        self.samples = []
        self.proc = None

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.device), f"--query-gpu={self.FIELDS}",
                 "--format=csv,noheader,nounits", "-lms", "200"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.samples.append([x.strip() for x in line.split(",")])

    def __exit__(self, *a):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(2)
            except Exception:
                self.proc.kill()

    def summary(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        sm = [float(s[0]) for s in self.samples if s[0].replace(".", "").isdigit()]
        mx = [float(s[1]) for s in self.samples if s[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for s in self.samples for i in range(4)
                          if len(s) > 2 + i and s[2 + i].lower() == "active"})
        load = [x for x in sm if x > 0.5 * max(sm)] if sm else []
        return {"sm_mhz": statistics.median(load) if load else None,
                "sm_max_mhz": max(mx) if mx else None, "reasons": reasons,
                "samples": len(self.samples)}


def dist_env():
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return ws, rank, local


# ---------------------------------------------------------------- workloads
def c2_workload(n=512, nt=2000, nz=None):
    from paper_conf_ppopp_qawasmehchc15_b200 import inputs

    wl = inputs.c2(n=n, nt=nt, nb=20)
    if nz is not None and nz != n:
        wl.model = inputs.layered_acoustic(n, n, nz, scale=n / 512.0)
        wl.nz = nz
    return wl


def c2_config(wl, nz, nt, nrec, ws, args):
    """The `config` both arms report (the reference arm times a bounded sample of it)."""
    return {"workload": f"C2 acoustic {wl.nx}x{wl.ny}x{nz} layered, {nt} steps, C-PML nb={wl.nb}, "
                        f"{nrec}-receiver line, 1 shot per step",
            "grid": [wl.nx, wl.ny, nz], "nt": nt, "dt": wl.dt, "h": wl.h,
            "parallelism": f"z-slab x{ws}" if ws > 1 else "single GPU",
            "scaling": args.scaling if ws > 1 else None,
            "halo": (args.halo if ws > 1 else None),
            "l2": "inputs larger than L2 (each 512^3 field is 512 MiB > 126 MB)"}


def psi_bytes_per_point(nx, ny, nz, nb, axes_per_dir, free_surface=False):
    """C-PML memory-variable RMW bytes per grid point (8 B per point inside a layer, per axis;
    a free-surface top has no layer)."""
    if nb == 0:
        return 0.0
    W = nb + 1
    frac = [min(1.0, 2 * W / nx), min(1.0, 2 * W / ny), min(1.0, (W if free_surface else 2 * W) / nz)]
    return 8.0 * sum(frac) * axes_per_dir / 3.0


# ---------------------------------------------------------------- product arm
def run_product(args):
    import torch
    import torch.distributed as dist

    import paper_conf_ppopp_qawasmehchc15_b200 as seis

    ws, rank, local = dist_env()
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    comm = None
    if ws > 1:
        dist.init_process_group("nccl", device_id=dev)
        comm = seis.Comm.from_torch_distributed(local)
    n, nt = args.n, args.nt
    # weak scaling (default): each rank holds n^3 points; strong: the n^3 grid is split
    nz = n if args.scaling == "strong" else n * ws
    wl = c2_workload(n=n, nt=nt, nz=nz)
    z0, nzl = seis.slab_bounds(nz, ws, rank)
    grid = seis.Grid(wl.nx, wl.ny, nz, wl.h, wl.dt, nb=wl.nb, pml_R=wl.pml_R, pml_f=wl.fp)
    model = seis.Model(grid, "acoustic", wl.model["vp"][z0:z0 + nzl], rho=wl.model["rho"][z0:z0 + nzl],
                       comm=comm, device=local)
    if ws > 1 and args.halo == "peer":
        model.enable_peer_halo()  # f4: rank faces by direct NVLink ghost stores (CUDA IPC)
    shot = seis.Shot(wl.src, wl.wavelet, wl.rec)
    seis_dev = torch.empty((nt, shot.nrec), dtype=torch.float32, device=dev)
    stream = torch.cuda.current_stream()

    def barrier():
        if ws > 1:
            dist.barrier()
        torch.cuda.synchronize()

    for _ in range(args.warmup):
        model.forward_model(shot, seis_dev, stream)
    barrier()
    launches = 0
    seis.profile(True)
    with Clocks(local) as clk:
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for _ in range(args.steps):
            model.forward_model(shot, seis_dev, stream)
            launches += seis.Model.launches()
        e1.record(stream)
        barrier()
    seis.profile(False)
    ms = e0.elapsed_time(e1)
    kprof = seis.profile_read()
    if ws > 1:
        t = torch.tensor([ms], device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t.item())
    pts = float(wl.nx) * wl.ny * nz  # all ranks
    value = pts * nt * args.steps / (ms * 1e-3) / 1e9

    # e2e: HOST buffers through the C ABI (pinned seismogram; wavelet + receivers are host)
    host_seis = torch.empty((nt, shot.nrec), dtype=torch.float32).pin_memory()
    model.forward_model(shot, host_seis.numpy(), stream)
    barrier()
    t0 = time.perf_counter()
    f0, f1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    f0.record(stream)
    for _ in range(args.steps):
        model.forward_model(shot, host_seis.numpy(), stream)
    f1.record(stream)
    barrier()
    e2e_ms = max(f0.elapsed_time(f1), (time.perf_counter() - t0) * 1e3)
    if ws > 1:
        t = torch.tensor([e2e_ms], device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        e2e_ms = float(t.item())
    e2e = {"value": round(pts * nt * args.steps / (e2e_ms * 1e-3) / 1e9, 3), "unit": "Gpts/s",
           "h2d_bytes_per_step": int(shot.nt * 4 + shot.nrec * 12),
           "d2h_bytes_per_step": int(shot.nt * shot.nrec * 4)}

    # roofline of the dominant kernel
    hbm, peak_src = peaks()
    dom = max(("ac_v", "ac_p"), key=lambda k: kprof.get(k, (0, 1))[0])
    kms, kn = kprof[dom]
    local_pts = float(wl.nx) * wl.ny * nzl
    bpp = ALG_BYTES[dom] + psi_bytes_per_point(wl.nx, wl.ny, nz, wl.nb, PSI_AXES[dom])
    achieved = local_pts * bpp / (kms / kn * 1e-3) / 1e9
    traffic = None  # DRAM bytes per launch from the committed ncu capture (same kernel, same size)
    try:
        with open(os.path.join(ROOT, "profiles", "traffic.json")) as f:
            tr = json.load(f).get(f"C2_{n}_{dom}")
            if tr and ws == 1:
                traffic = int(tr)
    except Exception:
        pass
    roof = {"bound": "hbm", "kernel": dom, "achieved": round(achieved, 1), "peak": hbm,
            "peak_source": peak_src, "unit": "GB/s", "frac": round(achieved / hbm, 4),
            "traffic": traffic, "traffic_unit": "DRAM bytes per launch (ncu, profiles/traffic.json)",
            "alg_bytes_per_launch": round(local_pts * bpp),
            "traffic_over_alg": round(traffic / (local_pts * bpp), 3) if traffic else None,
            "alg_bytes_per_point": round(bpp, 2),
            "kernel_ms_avg": round(kms / kn, 4),
            "kernels": {k: {"ms_avg": round(v[0] / v[1], 4), "launches": v[1],
                            "share": round(v[0] / sum(x[0] for x in kprof.values()), 4)}
                        for k, v in kprof.items()}}

    out = {"metric": METRIC, "value": round(value, 3), "unit": "Gpts/s", "n_gpus": ws,
           "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(ms / args.steps, 3),
           "higher_is_better": True, "scaling": args.scaling, "vs_baseline": None, "dtype": "f32",
           "data": "synthetic (seeded layered model, Ricker source)",
           "config": c2_config(wl, nz, nt, shot.nrec, ws, args),
           "e2e": e2e, "gpu_launches": launches, "roofline": roof}
    if rank == 0:
        out["clocks"] = clk.summary()
    model.close()
    del model
    torch.cuda.empty_cache()
    if rank == 0 and ws == 1:
        if not args.no_extras:
            out["extras"] = run_extras(args, local)
        out["cpu_baseline"] = cpu_baseline(args)
    if ws > 1:
        dist.destroy_process_group()
    if rank == 0:
        print(json.dumps(out))


def _timed_shots(fn, reps, stream):
    import torch

    fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    for _ in range(reps):
        fn()
    e1.record(stream)
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps


def run_extras(args, local):
    """Other propagators + RTM on one GPU (fewer repetitions; each line is its own workload)."""
    import torch

    import paper_conf_ppopp_qawasmehchc15_b200 as seis
    from paper_conf_ppopp_qawasmehchc15_b200 import inputs

    stream = torch.cuda.current_stream()
    dev = torch.device("cuda", local)
    res = {}
    hbm, _ = peaks()

    def kernel_frac(name, npts, bpp):
        kp = seis.profile_read().get(name)
        if not kp:
            return None
        gbs = npts * bpp / (kp[0] / kp[1] * 1e-3) / 1e9
        return {"kernel": name, "achieved_GBs": round(gbs, 1), "frac": round(gbs / hbm, 4),
                "ms_avg": round(kp[0] / kp[1], 4)}

    # C1: ISO 64^3, 200 steps (L2-resident: Gpts/s only)
    wl = inputs.c1()
    g = seis.Grid(wl.nx, wl.ny, wl.nz, wl.h, wl.dt, nb=wl.nb)
    m = seis.Model(g, "iso", wl.model["vp"], device=local)
    shot = seis.Shot(wl.src, wl.wavelet, wl.rec)
    buf = torch.empty((wl.nt, shot.nrec), device=dev)
    ms = _timed_shots(lambda: m.forward_model(shot, buf, stream), 5, stream)
    res["C1_iso_64"] = {"gpts_s": round(wl.npts * wl.nt / (ms * 1e-3) / 1e9, 3), "ms_per_shot": round(ms, 3),
                        "note": "4 MB working set, L2-resident; launch-bound"}
    m.close()
    # ISO 512^3 sweep (the iso kernel at HBM scale), 200 steps, nb = 20
    n = args.n
    vp = np.full((n, n, n), 2000.0, np.float32)
    vp[n // 3:] = 3000.0
    g = seis.Grid(n, n, n, 10.0, 1e-3, nb=20)
    m = seis.Model(g, "iso", vp, device=local)
    w = inputs.source_series("iso", 200, 1e-3, 15.0)
    shot = seis.Shot((n // 2, n // 2, 24), w, np.asarray([[n // 2, n // 2, 24]], np.int32))
    buf = torch.empty((200, 1), device=dev)
    m.forward_model(shot, buf, stream)
    seis.profile(True)
    ms = _timed_shots(lambda: m.forward_model(shot, buf, stream), 2, stream)
    seis.profile(False)
    res["iso_512"] = {"gpts_s": round(n ** 3 * 200 / (ms * 1e-3) / 1e9, 3), "ms_per_shot": round(ms, 3),
                      "roofline": kernel_frac("iso_step", float(n) ** 3, 16.0)}
    m.close()
    # the same with the split-field PML (O6b): layer points also read u^(d) at two levels and
    # write the new level (36 B per layer point)
    g = seis.Grid(n, n, n, 10.0, 1e-3, nb=20, iso_pml=1)
    m = seis.Model(g, "iso", vp, device=local)
    m.forward_model(shot, buf, stream)
    seis.profile(True)
    ms = _timed_shots(lambda: m.forward_model(shot, buf, stream), 2, stream)
    seis.profile(False)
    lay = 1.0 - ((n - 40) / n) ** 3
    res["iso_512_split_pml"] = {"gpts_s": round(n ** 3 * 200 / (ms * 1e-3) / 1e9, 3), "ms_per_shot": round(ms, 3),
                                "alg_bytes_per_point": round(16.0 + 36.0 * lay, 2),
                                "roofline": kernel_frac("iso_step", float(n) ** 3, 16.0 + 36.0 * lay)}
    m.close()
    del vp
    torch.cuda.empty_cache()
    # C3: elastic 384^3, 1500 steps, free surface, C-PML on 5 faces
    wl = inputs.c3()
    g = seis.Grid(wl.nx, wl.ny, wl.nz, wl.h, wl.dt, nb=wl.nb, free_surface=1, pml_f=wl.fp)
    m = seis.Model(g, "elastic", wl.model["vp"], vs=wl.model["vs"], rho=wl.model["rho"], device=local)
    shot = seis.Shot(wl.src, wl.wavelet, wl.rec, rec_component=2)
    buf = torch.empty((wl.nt, shot.nrec), device=dev)
    seis.profile(True)
    ms = _timed_shots(lambda: m.forward_model(shot, buf, stream), 1, stream)
    seis.profile(False)
    psi_el = psi_bytes_per_point(wl.nx, wl.ny, wl.nz, wl.nb, PSI_AXES["el_v"], free_surface=True)
    res["C3_elastic_384"] = {"gpts_s": round(wl.npts * wl.nt / (ms * 1e-3) / 1e9, 3),
                             "ms_per_shot": round(ms, 3),
                             "alg_bytes_per_point": {"el_v": round(52.0 + psi_el, 2), "el_s": round(68.0 + psi_el, 2)},
                             "roofline_v": kernel_frac("el_v", float(wl.npts), 52.0 + psi_el),
                             "roofline_s": kernel_frac("el_s", float(wl.npts), 68.0 + psi_el)}
    m.close()
    torch.cuda.empty_cache()
    # C4: RTM 512^3 salt model: observed data on the true model, migration on the smoothed one
    wl = inputs.c4(n=args.n)
    g = seis.Grid(wl.nx, wl.ny, wl.nz, wl.h, wl.dt, nb=wl.nb, pml_f=wl.fp)
    true = seis.Model(g, "acoustic", wl.model["vp"], rho=wl.model["rho"], device=local)
    shot = seis.Shot(wl.src, wl.wavelet, wl.rec, snap_period=wl.snap)
    data = torch.empty((wl.nt, shot.nrec), device=dev)
    true.forward_model(shot, data, stream)
    true.close()
    torch.cuda.empty_cache()
    smooth = inputs.smooth(wl.model, 5.0)
    mig = seis.Model(g, "acoustic", smooth["vp"], rho=smooth["rho"], device=local)
    img = torch.zeros((wl.nz, wl.ny, wl.nx), device=dev)
    ms = _timed_shots(lambda: mig.migrate(shot, data, img, stream), 1, stream)
    res["C4_rtm_512"] = {"shots_per_hour": round(3600.0 / (ms * 1e-3), 1), "ms_per_shot": round(ms, 1),
                         "gpts_s_both_phases": round(2 * wl.npts * wl.nt / (ms * 1e-3) / 1e9, 3),
                         "snapshots_in_hbm": (wl.nt - 1) // wl.snap, "receivers": shot.nrec}
    mig.close()
    return res


# ---------------------------------------------------------------- oracle arm
def cpu_baseline(args, steps=2):
    """The fp64 oracle (as it stands) on the host cores: `steps` time steps of the full C2 grid."""
    import oracle

    n = args.n
    wl = c2_workload(n=n, nt=args.nt)
    g = oracle.Grid(wl.nx, wl.ny, wl.nz, wl.h, wl.dt, nb=wl.nb, pml_R=wl.pml_R, pml_f=wl.fp)
    st = oracle.ac_state(g)
    t0 = time.perf_counter()
    oracle.ac_run(g, wl.model["vp"], wl.model["rho"], st, 0, steps, [wl.src], wl.wavelet[:, None],
                  wl.rec)
    dt = time.perf_counter() - t0
    cores = int(os.environ.get("OMP_NUM_THREADS", os.cpu_count() or 1))
    return {"value": round(wl.npts * steps / dt / 1e9, 5), "unit": "Gpts/s", "cores": cores,
            "kind": "oracle",
            "sample": f"{steps} time steps of the C2 {n}^3 acoustic shot on the full grid "
                      f"(oracle.ac_run, fp64, OpenMP), {dt:.1f} s"}


def run_reference(args):
    ws, rank, local = dist_env()
    if rank != 0:
        return
    import oracle

    n = args.n
    wl = c2_workload(n=n, nt=args.nt)
    g = oracle.Grid(wl.nx, wl.ny, wl.nz, wl.h, wl.dt, nb=wl.nb, pml_R=wl.pml_R, pml_f=wl.fp)
    st = oracle.ac_state(g)
    per = args.ref_steps
    for _ in range(args.warmup):
        oracle.ac_run(g, wl.model["vp"], wl.model["rho"], st, 0, 1, [wl.src], wl.wavelet[:, None], wl.rec)
    t0 = time.perf_counter()
    for s in range(args.steps):
        oracle.ac_run(g, wl.model["vp"], wl.model["rho"], st, s * per, per, [wl.src], wl.wavelet[:, None],
                      wl.rec)
    dt = time.perf_counter() - t0
    value = wl.npts * per * args.steps / dt / 1e9
    cores = int(os.environ.get("OMP_NUM_THREADS", os.cpu_count() or 1))
    sample = (f"each step = {per} time steps of the C2 {n}^3 acoustic shot on the full grid "
              f"(oracle.ac_run, fp64)")
    print(json.dumps({
        "impl": "reference", "metric": METRIC, "value": round(value, 5), "unit": "Gpts/s", "n_gpus": ws,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(dt / args.steps * 1e3, 1),
        "higher_is_better": True, "scaling": args.scaling, "vs_baseline": None, "dtype": "f64",
        "data": "synthetic (seeded layered model, Ricker source)",
        "config": c2_config(wl, n * ws if args.scaling == "weak" else n, args.nt, wl.rec.shape[0], ws, args),
        "cpu_baseline": {"value": round(value, 5), "unit": "Gpts/s", "cores": cores, "kind": "oracle",
                         "sample": sample},
        "e2e": {"value": round(value, 5), "unit": "Gpts/s", "h2d_bytes_per_step": 0,
                "d2h_bytes_per_step": 0}}))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="product", choices=["product", "reference"])
    ap.add_argument("--n", type=int, default=512, help="grid edge (512 = the C2 config)")
    ap.add_argument("--nt", type=int, default=2000, help="time steps per shot (2000 = C2)")
    ap.add_argument("--ref-steps", type=int, default=1, help="oracle time steps per reference step")
    ap.add_argument("--no-extras", action="store_true")
    ap.add_argument("--scaling", default="weak", choices=["weak", "strong"],
                    help="N>1: weak = n^3 per rank (default), strong = one n^3 grid split in z-slabs")
    ap.add_argument("--halo", default="nccl", choices=["nccl", "peer"],
                    help="N>1 rank-face ghost exchange: NCCL send/recv overlapped with the interior "
                         "(default) or direct peer stores from the kernels (f4)")
    args = ap.parse_args()
    if args.warmup < 3:
        print("warning: --warmup < 3 violates the timing rules", file=sys.stderr)
    if args.impl == "reference":
        run_reference(args)
    else:
        run_product(args)


if __name__ == "__main__":
    main()
