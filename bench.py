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
* e2e:    the same shots through the C ABI with HOST buffers: every call copies the wavelet
          (host [nt] fp32) to the device and the seismogram (pinned host [nt][nrec]) back,
          inside the timed region; the receiver table is re-uploaded only when the geometry
          changes (here: never after the first call, so its bytes are not counted).
* roofline: dominant kernel's algorithmic bytes per launch / its average CUDA-event launch
          time (library event pairs on the launching stream, recorded over the timed region),
          against MEASURED_PEAKS.json hbm_gbs.
* cpu_baseline: the fp64 oracle (oracle/, test infrastructure) timed on the host cores
          (child process, OMP_PROC_BIND=close, all cores) on a bounded sample of the same
          workload: 1 untimed + 5 timed time steps of the full 512^3 grid; C1 and C3 oracle
          timings ride along under other_configs.
* extras (N = 1, unless --no-extras): Gpts/s of the other propagators (C1 ISO 64^3, an ISO 512^3
          sweep, C3 elastic 384^3) and RTM shots/hour (C4, 512^3 salt model, 2000 steps,
          snapshots every 20 steps in HBM; C5, 1024^3, 1000 steps, checkpointed, --no-c5 skips).
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
# graph-sampled profiling: event nodes around the launches of every PROF_SAMPLE-th time step
# inside the production shot graph (seis.h seis_profile)
PROF_SAMPLE = 20
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
def c2_workload(n=512, nt=2000, nz=None, z0=0, nzl=None):
    """The C2 workload on an n x n x nz grid (nz = n: the BASELINE config); with z0 / nzl only
    that z-slab of the model is generated (each rank builds its own slab: host memory per rank
    is bounded by the slab, not the global grid)."""
    from paper_conf_ppopp_qawasmehchc15_b200 import inputs

    nz = n if nz is None else nz
    nzl = nz - z0 if nzl is None else nzl
    wl = inputs.c2(n=n, nt=nt, nb=20, model=False)
    wl.model = inputs.layered_acoustic(n, n, nz, scale=n / 512.0, z0=z0, nzl=nzl)
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
    z0, nzl = seis.slab_bounds(nz, ws, rank)
    wl = c2_workload(n=n, nt=nt, nz=nz, z0=z0, nzl=nzl)  # this rank's slab only
    grid = seis.Grid(wl.nx, wl.ny, nz, wl.h, wl.dt, nb=wl.nb, pml_R=wl.pml_R, pml_f=wl.fp)
    model = seis.Model(grid, "acoustic", wl.model["vp"], rho=wl.model["rho"], comm=comm, device=local)
    del wl.model
    if ws > 1 and args.halo == "peer":
        model.enable_peer_halo()  # f4: rank faces by direct NVLink ghost stores (CUDA IPC)
    shot = seis.Shot(wl.src, wl.wavelet, wl.rec)
    seis_dev = torch.empty((nt, shot.nrec), dtype=torch.float32, device=dev)
    stream = torch.cuda.current_stream()

    def barrier():
        if ws > 1:
            dist.barrier()
        torch.cuda.synchronize()

    # per-kernel times from event nodes inside the production shot graph (every PROF_SAMPLE-th
    # time step), so the timed region is the graph replay a user runs; the warm-up captures it
    seis.profile(True, sample=PROF_SAMPLE)
    for _ in range(args.warmup):
        model.forward_model(shot, seis_dev, stream)
    barrier()
    launches = 0
    seis.profile(True, sample=PROF_SAMPLE)  # (same mode: zero the counters, keep the graph)
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

    # e2e: HOST buffers through the C ABI (the wavelet is uploaded and the pinned seismogram
    # read back by every call)
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
           "h2d_bytes_per_step": int(shot.nt * 4),  # the wavelet (receivers cached by geometry)
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
            "timing": f"CUDA event nodes inside the replayed shot graph around every {PROF_SAMPLE}th "
                      "time step's launches, over the timed region",
            "kernels": {k: {"ms_avg": round(v[0] / v[1], 4), "sampled_launches": v[1],
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
            try:
                out["extras"] = run_extras(args, local)
            except Exception as e:  # (reported, never fatal to the headline line)
                out["extras"] = {"error": repr(e)[:300]}
        out["cpu_baseline"] = cpu_baseline(args)
    if ws > 1:
        dist.destroy_process_group()
    if rank == 0:
        print(json.dumps(out))


def _timed_shots(fn, reps, stream, prof=False):
    """prof: graph-sampled per-kernel timing over the timed shots (the untimed first call
    captures the graph with its event nodes)."""
    import torch

    import paper_conf_ppopp_qawasmehchc15_b200 as seis

    if prof:
        seis.profile(True, sample=PROF_SAMPLE)
    fn()
    torch.cuda.synchronize()
    if prof:
        seis.profile(True, sample=PROF_SAMPLE)  # zero the counters, keep the graph
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
    ms = _timed_shots(lambda: m.forward_model(shot, buf, stream), 2, stream, prof=True)
    seis.profile(False)
    res["iso_512"] = {"gpts_s": round(n ** 3 * 200 / (ms * 1e-3) / 1e9, 3), "ms_per_shot": round(ms, 3),
                      "roofline": kernel_frac("iso_step", float(n) ** 3, 16.0)}
    m.close()
    # the same with the ISO 2-step kernel (f1, opt-in SEIS_ISO2=1 at model creation; 20 B per
    # point per launch of two steps)
    old = os.environ.get("SEIS_ISO2")
    os.environ["SEIS_ISO2"] = "1"
    try:
        m = seis.Model(g, "iso", vp, device=local)
    finally:
        if old is None:
            del os.environ["SEIS_ISO2"]
        else:
            os.environ["SEIS_ISO2"] = old
    m.forward_model(shot, buf, stream)
    ms = _timed_shots(lambda: m.forward_model(shot, buf, stream), 2, stream, prof=True)
    seis.profile(False)
    res["iso_512_two_step"] = {"gpts_s": round(n ** 3 * 200 / (ms * 1e-3) / 1e9, 3), "ms_per_shot": round(ms, 3),
                               "roofline": kernel_frac("iso2", float(n) ** 3, 20.0),
                               "note": "f1 2-step temporal blocking, opt-in (slower than the one-step kernel)"}
    m.close()
    # the same with the split-field PML (O6b): layer points also read u^(d) at two levels and
    # write the new level (36 B per layer point)
    g = seis.Grid(n, n, n, 10.0, 1e-3, nb=20, iso_pml=1)
    m = seis.Model(g, "iso", vp, device=local)
    m.forward_model(shot, buf, stream)
    ms = _timed_shots(lambda: m.forward_model(shot, buf, stream), 2, stream, prof=True)
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
    ms = _timed_shots(lambda: m.forward_model(shot, buf, stream), 1, stream, prof=True)
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
    del mig, true, data, img, smooth, wl
    torch.cuda.empty_cache()
    if not args.no_c5:
        try:
            res["C5_rtm_1024_1gpu"] = run_c5(local)
        except Exception as e:  # an extra must never sink the headline line
            res["C5_rtm_1024_1gpu"] = {"error": repr(e)[:300]}
            torch.cuda.empty_cache()
    return res


def run_c5(local, n=1024, nt=1000):
    """C5 (BASELINE configs[4]) on ONE B200: acoustic RTM 1024^3, 1000 steps, snapshots every
    20 steps, 13 924-receiver carpet.  The 49 fp32 snapshots (196 GiB) do not fit in 180 GB, so
    the migration keeps source-state checkpoints and recomputes earlier segments (f2, P:181;
    the largest segment length that fits is chosen).  Observed data: forward modeling on the
    true salt model; migration on its Gaussian-smoothed copy (sigma 5 points)."""
    import torch

    import paper_conf_ppopp_qawasmehchc15_b200 as seis
    from paper_conf_ppopp_qawasmehchc15_b200 import inputs

    dev = torch.device("cuda", local)
    stream = torch.cuda.current_stream()
    t0 = time.perf_counter()
    wl = inputs.c5(n=n, nt=nt)
    build_s = time.perf_counter() - t0
    g = seis.Grid(wl.nx, wl.ny, wl.nz, wl.h, wl.dt, nb=wl.nb, pml_f=wl.fp)
    shot = seis.Shot(wl.src, wl.wavelet, wl.rec, snap_period=wl.snap)
    true = seis.Model(g, "acoustic", wl.model["vp"], rho=wl.model["rho"], device=local)
    data = torch.empty((wl.nt, shot.nrec), device=dev)
    fms = _timed_shots(lambda: true.forward_model(shot, data, stream), 1, stream)
    true.close()
    del true
    torch.cuda.empty_cache()
    sm = inputs.smooth_torch(wl.model, 5.0, dev)
    del wl.model
    free, _ = torch.cuda.mem_get_info(dev)
    img_bytes = float(wl.npts) * 4
    nsnap = (wl.nt - 1) // wl.snap
    c = 0
    if seis.memory_required(g, "acoustic", shot) + img_bytes > 0.95 * free:
        fits = [cc for cc in range(1, nsnap + 1)
                if seis.memory_required(g, "acoustic", seis.Shot(wl.src, wl.wavelet, wl.rec, snap_period=wl.snap,
                                                                 ckpt_period=cc)) + img_bytes <= 0.95 * free]
        # fewest recomputed steps: every segment but the last is recomputed once, (nseg - 1) c
        c = min(fits, key=lambda cc: ((nsnap + cc - 1) // cc - 1) * cc)
    rshot = seis.Shot(wl.src, wl.wavelet, wl.rec, snap_period=wl.snap, ckpt_period=c)
    mig = seis.Model(g, "acoustic", sm["vp"], rho=sm["rho"], device=local)
    del sm
    img = torch.zeros((wl.nz, wl.ny, wl.nx), device=dev)
    ms = _timed_shots(lambda: mig.migrate(rshot, data, img, stream), 1, stream)
    nseg = (nsnap + c - 1) // c if c else 1
    recomputed = sum(min((s_ + 1) * c, nsnap) * wl.snap - s_ * c * wl.snap for s_ in range(nseg - 1)) if c else 0
    mig.close()
    del mig, img, data
    torch.cuda.empty_cache()
    return {"shots_per_hour": round(3600.0 / (ms * 1e-3), 1), "ms_per_shot": round(ms, 1),
            "gpts_s_both_phases": round(2 * wl.npts * wl.nt / (ms * 1e-3) / 1e9, 3),
            "gpts_s_all_propagated_steps": round(wl.npts * (2 * wl.nt + recomputed) / (ms * 1e-3) / 1e9, 3),
            "forward_gpts_s": round(wl.npts * wl.nt / (fms * 1e-3) / 1e9, 3),
            "snapshots": nsnap, "ckpt_period": c, "segments": nseg, "recomputed_steps": recomputed,
            "receivers": shot.nrec, "model_build_s": round(build_s, 1),
            "note": "1 GPU; BASELINE C5 names 2/4/8 B200 (the driver's scaling run of the C2 line covers N > 1)"}


# ---------------------------------------------------------------- oracle arm
def cpu_model():
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    return line.split(":", 1)[1].strip()
    except Exception:
        pass
    return "unknown"


def _oracle_env():
    """OpenMP settings of every oracle timing: all host cores, threads bound close.
    Set before liboracle (and libgomp) is loaded in this process."""
    os.environ.setdefault("OMP_NUM_THREADS", str(os.cpu_count() or 1))
    os.environ.setdefault("OMP_PROC_BIND", "close")
    os.environ.setdefault("OMP_PLACES", "cores")
    return int(os.environ["OMP_NUM_THREADS"])


def _mem_available():
    try:
        with open("/proc/meminfo") as f:
            for line in f:
                if line.startswith("MemAvailable:"):
                    return int(line.split()[1]) * 1024
    except Exception:
        pass
    return 0


def oracle_timing(which, n=512, nz=None, nt=2000, warm=1, steps=5):
    """Time the fp64 oracle (as it stands) on `which` in THIS process: `warm` untimed time steps
    (first touch of the fp64 state), then `steps` timed ones (C1: whole shots).  Returns
    (Gpts/s, sample description).  C2 with nz > n (weak scaling config): the whole global grid
    when its fp64 state fits in half the available host memory, else the top n^3 z-block of
    the same model (same per-point work; stated in the sample)."""
    import oracle
    from paper_conf_ppopp_qawasmehchc15_b200 import inputs

    if which == "C1":
        wl = inputs.c1()
        g = oracle.Grid(wl.nx, wl.ny, wl.nz, wl.h, wl.dt, nb=wl.nb)
        run = lambda st, n0, k: oracle.iso_run(g, wl.model["vp"], st, 0, wl.nt, [wl.src], wl.wavelet[:, None],
                                               wl.rec)
        new = lambda: oracle.iso_state(g)
        pts, per, what = wl.npts, wl.nt, f"C1 ISO 64^3: {{k}} whole {wl.nt}-step shot(s)"
    elif which == "C3":
        wl = inputs.c3(n=n * 3 // 4)
        g = oracle.Grid(wl.nx, wl.ny, wl.nz, wl.h, wl.dt, nb=wl.nb, free_surface=1, pml_R=wl.pml_R, pml_f=wl.fp)
        m = wl.model
        run = lambda st, n0, k: oracle.el_run(g, m["vp"], m["vs"], m["rho"], st, n0, k, [wl.src],
                                              wl.wavelet[:, None], wl.rec, component=2)
        new = lambda: oracle.el_state(g)
        pts, per, what = wl.npts, 1, f"C3 elastic {wl.nx}^3: {{k}} time steps of the shot on the full grid"
    else:
        nz = n if nz is None else nz
        full = nz * n * n * (10 * 8 + 2 * 4) <= 0.5 * _mem_available() or nz == n
        nzs = nz if full else n
        wl = c2_workload(n=n, nt=nt, nz=nz, z0=0, nzl=nzs)
        g = oracle.Grid(wl.nx, wl.ny, nzs, wl.h, wl.dt, nb=wl.nb, pml_R=wl.pml_R, pml_f=wl.fp)
        m = wl.model
        run = lambda st, n0, k: oracle.ac_run(g, m["vp"], m["rho"], st, n0, k, [wl.src], wl.wavelet[:, None],
                                              wl.rec)
        new = lambda: oracle.ac_state(g)
        pts, per = float(n) * n * nzs, 1
        what = (f"C2 acoustic {n}x{n}x{nz}: {{k}} time steps of the shot on the full grid" if full else
                f"C2 acoustic {n}x{n}x{nz}: {{k}} time steps on its top {n}^3 z-block (the global grid's "
                f"fp64 state exceeds half the host memory)")
    st = new()
    if warm:
        run(st, 0, warm * per if per == 1 else per)
    t0 = time.perf_counter()
    if per == 1:
        run(st, warm, steps)
    else:
        for _ in range(steps):
            run(new(), 0, per)
    dt = time.perf_counter() - t0
    return pts * per * steps / dt / 1e9, what.format(k=steps) + f", after {warm} untimed warm-up, {dt:.1f} s"


def cpu_baseline(args):
    """The fp64 oracle (as it stands, test infrastructure) on the host cores, in a child process
    with OMP_NUM_THREADS = all cores and OMP_PROC_BIND=close: C2 (the headline config: 1 warm-up +
    5 timed time steps of the full 512^3 grid), plus C1 (whole shots) and C3 (2 steps)."""
    env = dict(os.environ, OMP_NUM_THREADS=str(os.cpu_count() or 1), OMP_PROC_BIND="close", OMP_PLACES="cores")
    out = {}
    for which, steps in (("C2", 5), ("C1", 3), ("C3", 2)):
        cmd = [sys.executable, os.path.abspath(__file__), "--oracle-timing", which, "--n", str(args.n),
               "--nt", str(args.nt), "--oracle-steps", str(steps)]
        try:
            r = subprocess.run(cmd, env=env, capture_output=True, text=True, timeout=600)
            out[which] = json.loads(r.stdout.strip().splitlines()[-1])
        except Exception as e:  # pragma: no cover - reported, not fatal
            out[which] = {"error": repr(e)[:200]}
    c2 = out.pop("C2")
    return {"value": c2.get("value"), "unit": "Gpts/s", "cores": int(env["OMP_NUM_THREADS"]), "kind": "oracle",
            "sample": c2.get("sample"), "cpu_model": cpu_model(), "omp": "OMP_PROC_BIND=close, OMP_PLACES=cores",
            "other_configs": out}


def run_reference(args):
    ws, rank, local = dist_env()
    if rank != 0:
        return
    cores = _oracle_env()
    n = args.n
    nz = n * ws if args.scaling == "weak" else n
    per = args.ref_steps
    value, sample = oracle_timing("C2", n=n, nz=nz, nt=args.nt, warm=args.warmup, steps=args.steps * per)
    wl = c2_workload(n=n, nt=args.nt, nz=nz, z0=0, nzl=1)  # geometry for the config (one plane)
    print(json.dumps({
        "impl": "reference", "metric": METRIC, "value": round(value, 5), "unit": "Gpts/s", "n_gpus": ws,
        "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": round(float(n) * n * nz * per / (value * 1e9) * 1e3, 1),
        "higher_is_better": True, "scaling": args.scaling, "vs_baseline": None, "dtype": "f64",
        "data": "synthetic (seeded layered model, Ricker source)",
        "config": c2_config(wl, nz, args.nt, wl.rec.shape[0], ws, args),
        "cpu_baseline": {"value": round(value, 5), "unit": "Gpts/s", "cores": cores, "kind": "oracle",
                         "sample": f"each step = {per} time step(s); " + sample, "cpu_model": cpu_model()},
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
    ap.add_argument("--no-c5", action="store_true", help="skip the 1024^3 RTM extra (about 2 minutes)")
    ap.add_argument("--scaling", default="weak", choices=["weak", "strong"],
                    help="N>1: weak = n^3 per rank (default), strong = one n^3 grid split in z-slabs")
    ap.add_argument("--halo", default="nccl", choices=["nccl", "peer"],
                    help="N>1 rank-face ghost exchange: NCCL send/recv overlapped with the interior "
                         "(default) or direct peer stores from the kernels (f4)")
    ap.add_argument("--oracle-timing", default=None, help=argparse.SUPPRESS)  # cpu_baseline child
    ap.add_argument("--oracle-steps", type=int, default=5, help=argparse.SUPPRESS)
    args = ap.parse_args()
    if args.oracle_timing:
        _oracle_env()
        v, smp = oracle_timing(args.oracle_timing, n=args.n, nt=args.nt, steps=args.oracle_steps)
        print(json.dumps({"value": round(v, 5), "unit": "Gpts/s", "sample": smp}))
        return
    if args.warmup < 3:
        print("warning: --warmup < 3 violates the timing rules", file=sys.stderr)
    if args.impl == "reference":
        run_reference(args)
    else:
        run_product(args)


if __name__ == "__main__":
    main()
