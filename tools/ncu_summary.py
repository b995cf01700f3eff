"""Summarise ncu reports / launch lists into the compact text committed under profiles/.

    python tools/ncu_summary.py full <report.ncu-rep> [points_per_launch alg_bytes_per_point]
    python tools/ncu_summary.py launches <launches.csv>
"""
import csv
import io
import subprocess
import sys
from collections import defaultdict

KEYS = [
    "gpu__time_duration.sum",
    "dram__bytes_read.sum",
    "dram__bytes_write.sum",
    "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
    "dram__throughput.avg.pct_of_peak_sustained_elapsed",
    "lts__t_bytes.sum",
    "l1tex__t_bytes.sum",
    "sm__throughput.avg.pct_of_peak_sustained_elapsed",
    "sm__warps_active.avg.pct_of_peak_sustained_active",
    "sm__maximum_warps_per_active_cycle_pct",
    "launch__registers_per_thread",
    "launch__occupancy_limit_registers",
    "launch__occupancy_limit_shared_mem",
    "launch__grid_size",
    "launch__block_size",
    "sm__cycles_elapsed.avg.per_second",
    "smsp__inst_executed.sum",
    "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active",
    "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum",
    "smsp__average_warp_latency_issue_stalled_barrier",
    "smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_barrier_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_mio_throttle_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_lg_throttle_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_short_scoreboard_per_issue_active.ratio",
    "smsp__issue_active.avg.pct_of_peak_sustained_active",
]


def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    if len(rows) < 3:
        return []
    hdr, units = rows[0], rows[1]
    res = []
    for r in rows[2:]:
        res.append({h: (v, u) for h, u, v in zip(hdr, units, r)})
    return res


def num(v):
    try:
        return float(str(v).replace(",", ""))
    except ValueError:
        return None


def full(rep, pts=None, bpp=None):
    for rec in raw(rep):
        name = rec.get("Kernel Name", ("?", ""))[0]
        print(f"kernel: {name[:120]}")
        for k in KEYS:
            if k in rec:
                print(f"  {k} = {rec[k][0]} {rec[k][1]}")
        t = num(rec.get("gpu__time_duration.sum", (None,))[0])
        unit = rec.get("gpu__time_duration.sum", ("", ""))[1]
        scale = {"ns": 1e-9, "us": 1e-6, "usecond": 1e-6, "nsecond": 1e-9, "ms": 1e-3, "msecond": 1e-3}.get(unit, 1e-9)
        bs = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
        rb = num(rec.get("dram__bytes_read.sum", (None,))[0])
        wb = num(rec.get("dram__bytes_write.sum", (None,))[0])
        if t and rb is not None and wb is not None:
            rb *= bs.get(rec["dram__bytes_read.sum"][1], 1)
            wb *= bs.get(rec["dram__bytes_write.sum"][1], 1)
            tr = rb + wb
            print(f"  => dram traffic {tr / 1e6:.1f} MB, {tr / (t * scale) / 1e9:.1f} GB/s over {t * scale * 1e3:.3f} ms")
            if pts and bpp:
                alg = float(pts) * float(bpp)
                print(f"  => algorithmic {alg / 1e6:.1f} MB ({bpp} B/pt x {pts} pts): traffic/alg = {tr / alg:.3f}, "
                      f"alg GB/s = {alg / (t * scale) / 1e9:.1f}")


def launches(path):
    txt = open(path).read()
    i = txt.find('"ID"')
    rows = list(csv.reader(io.StringIO(txt[i:])))
    hdr = rows[0]
    ki, vi, ui = hdr.index("Kernel Name"), hdr.index("Metric Value"), hdr.index("Metric Unit")
    tot = defaultdict(float)
    cnt = defaultdict(int)
    for r in rows[1:]:
        if len(r) <= vi:
            continue
        v = num(r[vi])
        if v is None:
            continue
        s = {"nsecond": 1e-3, "usecond": 1.0, "msecond": 1e3}.get(r[ui], 1e-3)
        name = r[ki].split("(")[0]
        tot[name] += v * s
        cnt[name] += 1
    T = sum(tot.values())
    print(f"{'kernel':60s} {'launches':>8s} {'total us':>12s} {'avg us':>10s} {'share':>7s}")
    for k in sorted(tot, key=lambda k: -tot[k]):
        print(f"{k[:60]:60s} {cnt[k]:8d} {tot[k]:12.1f} {tot[k] / cnt[k]:10.2f} {tot[k] / T:7.1%}")


if __name__ == "__main__":
    if sys.argv[1] == "full":
        full(sys.argv[2], *(sys.argv[3:5] if len(sys.argv) > 4 else (None, None)))
    else:
        launches(sys.argv[2])
