"""Per-instruction stall breakdown from an ncu report's source page: the top-N SASS lines by
stall samples with their dominant reasons, plus totals per reason.

    python tools/ncu_stalls.py <report.ncu-rep> [top]
"""
import csv
import io
import subprocess
import sys


def main(rep, top=25):
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    h = rows[1]
    iS, iN, iE = h.index("Source"), h.index("Warp Stall Sampling (All Samples)"), h.index("Instructions Executed")
    reasons = [(i, k) for i, k in enumerate(h) if k.startswith("stall_") and "Not Issued" not in k]
    tot = {k: 0.0 for _, k in reasons}
    lines = []
    for n, r in enumerate(rows[2:]):
        if len(r) <= iE:
            continue
        vals = {k: float(r[i] or 0) for i, k in reasons}
        for k, v in vals.items():
            tot[k] += v
        lines.append((float(r[iN] or 0), n, r[iE], r[iS].strip(), vals))
    s = sum(tot.values())
    print("totals:", ", ".join(f"{k[6:]} {100*v/s:.1f}%" for k, v in sorted(tot.items(), key=lambda x: -x[1]) if v))
    for smp, n, ex, src, vals in sorted(lines, reverse=True)[:top]:
        why = ", ".join(f"{k[6:]}:{int(v)}" for k, v in sorted(vals.items(), key=lambda x: -x[1])[:3] if v)
        print(f"{n:5d} {int(smp):6d} {ex:>9s}  {src[:60]:60s} {why}")


if __name__ == "__main__":
    main(sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else 25)
