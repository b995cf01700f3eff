"""Instruction mix and stall samples by SASS opcode from an ncu report's source page.

    python tools/ncu_sass_mix.py <report.ncu-rep> [top]
"""
import csv
import io
import subprocess
import sys
from collections import defaultdict


def main(rep, top=30):
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    h = rows[1]
    iS, iN, iE = h.index("Source"), h.index("Warp Stall Sampling (All Samples)"), h.index("Instructions Executed")
    inst, samp = defaultdict(float), defaultdict(float)
    for r in rows[2:]:
        if len(r) <= iE:
            continue
        op = r[iS].strip().split()
        if not op:
            continue
        o = op[0] if not op[0].startswith("@") else op[1]
        o = o.split(".")[0]
        inst[o] += float(r[iE] or 0)
        samp[o] += float(r[iN] or 0)
    ti, ts = sum(inst.values()), sum(samp.values())
    print(f"{'opcode':12s} {'inst':>12s} {'%inst':>6s} {'%stall':>6s}")
    for o in sorted(inst, key=lambda k: -inst[k])[:top]:
        print(f"{o:12s} {inst[o]:12.0f} {100*inst[o]/ti:6.1f} {100*samp[o]/ts:6.1f}")
    print(f"total inst {ti:.0f}")


if __name__ == "__main__":
    main(sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else 30)
