"""Write profiles/traffic.json: DRAM bytes (read + write) per launch of the kernels
bench.py reports a roofline for, taken from one `ncu --set full` capture each.

    python tools/ncu_traffic.py <tag>      # reads gpurun_out/<tag>_{ac_v,ac_p,iso,el_v,el_s}.ncu-rep
"""
import csv
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
UNIT = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
# report name -> (bench key, workload)
REPORTS = {"ac_v": "C2_512_ac_v", "ac_p": "C2_512_ac_p", "iso": "iso_512_iso_step",
           "el_v": "C3_384_el_v", "el_s": "C3_384_el_s"}


def dram_bytes(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units, vals = rows[0], rows[1], rows[2]
    get = lambda k: float(vals[hdr.index(k)].replace(",", "")) * UNIT.get(units[hdr.index(k)], 1)
    return get("dram__bytes_read.sum") + get("dram__bytes_write.sum")


def main(tag):
    path = os.path.join(ROOT, "profiles", "traffic.json")
    res = json.load(open(path)) if os.path.exists(path) else {}
    for rep, key in REPORTS.items():
        f = os.path.join(ROOT, "gpurun_out", f"{tag}_{rep}.ncu-rep")
        if os.path.exists(f):
            res[key] = round(dram_bytes(f))
    res["_source"] = f"ncu --set full --clock-control none, one launch each, capture {tag}"
    json.dump(res, open(path, "w"), indent=1, sort_keys=True)
    print(json.dumps(res, indent=1))


if __name__ == "__main__":
    main(sys.argv[1])
