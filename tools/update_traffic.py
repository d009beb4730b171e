"""Refresh profiles/ncu_traffic.json (the `traffic` field of bench.py's
roofline: dram__bytes_read.sum + dram__bytes_write.sum per launch of a
workload's dominant kernel) from ncu --set full reports of a gpurun pass.

usage: python tools/update_traffic.py gpurun_out/<tag> workload=report.ncu-rep [...]
e.g.   python tools/update_traffic.py gpurun_out/r2final syrk=ncu_t2_syrk.ncu-rep atax=ncu_default.ncu-rep
"""
import csv
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def dram_bytes(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True, check=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    h, units, vals = rows[0], rows[1], rows[2]
    d = dict(zip(h, vals))
    u = dict(zip(h, units))
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
    tot = 0.0
    for k in ("dram__bytes_read.sum", "dram__bytes_write.sum"):
        tot += float(d[k].replace(",", "")) * scale.get(u[k], 1)
    return int(round(tot)), d.get("Kernel Name", "")


def main():
    base = sys.argv[1]
    path = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    cur = json.load(open(path))
    notes = []
    for arg in sys.argv[2:]:
        wl, rep = arg.split("=", 1)
        b, kname = dram_bytes(os.path.join(base, rep))
        cur[wl] = b
        notes.append(f"{wl}: {kname[:40]} ({os.path.join(base, rep)})")
        print(wl, b, kname[:60])
    cur["_source"] = (cur.get("_source", "") + " | round 2: " + "; ".join(notes)).strip(" |")
    json.dump(cur, open(path, "w"), indent=1)


if __name__ == "__main__":
    main()
