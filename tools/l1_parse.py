"""Join tools/l1_study.py's case list with its ncu CSV: one row per case with
L1 sector hit rate, DRAM bytes, duration. usage: python tools/l1_parse.py cases.txt ncu.csv"""
import csv
import json
import sys

cases = [json.loads(l) for l in open(sys.argv[1]) if l.startswith("{")]
rows = list(csv.reader(open(sys.argv[2])))
hdr = next(i for i, r in enumerate(rows) if r and r[0] == "ID")
h = rows[hdr]
per = {}
for r in rows[hdr + 1:]:
    if len(r) < len(h):
        continue
    rid = int(r[h.index("ID")])
    per.setdefault(rid, {})[r[h.index("Metric Name")]] = (r[h.index("Metric Value")], r[h.index("Metric Unit")])
out = []
for c in cases:
    m = per.get(2 * c["i"] + 1, {})
    g = lambda k: m.get(k, ("nan", ""))
    c.update(l1_hit_pct=float(g("l1tex__t_sector_hit_rate.pct")[0].replace(",", "") or "nan"),
             dram_read=g("dram__bytes_read.sum"), duration=g("gpu__time_duration.sum"))
    out.append(c)
    print(f"{c['workload']:11s} {c['loop'][:28]:28s} cta {c['cta']:4d} carve {c['carveout_kb']:3d} {c['label']:5s} "
          f"{c['throttle']}  L1 hit {c['l1_hit_pct']:6.2f}%  dram {c['dram_read'][0]} {c['dram_read'][1]}  "
          f"dur {c['duration'][0]} {c['duration'][1]}")
json.dump(out, open(sys.argv[2].replace(".csv", ".json"), "w"), indent=1)
