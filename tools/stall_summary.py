"""Stall reasons and instruction mix of one kernel from an ncu source export
(`ncu -i X.ncu-rep --page source --print-source sass --csv`).
usage: python tools/stall_summary.py file.csv"""
import csv
import sys
from collections import Counter

r = list(csv.reader(open(sys.argv[1], encoding="latin-1")))
h = r[1]
ii = h.index("Instructions Executed")
cols = [k for k, x in enumerate(h) if x.startswith("stall_") and "Not Issued" not in x]
tot = Counter()
mix = Counter()
ninst = 0.0
for row in r[2:]:
    try:
        n = float(row[ii] or 0)
    except (ValueError, IndexError):
        continue
    ninst += n
    op = row[1].strip().split()
    op = (op[1] if op and op[0].startswith("@") and len(op) > 1 else (op[0] if op else "?")).split(".")[0]
    mix[op] += n
    for k in cols:
        try:
            tot[h[k]] += float(row[k] or 0)
        except ValueError:
            pass
s = sum(tot.values()) or 1
print("stall samples:", int(s), " warp instructions:", int(ninst))
for k, v in tot.most_common(10):
    print(f"  {k:28s} {100 * v / s:5.1f}%")
print("instruction mix:")
for k, v in mix.most_common(12):
    print(f"  {k:10s} {100 * v / ninst:5.1f}%")
