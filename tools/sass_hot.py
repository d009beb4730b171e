"""Summarise an ncu `--page source --print-source sass --csv` export: instruction
mix and stall samples by opcode, and the hottest SASS lines.
usage: python tools/sass_hot.py file.csv [top]"""
import csv
import sys
from collections import Counter

r = list(csv.reader(open(sys.argv[1])))
top = int(sys.argv[2]) if len(sys.argv) > 2 else 25
h = r[1]
ci = h.index("Warp Stall Sampling (All Samples)")
ii = h.index("Instructions Executed")
rows = []
for k, row in enumerate(r[2:]):
    try:
        s, n = float(row[ci] or 0), float(row[ii] or 0)
    except (ValueError, IndexError):
        continue
    rows.append((s, n, row[0], row[1][:100]))
tot = sum(x[0] for x in rows) or 1
totn = sum(x[1] for x in rows) or 1
print("samples", tot, "warp instructions", totn)
cs, cn = Counter(), Counter()
for s, n, a, src in rows:
    parts = src.split()
    op = parts[1] if parts and parts[0].startswith("@") and len(parts) > 1 else (parts[0] if parts else "")
    op = op.split(".")[0]
    cs[op] += s
    cn[op] += n
for op, v in cn.most_common(24):
    print(f"{op:10s} inst {100 * v / totn:5.1f}%  samples {100 * cs[op] / tot:5.1f}%")
print("--- hottest lines")
for s, n, a, src in sorted(rows, reverse=True)[:top]:
    print(f"{100 * s / tot:5.1f}% {int(n):>10d} {a} {src}")
