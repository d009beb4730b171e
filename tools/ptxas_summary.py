"""Summarise an nvcc -Xptxas -v log: kernel, registers, spill bytes, smem."""
import re, subprocess, sys
txt = open(sys.argv[1]).read()
cur = None
rows = []
for line in txt.splitlines():
    m = re.search(r"Compiling entry function '(\S+)'", line)
    if m:
        cur = {"name": m.group(1)}
        rows.append(cur)
        continue
    m = re.search(r"(\d+) bytes spill stores, (\d+) bytes spill loads", line)
    if m and cur is not None:
        cur["spill"] = int(m.group(1)) + int(m.group(2))
    m = re.search(r"Used (\d+) registers.*?(\d+) bytes smem", line) or re.search(r"Used (\d+) registers", line)
    if m and cur is not None:
        cur["regs"] = int(m.group(1))
        cur["smem"] = int(m.group(2)) if m.lastindex and m.lastindex >= 2 else 0
names = [r["name"] for r in rows]
dem = subprocess.run(["c++filt"], input="\n".join(names), capture_output=True, text=True).stdout.splitlines()
for r, d in zip(rows, dem):
    d = d.replace("catt::", "").replace("(catt::", "(")
    print(f"{r.get('regs','?'):>4} regs  spill {r.get('spill',0):>4} B  smem {r.get('smem',0):>6}  {d[:90]}")
