"""Per-kernel SASS opcode summary of libcatt.so (cuobjdump -sass, static
counts): the opcodes that show which hardware path each kernel uses --
UBLKCP (bulk async copy), UTMALDG (TMA tensor load), SYNCS (mbarrier),
FFMA2 / FFMA (packed / scalar FP32 FMA), LDG / LDS / STG, and the tensor-core
opcodes (HMMA, UTC*MMA), which must be absent (north_star: no tensor cores on
these paths).
usage: python tools/sass_summary.py [libcatt.so] > profiles/.../sass_summary.txt"""
import re
import subprocess
import sys
from collections import Counter, defaultdict

lib = sys.argv[1] if len(sys.argv) > 1 else "paper_conf_icpp_kimhlsh19_b200/libcatt.so"
out = subprocess.run(["cuobjdump", "-sass", lib], capture_output=True, text=True, check=True).stdout
COLS = ["UBLKCP", "UTMALDG", "SYNCS", "FFMA2", "FFMA", "FADD2", "LDG", "LDS", "STG", "ATOM", "RED", "SHFL", "BAR",
        "HMMA", "UTCMMA"]
per = defaultdict(Counter)
name = None
for line in out.splitlines():
    m = re.search(r"Function : (\S+)", line)
    if m:
        name = m.group(1)
        continue
    m = re.match(r"\s+/\*[0-9a-f]{4,}\*/\s+(?:@!?U?P\w+\s+)?([A-Z][A-Z0-9_]*)", line)
    if m and name:
        op = m.group(1)
        per[name][op] += 1
        for c in COLS:
            if op == c or (c == "UTCMMA" and op.startswith("UTC") and "MMA" in op) or \
                    (c == "HMMA" and op in ("HMMA", "IMMA", "DMMA", "QMMA", "OMMA")) or \
                    (c == "ATOM" and op in ("ATOMG", "ATOMS")) or (c == "RED" and op in ("REDG", "REDAS")):
                per[name]["#" + c] += 1


def demangle(n):
    try:
        return subprocess.run(["c++filt", n], capture_output=True, text=True).stdout.strip()
    except Exception:
        return n


print(f"# static SASS opcode counts per kernel of {lib} (cuobjdump -sass, sm_100a)")
print("# kernel".ljust(92) + "".join(c.rjust(8) for c in COLS) + "   total")
tot = Counter()
for n in sorted(per, key=demangle):
    c = per[n]
    row = [c["#" + k] for k in COLS]
    tot.update({k: c["#" + k] for k in COLS})
    print(demangle(n)[:90].ljust(92) + "".join(str(v).rjust(8) for v in row) + str(sum(c.values())).rjust(8))
print("TOTAL".ljust(92) + "".join(str(tot[k]).rjust(8) for k in COLS))
print(f"# tensor-core opcodes (HMMA/IMMA/UTC*MMA) in the library: {tot['HMMA'] + tot['UTCMMA']}")
