"""One line per bench JSON (value, step time, roofline, e2e, cpu baseline) and
the throttle-study rows. usage: python tools/summarize_bench.py DIR"""
import glob
import json
import os
import sys

for f in sorted(glob.glob(os.path.join(sys.argv[1], "bench_*.json"))):
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
    except Exception as e:
        print(os.path.basename(f), "unreadable:", e)
        continue
    r = d.get("roofline") or {}
    e2e = d.get("e2e") or {}
    cpu = d.get("cpu_baseline") or {}
    print(f"{os.path.basename(f):26s} {d.get('value')} {d.get('unit')}  {d.get('ms_per_step')} ms/step  "
          f"roofline[{r.get('kernel')}] {r.get('achieved')} / {r.get('peak')} {r.get('unit')} = {r.get('frac')} "
          f"traffic {r.get('traffic')}  read-ctx {r.get('frac_of_same_size_read')}  e2e {e2e.get('value')}  "
          f"cpu {cpu.get('value')}  clocks {(d.get('clocks') or {}).get('sm_mhz')}")
    for lname, lv in (d.get("loops") or {}).items():
        print(f"      loop {lname:28s} {lv.get('ms')} ms  {lv.get('gbs')} GB/s  plan {(lv.get('plan') or {}).get('throttle')}")
    for s in d.get("throttle_study") or []:
        print(f"      study {s['loop'][:40]:40s} cta {s['cta_threads']:4d} carve {s['carveout_kb']:3d}  B200 {s['catt']} "
              f"{s['catt_over_best']}x best  paper {s['catt_paper']} {s['paper_over_best']}x  full/best "
              f"{round(s['full_ms'] / s['best_ms'], 3)}  best {s['best']}  bypass/best {s.get('bypass_over_best')}")
    for s in d.get("bftt_vs_catt") or []:
        print(f"      bftt  carve {s['carveout_kb']} catt {s['catt_ms']} ms  bftt {s['bftt_ms']} ms  "
              f"speedup {s['catt_speedup_over_bftt']}")
