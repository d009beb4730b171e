"""Evaluate throttle rules offline on every stored sweep (profiles/**/*.json
rows with a `swept` table): the B200 rule's pick, the alternative "keep full
TLP when the fit is below the TLP floor" (guarded, throttled picks -> full),
and full TLP, each as time / best swept time.
usage: python tools/rule_eval.py"""
import glob
import json

rows, seen = [], set()
for f in sorted(glob.glob("profiles/**/*.json", recursive=True)):
    try:
        txt = open(f).read().strip()
        d = json.loads(txt) if txt.startswith("[") else json.loads(txt.splitlines()[-1])
    except Exception:
        continue
    for r in d if isinstance(d, list) else (d.get("throttle_study") or []):
        if not isinstance(r, dict) or "swept" not in r:
            continue
        key = (r["loop"], r.get("cta_threads", r.get("cta")), r["carveout_kb"])
        if key in seen:
            continue
        seen.add(key)
        W, T = r["base"]
        sw = r["swept"]
        best = min(sw.values())
        pick = list(r.get("catt", r.get("b200")))
        rule = r.get("catt_rule", "?")
        guarded = "guard" in str(rule) or (isinstance(rule, int) and rule & 16)
        alt = [W, T] if (guarded and pick != [W, T]) else pick
        t = lambda p: sw[f"{p[0]},{p[1]}"] / best
        rows.append((r["loop"], key[1], key[2], pick, t(pick), alt, t(alt), t([W, T]), f.split("/")[-1]))
for loop, cta, carve, pick, tp, alt, ta, tf, src in rows:
    print(f"{loop[:34]:34s} cta{cta:5} carve{carve:4}  rule {pick} {tp:.3f}  alt {alt} {ta:.3f}  full {tf:.3f}  [{src}]")
print("worst: rule %.3f  alt %.3f  full %.3f" % (max(r[4] for r in rows), max(r[6] for r in rows), max(r[7] for r in rows)))
