"""L1 hit rate, DRAM bytes and duration of the picks at every launch of a
stored held-out study (row loops only: the literal row_thread kernel): the
library's pick, the pick without R27 ("r24"), full TLP and the best swept.
Run under ncu (each case launches twice, warm-up then measured: case i is
ncu launch 2i + 1):
  ncu --metrics l1tex__t_sector_hit_rate.pct,dram__bytes_read.sum,gpu__time_duration.sum \\
      -k regex:row_thread --csv --log-file OUT.csv python tools/l1_heldout.py STUDY.json
then python tools/l1_parse.py CASES.txt OUT.csv."""
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_kimhlsh19_b200 as catt  # noqa: E402

rows = json.load(open(sys.argv[1]))
dev = torch.device("cuda")
cases = []
arrays = {}
for r in rows:
    pr = r["prob"]
    if pr["loop"] not in (catt.K_BICG_2, catt.K_ATAX_1, catt.K_MVT_1):
        continue
    m = pr["m"] if pr["loop"] in (catt.K_BICG_2, catt.K_ATAX_1) else pr["n"]
    n = pr["n"]
    key = (m, n)
    if key not in arrays:
        A = torch.empty(m, n, device=dev)
        catt.fill_hash(A, 2)
        x = torch.empty(n, device=dev)
        catt.fill_hash(x, 102)
        arrays[key] = (A, x, torch.empty(m, device=dev))
    A, x, y = arrays[key]
    mode = catt.ROWS_ACCUM if pr["loop"] == catt.K_MVT_1 else catt.ROWS_STORE
    W, T = r["base"]
    launch = catt.Throttle(cta_threads=r["cta"], carveout_kb=r["carveout_kb"], variant=r.get("variant", "literal"))
    for label, (a, mm) in (("lib", r["b200"]), ("r24", r.get("r24", r["b200"])), ("full", [W, T]), ("best", r["best"])):
        th = launch.copy(active_warps=a, active_ctas=mm if mm < T else 0)
        cases.append((r["loop"], r["cta"], r["carveout_kb"], label, [a, mm],
                      lambda A=A, x=x, y=y, th=th, mode=mode: catt.rows(A, x, y, mode, t=th)))
torch.cuda.synchronize()
for i, c in enumerate(cases):
    print(json.dumps({"i": i, "workload": "heldout", "loop": c[0], "cta": c[1], "carveout_kb": c[2], "label": c[3],
                      "throttle": c[4]}), flush=True)
    c[5]()
    c[5]()
    torch.cuda.synchronize()
