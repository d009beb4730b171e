"""L1 hit rate of the CATT pick, the paper rule's pick, full TLP and the best
swept throttle (SURVEY 8(d) metric; BASELINE north_star reporting), for every
throttle-study row stored in a bench JSON directory.

Run under ncu (one launch per case, after one warm-up launch each):
  ncu --metrics l1tex__t_sector_hit_rate.pct,dram__bytes_read.sum,gpu__time_duration.sum \\
      --csv --log-file OUT.csv python tools/l1_study.py DIR [workload ...]
Filter ncu to the literal study kernels (-k regex:"row_thread|kmeans_kernel|
syrk_thread|syr2k_thread|km_transpose_thread"). Every case launches twice
(warm-up, then measured): case i is ncu launch 2i + 1. The workloads must be
the ones whose study loop is among those kernels."""
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
import paper_conf_icpp_kimhlsh19_b200 as catt  # noqa: E402

src = sys.argv[1]
names = sys.argv[2:] or ["bicg_mvt", "kmeans", "gesummv", "syrk", "syr2k", "kmeans_iter", "atax256"]
cases = []
for name in names:
    path = os.path.join(src, f"bench_{name}.json")
    if not os.path.exists(path):
        continue
    d = json.loads(open(path).read().strip().splitlines()[-1])
    rows = d.get("throttle_study") or []
    if not rows:
        continue
    w = bench.WORKLOADS[name](catt, torch, 0, 1, None)
    parts = {}
    for r in rows:
        W, T = r["base"]
        launch = catt.Throttle(cta_threads=r["cta_threads"], carveout_kb=r["carveout_kb"], variant="literal")
        picks = [("b200", r["catt"]), ("paper", r["catt_paper"]), ("full", [W, T]), ("best", r["best"])]
        for label, (a, m) in picks:
            th = launch.copy(active_warps=a, active_ctas=m if m < T else 0)
            fn = bench.study_fn(catt, w, th)
            sms = r.get("sm_partition")
            if sms:                                    # the row was measured on an SM partition (green context)
                if sms not in parts:
                    parts[sms] = catt.SmPartition(sms)

                def fn(f=fn, p=parts[sms]):
                    with torch.cuda.stream(p.stream):
                        f()
                    p.stream.synchronize()
            cases.append((name, r["loop"] + (f" [{sms} SMs]" if sms else ""), r["cta_threads"], r["carveout_kb"],
                          label, [a, m], fn))
    del w
    torch.cuda.empty_cache()
torch.cuda.synchronize()
for i, c in enumerate(cases):
    print(json.dumps({"i": i, "workload": c[0], "loop": c[1], "cta": c[2], "carveout_kb": c[3], "label": c[4],
                      "throttle": c[5]}), flush=True)
    c[6]()                                         # warm-up launch (odd ncu index)
    c[6]()                                         # the measured launch (even ncu index = 2i + 1)
    torch.cuda.synchronize()
