"""Re-plan every stored throttle sweep under a rule and score the pick.

Each stored sweep row (profiles/**: bench.py throttle_study rows, held-out
studies) has the time of every (a, m) at one launch. The problem of each loop
name is rebuilt here, the analyser (catt_plan, no GPU) picks (a, m) under the
rule, and the pick's time is divided by the best swept time.

usage: python tools/rule_replay.py [--rule b200|r24|r23|r18|paper] [--set final|heldout|heldout2|heldout3|heldout4|heldout5|heldout6|heldout7|heldout8|heldout9|partition|all] [-v]
  b200  = the library's B200 table (R18 + R19 + R23 re-touch term + R24 + R27 + R29 + R32)
  r29   = b200 without R32 (a divergent load shared by the CTA's warps is not a stream)
  r27   = the round-1 rule (b200 without R29's divergent-streams floor)
  r24   = the same without R27 (the floor fallback gates warps also with several CTAs per SM)
  r23   = R18 + R19 + R23 (re-touch and reuse-trip terms), as held-out study 2 tested it
  r18   = the new terms off (the round-1 rule as fitted)
  paper = guards off (the paper's Eq 9 as printed)
"""
import argparse
import ctypes
import glob
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_kimhlsh19_b200 as catt  # noqa: E402

P = catt.problem
# loop name -> (problem, variant), for the files of each set
LOOPS = {
    ("final", "bicg2 q=A p (literal, row per thread)"): (P(catt.K_BICG_2, m=4096, n=4096), "literal"),
    ("final", "gesummv (literal, row per thread)"): (P(catt.K_GESUMMV, n=8192), "literal"),
    ("final", "kmeans assign (literal, feature-major)"): (P(catt.K_KMEANS, m=494020, n=34, k=5, ld=494020), "literal"),
    ("final", "kmeans transpose (literal, point-major -> feature-major)"):
        (P(catt.K_KMEANS_T, m=494020, n=34, ld=494020), "literal"),
    ("final", "syrk (literal, 2-D block 32 x 8)"): (P(catt.K_SYRK, n=2048, k=2048), "literal"),
    ("final", "syr2k (literal, 2-D block 32 x 8)"): (P(catt.K_SYR2K, n=2048, k=2048), "literal"),
    ("final", "corr loop (literal, thread per column j1)"): (P(catt.K_CORR, n=2048, k=2048), "literal"),
    ("final", "gemm (literal, 2-D block 32 x 8)"): (P(catt.K_GEMM, m=512, n=512, k=512), "literal"),
    ("partition", "gesummv (literal, row per thread)"): (P(catt.K_GESUMMV, n=8192), "literal"),
    ("heldout", "syrk2048 literal"): (P(catt.K_SYRK, n=2048, k=2048), "literal"),
    ("heldout", "mvt1 literal"): (P(catt.K_MVT_1, n=4096), "literal"),
    ("heldout", "bicg2 vec4"): (P(catt.K_BICG_2, m=4096, n=4096), "vec4"),
    ("heldout", "kmeans ld=494048"): (P(catt.K_KMEANS, m=494020, n=34, k=5, ld=494048), "literal"),
}
FILES = {"final": sorted(glob.glob("profiles/r1p/bench_*.json")), "heldout": ["profiles/r1/heldout_study.json"],
         "heldout2": sorted(glob.glob("profiles/r1q/heldout2_study.json")),
         "heldout3": sorted(glob.glob("profiles/r1q/heldout3_study.json")),
         # 512/1024-thread row loops, measured to test the candidate R25 (not adopted)
         "heldout4": ["profiles/r1h4/heldout4_study.json"],
         # new loop shapes and CTA sizes (384/640/768 threads), no rule change under test
         "heldout5": ["profiles/r1h5/heldout5_study.json"],
         # 384-896-thread CTAs, measured to test the candidate R26 (not adopted)
         "heldout6": ["profiles/r1h6/heldout6_study.json"],
         # 320-1024-thread CTAs, measured to test the candidate R27 (adopted for T >= 2)
         "heldout7": ["profiles/r1h7/heldout7_study.json"],
         # several CTAs per SM, W = 12 / 16: R27 as adopted, pre-registered
         "heldout8": ["profiles/r1h8/heldout8_study.json"],
         # one CTA per SM at W = 10 / 12 / 14, measured to test the candidate R28 (not adopted)
         "heldout9": ["profiles/r1h9/heldout9_study.json"],
         # GESUMMV on SM partitions of 8 / 16 SMs (4 / 2 CTAs per SM), measured
         # after R24 was fixed: the CTA-level regime (SURVEY 8(d) [3])
         "partition": ["profiles/r1g/bench_gesummv.json"],
         # round 2: 2- and 3-stream rows at T = 1, testing the candidate R29 (adopted)
         "heldout10": ["profiles/r2/heldout10/heldout10_study.json"],
         # round 2: SYRK / SYR2K 2-D blocks, testing the candidate R32 (adopted)
         "heldout11": ["profiles/r2/heldout11/heldout11_study.json"],
         # round 2, closing: an out-of-sample check of the final rule (no change under test)
         "heldout12": ["profiles/r2/heldout12/heldout12_study.json"],
         # round 2, last session: a second out-of-sample check (no change under test)
         "heldout13": ["profiles/r2/heldout13/heldout13_study.json"],
         "heldout14": ["profiles/r2/heldout14/heldout14_study.json"]}
ATAX = {"bench_atax.json": P(catt.K_ATAX_1, m=65536, n=16384), "bench_atax256.json": P(catt.K_ATAX_1, m=256, n=256)}


def rows_of(f):
    txt = open(f).read().strip()
    d = json.loads(txt) if txt.startswith("[") else json.loads(txt.splitlines()[-1])
    return d if isinstance(d, list) else (d.get("throttle_study") or [])


def problem_of(s, f, r):
    if "prob" in r:                                   # rows that carry their problem (heldout2 and later)
        return P(r["prob"]["loop"], **{k: v for k, v in r["prob"].items() if k != "loop"}), r.get("variant", "literal")
    if r["loop"].startswith("atax1"):
        return ATAX[os.path.basename(f)], "literal"
    return LOOPS[(s, r["loop"])]


def rule_hw(name):
    hw = catt.hw_b200()
    if name == "b200":
        return hw
    hw.private_streams = 0                     # every older rule predates R32
    if name == "r29":                          # the library's rule before R32
        return hw
    if name != "b200":
        hw.stream_floor = 0                    # every older rule predates R29
    if name == "r18":
        hw.min_retouch, hw.min_reuse_trip, hw.max_stream_pct, hw.cta_fallback = 0, 0, 0, 0
    elif name == "r23":                        # as pre-registered for held-out study 2
        hw.min_retouch, hw.min_reuse_trip, hw.max_stream_pct, hw.cta_fallback = 16, 128, 0, 0
    elif name == "r24":                        # the library's rule before R27
        hw.cta_fallback = 0
    elif name == "r27":                        # the library's rule before R29 (round 1)
        pass
    elif name == "paper":
        hw = catt.paper_rule(hw)
    return hw


def replay(rule, sets, verbose):
    hw = rule_hw(rule)
    out = []
    for s in sets:
        for f in FILES[s]:
            for r in rows_of(f):
                if "swept" not in r:
                    continue
                if (s == "partition") != ("sm_partition" in r):
                    continue
                prob, var = problem_of(s, f, r)
                cta = r.get("cta_threads", r.get("cta"))
                launch = catt.Throttle(cta_threads=cta, carveout_kb=r["carveout_kb"], variant=var)
                hw_l = hw
                if "sm_partition" in r:
                    hw_l = catt.Hw()
                    ctypes.memmove(ctypes.byref(hw_l), ctypes.byref(hw), ctypes.sizeof(catt.Hw))
                    hw_l.num_sms = r["sm_partition"]
                t, res = catt.plan(prob, launch, hw_l)
                W, T = res["base_warps"], res["base_ctas"]
                if [W, T] != list(r["base"]):
                    raise SystemExit(f"base mismatch {r['loop']} {cta} {r['carveout_kb']}: {W, T} vs {r['base']}")
                sw = dict(r["swept"]) if isinstance(r["swept"], list) else r["swept"]
                best = min(sw.values())
                pick = (t.active_warps or W, t.active_ctas or T)
                q = sw[f"{pick[0]},{pick[1]}"] / best
                full = sw[f"{W},{T}"] / best
                out.append((s, r["loop"], cta, r["carveout_kb"], pick, q, full))
                if verbose:
                    print(f"{s:8s} {r['loop'][:40]:40s} cta {cta:5d} carve {r['carveout_kb']:3d}  pick {pick}  "
                          f"{q:.3f}x best  full {full:.3f}x")
    return out


if __name__ == "__main__":
    ap = argparse.ArgumentParser()
    ap.add_argument("--rule", default="b200", choices=["b200", "r29", "r27", "r24", "r23", "r18", "paper"])
    ap.add_argument("--set", default="all", choices=["final", "heldout", "heldout2", "heldout3", "heldout4", "heldout5", "heldout6", "heldout7", "heldout8", "heldout9", "partition", "heldout10", "heldout11", "heldout12", "heldout13", "heldout14", "all"])
    ap.add_argument("-v", action="store_true")
    a = ap.parse_args()
    sets = ["final", "heldout", "heldout2", "heldout3", "heldout4", "heldout5", "heldout6", "heldout7", "heldout8", "heldout9", "partition", "heldout10", "heldout11", "heldout12", "heldout13", "heldout14"] if a.set == "all" else [a.set]
    res = replay(a.rule, sets, a.v)
    for s in sets:
        rs = [x for x in res if x[0] == s]
        if not rs:
            continue
        within = sum(1 for x in rs if x[5] <= 1.05)
        contended = [x for x in rs if x[6] > 1.05]
        beats = sum(1 for x in contended if x[5] < x[6] / 1.0)
        slower = sum(1 for x in rs if x[5] > 1.05 * x[6])
        print(f"[{a.rule}] {s}: {within}/{len(rs)} within 5% of best swept; worst {max(x[5] for x in rs):.3f}x; "
              f"launches where some throttle beats full TLP by >5%: {len(contended)}, pick beats full TLP on "
              f"{beats} of them; pick >5% slower than full TLP on {slower}")
    # the paper's headline form (P:7: speedup over the baseline's full TLP and
    # over the best static throttle), as geometric means over the launches
    import math
    gm = lambda v: math.exp(sum(math.log(x) for x in v) / len(v)) if v else float("nan")
    cont = [x for x in res if x[6] > 1.05]
    print(f"[{a.rule}] geomean over {len(res)} launches: speedup over full TLP {gm([x[6] / x[5] for x in res]):.3f}x, "
          f"pick / best swept {gm([x[5] for x in res]):.3f}x; over the {len(cont)} launches where full TLP is >5% "
          f"off the best: speedup over full TLP {gm([x[6] / x[5] for x in cont]):.3f}x "
          f"(best swept: {gm([x[6] for x in cont]):.3f}x)")
