"""Write tests/golden/b200_rule_picks.json: the B200 rule's pick at every
launch of the stored throttle sweeps (the 243 replayed launches of
tools/rule_replay.py: round 1's 160 and round 2's held-out studies 10-14), derived ONLY from oracle/ (address traces of the loop
bodies, the LRU L1D simulator, oracle.footprint.occupancy for W and T).

TEST INFRASTRUCTURE: calls nothing but oracle/ (no library, no device). The
launch specifications (problem, CTA size, carveout, SM partition) are read
from the stored sweep files; the library's own picks and bases in those files
are ignored. Trip counts of the row / tile loops are shortened (the footprint
per iteration and the re-touch count do not depend on them; the row start's
alignment, N mod 32, is kept); everything else is at the launch's full size.

usage: python tools/gen_rule_golden.py [-j JOBS]
"""
import argparse
import glob
import json
import math
import os
import sys
from concurrent.futures import ProcessPoolExecutor

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
os.chdir(ROOT)

from oracle import b200_rule as br  # noqa: E402
from oracle import footprint as fp  # noqa: E402
from oracle import lru  # noqa: E402

# catt.h CATT_K_* (ABI constants)
K_ATAX_1, K_ATAX_2, K_BICG_1, K_BICG_2, K_MVT_1, K_MVT_2, K_GESUMMV, K_SYRK, K_KMEANS, K_SYR2K, K_KMEANS_T, K_CORR, \
    K_GEMM, K_ROWS3 = range(14)
ROWS = (K_ATAX_1, K_BICG_2, K_MVT_1, K_GESUMMV, K_ROWS3)
MATS = {K_GESUMMV: ("A", "B"), K_ROWS3: ("A", "B", "C")}

LOOPS = {  # (set, loop name) -> (problem, variant) for the sweep rows that do not carry their problem
    ("final", "bicg2 q=A p (literal, row per thread)"): (dict(loop=K_BICG_2, m=4096, n=4096), "literal"),
    ("final", "gesummv (literal, row per thread)"): (dict(loop=K_GESUMMV, n=8192), "literal"),
    ("final", "kmeans assign (literal, feature-major)"): (dict(loop=K_KMEANS, m=494020, n=34, k=5, ld=494020), "literal"),
    ("final", "kmeans transpose (literal, point-major -> feature-major)"):
        (dict(loop=K_KMEANS_T, m=494020, n=34, ld=494020), "literal"),
    ("final", "syrk (literal, 2-D block 32 x 8)"): (dict(loop=K_SYRK, n=2048, k=2048), "literal"),
    ("final", "syr2k (literal, 2-D block 32 x 8)"): (dict(loop=K_SYR2K, n=2048, k=2048), "literal"),
    ("final", "corr loop (literal, thread per column j1)"): (dict(loop=K_CORR, n=2048, k=2048), "literal"),
    ("final", "gemm (literal, 2-D block 32 x 8)"): (dict(loop=K_GEMM, m=512, n=512, k=512), "literal"),
    ("partition", "gesummv (literal, row per thread)"): (dict(loop=K_GESUMMV, n=8192), "literal"),
    ("heldout", "syrk2048 literal"): (dict(loop=K_SYRK, n=2048, k=2048), "literal"),
    ("heldout", "mvt1 literal"): (dict(loop=K_MVT_1, n=4096), "literal"),
    ("heldout", "bicg2 vec4"): (dict(loop=K_BICG_2, m=4096, n=4096), "vec4"),
    ("heldout", "kmeans ld=494048"): (dict(loop=K_KMEANS, m=494020, n=34, k=5, ld=494048), "literal"),
}
ATAX = {"bench_atax.json": dict(loop=K_ATAX_1, m=65536, n=16384), "bench_atax256.json": dict(loop=K_ATAX_1, m=256, n=256)}
FILES = {"final": sorted(glob.glob("profiles/r1p/bench_*.json")), "heldout": ["profiles/r1/heldout_study.json"],
         "heldout2": ["profiles/r1q/heldout2_study.json"], "heldout3": ["profiles/r1q/heldout3_study.json"],
         "heldout4": ["profiles/r1h4/heldout4_study.json"], "heldout5": ["profiles/r1h5/heldout5_study.json"],
         "heldout6": ["profiles/r1h6/heldout6_study.json"], "heldout7": ["profiles/r1h7/heldout7_study.json"],
         "heldout8": ["profiles/r1h8/heldout8_study.json"], "heldout9": ["profiles/r1h9/heldout9_study.json"],
         "partition": ["profiles/r1g/bench_gesummv.json"],
         "heldout10": ["profiles/r2/heldout10/heldout10_study.json"],
         "heldout11": ["profiles/r2/heldout11/heldout11_study.json"],
         "heldout12": ["profiles/r2/heldout12/heldout12_study.json"],
         # round 2, last session: a second out-of-sample check (no change under test)
         "heldout13": ["profiles/r2/heldout13/heldout13_study.json"],
         "heldout14": ["profiles/r2/heldout14/heldout14_study.json"]}
SETS = list(FILES)


def rows_of(f):
    txt = open(f).read().strip()
    d = json.loads(txt) if txt.startswith("[") else json.loads(txt.splitlines()[-1])
    return d if isinstance(d, list) else (d.get("throttle_study") or [])


def launches():
    for s in SETS:
        for f in FILES[s]:
            for r in rows_of(f):
                if "swept" not in r or (s == "partition") != ("sm_partition" in r):
                    continue
                if "prob" in r:
                    prob, var = dict(r["prob"]), r.get("variant", "literal")
                elif r["loop"].startswith("atax1"):
                    prob, var = ATAX[os.path.basename(f)], "literal"
                else:
                    prob, var = LOOPS[(s, r["loop"])]
                yield dict(set=s, loop=r["loop"], prob=prob, variant=var, cta=r.get("cta_threads", r.get("cta")),
                           carveout_kb=r["carveout_kb"], sm_partition=r.get("sm_partition", 0))


def _short(n, floor=160, keep=128):
    """A shorter trip count with the same alignment mod 32 (and >= 32 steps)."""
    return n if n <= floor else keep + n % 32


def shape(L):
    """(trace kernel, oracle Loop for occupancy) of one launch."""
    p, cta, var = L["prob"], L["cta"], L["variant"]
    loop = p["loop"]
    smem = 16                                   # the literal kernels' static shared memory (gate slot)
    if loop in ROWS:
        M = p["n"] if loop in (K_MVT_1, K_GESUMMV) else p["m"]
        N = p["n"]
        vec = 4 if var == "vec4" else 1
        k = lru.RowKernel(M, _short(N), cta, vec=vec, matrices=MATS.get(loop, ("A",)))
        block, grid = (cta, 1, 1), (math.ceil(M / cta), 1, 1)
    elif loop in (K_SYRK, K_SYR2K, K_GEMM):
        by = cta // 32
        if loop == K_GEMM:
            k = lru.GemmKernel(p["m"], p["n"], _short(p["k"], 96, 64), bdim=(32, by))
            grid = (math.ceil(p["n"] / 32), math.ceil(p["m"] / by), 1)
        else:
            cls = lru.SyrkKernel if loop == K_SYRK else lru.Syr2kKernel
            k = cls(p["n"], _short(p["k"], 96, 64), bdim=(32, by))
            grid = (math.ceil(p["n"] / 32), math.ceil(p["n"] / by), 1)
        block = (32, by, 1)
    elif loop == K_KMEANS:
        k = lru.KmeansKernel(p["m"], p["n"], p["k"], p["ld"], cta)
        block, grid = (cta, 1, 1), (math.ceil(p["m"] / cta), 1, 1)
        smem += p["n"] * p["k"] * 4             # the centres staged in shared memory
    elif loop == K_KMEANS_T:
        k = lru.TransposeKernel(p["m"], p["n"], p["ld"], cta)
        block, grid = (cta, 1, 1), (math.ceil(p["m"] / cta), 1, 1)
    elif loop == K_CORR:
        k = lru.CorrKernel(p["n"], 4, cta)       # the i loop shortened: the reused line is the coalesced j1 column
        block, grid = (cta, 1, 1), (math.ceil(p["n"] / cta), 1, 1)
    else:
        raise ValueError(loop)
    return k, fp.Loop(refs=[], trips=(), block=block, grid=grid, smem=smem, force_carveout_kb=L["carveout_kb"])


def decide(L):
    k, lp = shape(L)
    hw = br.b200_hw(L["sm_partition"] or 148)
    W, T, carve, l1d = fp.occupancy(lp, hw)
    a, m, how = br.decide(k, W, T, l1d // 128, hw["num_sms"])
    return dict(L, W=W, T=T, l1d_lines=l1d // 128, pick=[a, m], how=how)


if __name__ == "__main__":
    ap = argparse.ArgumentParser()
    ap.add_argument("-j", type=int, default=os.cpu_count() or 1)
    ap.add_argument("--out", default=os.path.join("tests", "golden", "b200_rule_picks.json"))
    a = ap.parse_args()
    Ls = list(launches())
    with ProcessPoolExecutor(a.j) as ex:
        out = list(ex.map(decide, Ls))
    json.dump({"generator": "tools/gen_rule_golden.py (oracle/ only: lru traces + LRU fit + occupancy)",
               "guards": br.B200_GUARDS, "launches": out}, open(a.out, "w"), indent=1)
    print(f"{len(out)} launches -> {a.out}")
