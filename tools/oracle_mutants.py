"""Mutation check of the oracle's pins (task rule 3: the pins are "chosen so
that a plausible mistake anywhere in it (a dropped term, a wrong sign or
index, a transposed operand) fails one of them").

Each mutant is one plausible mistake typed into a copy of oracle/ (the C loop
nests, Eq 1-9, the LRU simulator, the B200 rule oracle, the exact k-means
update). The `-m "not gpu"` oracle tests then run against the copy (it comes
first on sys.path: the tests import `oracle` from the working directory);
the mutant is KILLED when some test fails. Nothing here touches the product
package or the GPU.

usage: python tools/oracle_mutants.py [--only NAME ...] [--jobs N] [--out FILE]
"""
import argparse
import os
import shutil
import subprocess
import sys
import tempfile
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
TESTS = ["tests/test_oracle.py", "tests/test_oracle_kmeans.py", "tests/test_b200_rule.py"]

# name: (file under oracle/, text, replacement, count, what the mistake is).
# count = how many occurrences are replaced (0 = all).
MUTANTS = {
    # ---- the loop nests (oracle/loops.c), seq-fmaf and f64 paths alike
    # control: no change (must survive, or the harness itself is broken)
    "control_unchanged": ("loops.c", "/* ---------------------------------------------------------------- ATAX",
                          "/* ---------------------------------------------------------------- ATAX", 1,
                          "no change (control: must survive)"),
    "atax_transposed_second_loop": ("loops.c", "acc = fmaf(A[i * n + j], tmp[i], acc);",
                                    "acc = fmaf(A[j * n + i], tmp[i], acc);", 1,
                                    "ATAX y = A^T tmp reads A untransposed"),
    "atax_first_loop_uses_y": ("loops.c", "acc = fmaf(A[i * n + j], x[j], acc);",
                               "acc = fmaf(A[i * n + j], x[i % n], acc);", 1, "ATAX tmp indexes x by the row"),
    "bicg_p_r_swapped": ("loops.c", "acc = fmaf(A[i * ny + j], p[j], acc);",
                         "acc = fmaf(A[i * ny + j], r[j % nx], acc);", 1, "BICG q = A r instead of A p"),
    "mvt_second_not_transposed": ("loops.c", "acc2 = fmaf(a[j * n + i], y2[j], acc2);",
                                  "acc2 = fmaf(a[i * n + j], y2[j], acc2);", 1, "MVT x2 += A y2 (not A^T)"),
    "mvt_drops_initial_x": ("loops.c", "float acc1 = x1[i], acc2 = x2[i];", "float acc1 = 0.0f, acc2 = x2[i];", 1,
                            "MVT x1 starts from 0 (drops the in/out term)"),
    "gesummv_alpha_beta_swapped": ("loops.c", "y[i] = fmaf(alpha, t, beta * yb);", "y[i] = fmaf(beta, t, alpha * yb);",
                                   1, "GESUMMV alpha and beta swapped"),
    "gesummv_drops_b": ("loops.c", "yb = fmaf(B[i * n + j], x[j], yb);", "yb = fmaf(A[i * n + j], x[j], yb);", 1,
                        "GESUMMV uses A for both products"),
    "rows3_drops_c": ("loops.c", "y[i] = (a + b) + c;", "y[i] = (a + b);", 1, "three-stream row loop drops C x"),
    "syrk_beta_dropped": ("loops.c", "float c = C[i * n + j] * beta;\n        for (int64_t k = 0; k < m; ++k) c = fmaf(alpha * A[i * m + k], A[j * m + k], c);\n        C[i * n + j] = c;",
                          "float c = C[i * n + j];\n        for (int64_t k = 0; k < m; ++k) c = fmaf(alpha * A[i * m + k], A[j * m + k], c);\n        C[i * n + j] = c;",
                          1, "SYRK forgets C *= beta"),
    "syrk_wrong_operand": ("loops.c", "for (int64_t k = 0; k < m; ++k) c = fmaf(alpha * A[i * m + k], A[j * m + k], c);\n        C[i * n + j] = c;",
                           "for (int64_t k = 0; k < m; ++k) c = fmaf(alpha * A[i * m + k], A[i * m + k], c);\n        C[i * n + j] = c;",
                           1, "SYRK squares row i (a_ik a_ik)"),
    "syr2k_drops_second_product": ("loops.c", "const float s = fmaf(p, B[j * m + k], t);", "const float s = p * B[j * m + k];",
                                   1, "SYR2K drops alpha b_ik a_jk"),
    "syr2k_sign": ("loops.c", "const float s = fmaf(p, B[j * m + k], t);", "const float s = fmaf(p, B[j * m + k], -t);",
                   1, "SYR2K subtracts the second product"),
    "gemm_b_transposed": ("loops.c", "c = fmaf(alpha * A[i * nk + k], B[k * nj + j], c);",
                          "c = fmaf(alpha * A[i * nk + k], B[j * nk + k], c);", 1, "GEMM reads B transposed"),
    "corr_sample_std": ("loops.c", "sd = sqrtf(sd / fn);", "sd = sqrtf(sd / (fn - 1.0f));", 1,
                        "CORR sample (n - 1) instead of population std"),
    "corr_eps_strict": ("loops.c", "if (sd <= eps) sd = 1.0f;", "if (sd < 0.0f) sd = 1.0f;", 1,
                        "CORR never replaces a tiny std by 1"),
    "kmeans_ties_last": ("loops.c", "if (d < min_dist) {", "if (d <= min_dist) {", 1,
                         "KMEANS ties go to the highest centre"),
    "seq_fmaf_unfused": ("loops.c", "for (int64_t j = 0; j < n; ++j) acc = fmaf(A[i * n + j], x[j], acc);",
                         "for (int64_t j = 0; j < n; ++j) acc = acc + A[i * n + j] * x[j];", 1,
                         "ATAX row dot rounded twice per step (mul then add)"),
    "kmeans_assign_unfused": ("loops.c", "\n        d = fmaf(diff, diff, d);", "\n        d = d + diff * diff;", 1,
                              "KMEANS distance rounded twice per feature"),
    "generator_constant": ("loops.c", "h *= 0x85EBCA6Bu;", "h *= 0x85EBCA6Du;", 1,
                           "the counter-based generator's mixing constant mistyped"),
    "generator_dyadic_grid": ("loops.c", "(float)(h & 15u) * (1.0f / 16.0f)", "(float)(h & 15u) * (1.0f / 8.0f)", 1,
                              "dyadic inputs on the 1/8 grid (range up to 15/8)"),
    # ---- Eq 1-9 (oracle/footprint.py)
    "eq6_not_strict": ("footprint.py", "abs(ref.c_iter[k]) * ref.elem_bytes < line and trips[k] >= 2 for k",
                       "abs(ref.c_iter[k]) * ref.elem_bytes <= line and trips[k] >= 2 for k", 1,
                       "Eq 6 with <= (a line-sized stride 'has locality')"),
    "eq7_floor": ("footprint.py", "return min(ws, _ceil_div(ws * c * e, line))", "return min(ws, (ws * c * e) // line)",
                  1, "Eq 7 rounds the lines per warp request down"),
    "eq2_no_registers": ("footprint.py", "            limits.append(warps // W)\n", "", 1,
                         "Eq 2 (register limit) dropped on B200"),
    "eq3_no_grid_bound": ("footprint.py", "    limits.append(_ceil_div(gx * gy * gz, hw[\"num_sms\"]))                 # grid bound (R8)\n",
                          "", 1, "Eq 3 without the grid bound"),
    "eq4_largest_carveout": ("footprint.py", "idx = next(i for i, c in enumerate(carve) if c * 1024 >= need)",
                             "idx = len(carve) - 1", 1, "Eq 4 always takes the largest shared-memory option"),
    "eq8_paper_drops_ctas": ("footprint.py", "return self.req * a * m", "return self.req * a", 1,
                             "Eq 8 (paper mode) forgets the co-resident CTAs"),
    # ---- the LRU simulator (oracle/lru.py)
    "lru_evicts_mru": ("lru.py", "cache.popitem(last=False)", "cache.popitem(last=True)", 1,
                       "the simulator evicts the most recent line"),
    "lru_no_refresh_on_hit": ("lru.py", "                    cache.move_to_end(ln)\n", "", 1,
                              "a hit does not refresh its line (FIFO, not LRU)"),
    "lru_row_trace_transposed": ("lru.py", "out.append((X, False, nb, tuple((_line(X, i * self.N + j), i) for i in rows)))",
                                 "out.append((X, False, nb, tuple((_line(X, j * self.M + i), i) for i in rows)))", 1,
                                 "the row loop's trace reads A column-major (coalesced)"),
    "lru_syrk_trace_aj_row": ("lru.py", 'out.append(("a_j", False, 4, tuple((_line("a", j * self.Mk + k), (i, j)) for i, j in th)))',
                              'out.append(("a_j", False, 4, tuple((_line("a", i * self.Mk + k), (i, j)) for i, j in th)))', 1,
                              "the SYRK trace reads row i for a_jk"),
    "lru_kmeans_trace_point_major": ("lru.py", 'ev.append(tuple((_line("F", f * self.ld + p), p) for p in pts))',
                                     'ev.append(tuple((_line("F", p * self.nf + f), p) for p in pts))', 1,
                                     "the KMEANS trace reads features point-major"),
    "lru_transpose_store_as_load": ("lru.py", 'out.append(("out", True, 4, tuple((_line("out", f * self.ld + p), p) for p in pts)))',
                                    'out.append(("out", False, 4, tuple((_line("out", f * self.ld + p), p) for p in pts)))', 1,
                                    "the KM transpose's store traced as a load"),
    # ---- the B200 rule oracle (oracle/b200_rule.py)
    "rule_floor_4": ("b200_rule.py", "min_warps_sm=8,", "min_warps_sm=4,", 1, "R18 floor of 4 warps instead of 8"),
    "rule_fewest_warps_first": ("b200_rule.py", "a, m = max(fitting, key=lambda am: (am[0] * am[1], am[0]))",
                                "a, m = min(fitting, key=lambda am: (am[0] * am[1], am[0]))", 1,
                                "Eq 9 takes the most throttled fitting pair"),
    "rule_no_stream_floor": ("b200_rule.py", "floor = -(-floor // S)", "floor = floor", 1, "R29 not applied"),
    "rule_retouch_2": ("b200_rule.py", "min_retouch=16,", "min_retouch=2,", 1, "R23 re-touch threshold 2 instead of 16"),
    "rule_stream_pct_50": ("b200_rule.py", "max_stream_pct=25,", "max_stream_pct=50,", 1, "R24 stream share 50 % instead of 25 %"),
    "rule_divergent_lines_2": ("b200_rule.py", "divergent_lines=8,", "divergent_lines=2,", 1,
                               "R18 divergence at 2 lines per request instead of 8"),
    "rule_shared_ignored": ("b200_rule.py", " and not (guards.get(\"private_streams\", 0) and inp.shared[i])", "", 1,
                            "R32 not applied (CTA-shared loads counted as streams)"),
    "exact_sum_drops_group": ("kmeans.py", "for ex in np.unique(e):", "for ex in np.unique(e)[1:]:", 1,
                              "the exact sum drops the smallest-exponent values"),
    "rule_stream_ignores_stores": ("b200_rule.py", "stream = sum(nbytes[i] for i in first if stored[i] or not reuse[i])",
                                   "stream = sum(nbytes[i] for i in first if not reuse[i])", 1,
                                   "R24's stream share leaves out the stores"),
    "rule_retouch_min": ("b200_rule.py", "retouch[instr] = max(retouch[instr], c)", "retouch[instr] = min(retouch[instr] or c, c)", 1,
                         "re-touches measured as the fewest, not the most, touches of a line"),
    # ---- the exact k-means update (oracle/kmeans.py)
    "round_ties_away": ("kmeans.py", "if rem > Fraction(1, 2) or (rem == Fraction(1, 2) and n % 2 == 1):",
                        "if rem >= Fraction(1, 2):", 1, "round half away from zero instead of to even"),
    "round_truncates": ("kmeans.py", "if rem > Fraction(1, 2) or (rem == Fraction(1, 2) and n % 2 == 1):",
                        "if False:", 1, "the centre is truncated, not rounded"),
    "empty_centre_zeroed": ("kmeans.py", "            continue                                           # empty centre keeps its value (R21)",
                            "            new[c, :] = 0.0\n            continue", 1, "an empty centre becomes 0"),
    "mean_divides_by_npoints": ("kmeans.py", "/ len(members))", "/ npoints)", 1, "the mean divides by all points"),
}


def run_mutant(name, jobs):
    fn, old, new, count, what = MUTANTS[name]
    with tempfile.TemporaryDirectory(prefix="orc_mut_") as tmp:
        dst = os.path.join(tmp, "oracle")
        shutil.copytree(os.path.join(ROOT, "oracle"), dst, ignore=shutil.ignore_patterns("liborc.so", "__pycache__"))
        p = os.path.join(dst, fn)
        src = open(p).read()
        n = src.count(old)
        if n == 0:
            return name, "NOT APPLIED", 0.0, what, ""
        src = src.replace(old, new) if count == 0 else src.replace(old, new, count)
        open(p, "w").write(src)
        env = dict(os.environ, PYTHONPATH=os.pathsep.join([tmp, ROOT]), PYTHONDONTWRITEBYTECODE="1")
        # build the copy's liborc.so once, before the test workers start (they
        # would otherwise race to compile it into the same file)
        b = subprocess.run([sys.executable, "-c", "import oracle; oracle.build()"], cwd=tmp, env=env,
                           capture_output=True, text=True)
        if b.returncode != 0:
            return name, "killed", 0.0, what, "does not compile"
        cmd = [sys.executable, "-m", "pytest", "-x", "-q", "-p", "no:cacheprovider", "-m", "not gpu",
               "--rootdir", ROOT] + (["-n", str(jobs)] if jobs > 1 else []) + [os.path.join(ROOT, t) for t in TESTS]
        t0 = time.time()
        out = subprocess.run(cmd, cwd=tmp, env=env, capture_output=True, text=True, timeout=1200)
        dt = time.time() - t0
        failed = [l.split(" ")[1] for l in out.stdout.splitlines() if l.startswith("FAILED ")]
        killer = failed[0].split("::", 1)[-1] if failed else ""
        if out.returncode == 0:
            return name, "SURVIVED", dt, what, ""
        if not failed:
            return name, f"ERROR rc={out.returncode}", dt, what, out.stdout[-300:].replace("\n", " ")
        return name, "killed", dt, what, killer


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--only", nargs="*")
    ap.add_argument("--jobs", type=int, default=8)
    ap.add_argument("--out")
    a = ap.parse_args()
    names = a.only or list(MUTANTS)
    lines = []
    for nm in names:
        r = run_mutant(nm, a.jobs)
        line = f"{r[1]:12s} {r[0]:30s} {r[2]:6.1f}s  {r[3]}" + (f"  [{r[4]}]" if r[4] else "")
        print(line, flush=True)
        lines.append((r, line))
    real = [(r, l) for r, l in lines if r[0] != "control_unchanged"]
    killed = sum(1 for r, _ in real if r[1] == "killed")
    control_ok = all(r[1] == "SURVIVED" for r, _ in lines if r[0] == "control_unchanged")
    summary = f"{killed}/{len(real)} mutants killed; control {'survived' if control_ok else 'FAILED'}"
    print(summary)
    if a.out:
        with open(a.out, "w") as f:
            f.write("Oracle mutation check (tools/oracle_mutants.py): each line is one plausible mistake typed into a\n"
                    "copy of oracle/; 'killed' = a -m 'not gpu' oracle test failed (the first failing test in brackets).\n\n")
            f.write("\n".join(l for _, l in lines) + "\n" + summary + "\n")
    return 0 if killed == len(real) and control_ok else 1


if __name__ == "__main__":
    sys.exit(main())
