#!/usr/bin/env python3
"""bench.py — the CATT hot path on B200, one JSON line.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--workload atax|bicg_mvt|kmeans|gesummv|syrk|atax256|...]
                    [--variant fused|fused_peer|coop|staged|vec4|literal] [--impl reference] [--no-l1]

A step is one pass of the whole hot path over one batch: the CATT analysis of
every loop (host, microseconds), then every loop of the workload launched with
its CATT throttle through the C ABI (catt_rows / catt_cols / catt_kmeans_assign
/ catt_syrk), plus the NCCL all-reduce of the A^T partials when N > 1.
Default workload = BASELINE.json configs[4], the largest configuration and the
scaling one: ATAX 65536 x 16384 fp32 (tmp = A x, y = A^T tmp), rows sharded
over the N ranks (16384 x 65536 / N rows each at N > 1), the A^T partials
all-reduced by NCCL (the only exchange the path has). At N = 1 it is the whole
4 GiB matrix on one B200. `--workload bicg_mvt` is configs[1] (BICG and MVT
4096 x 4096, weak-scaled over ranks).

After the timed region (N = 1): the throttle study of the workload's literal
loop (CATT pick, paper rule, full TLP, every swept (a, m)), and the L1 hit
rate and DRAM bytes of each pick from an ncu subprocess (the metric's other
half).

`value` = algorithmic bytes of the step (all ranks) / device time (max over
ranks), GB/s. L2 is flushed (256 MiB write) before every timed step.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "kernel runtime & L1 hit rate: CATT throttle vs full-TLP vs best swept, HBM GB/s"
# FP32 FMA throughput measured on this pool's B200 (tools/ffma_probe.cu, 1965 MHz):
# the ALU roofline reports its fraction beside the derived 148 x 128 x 2 x clock peak
FP32_MEASURED_TFLOPS = 72.3
FALLBACK_HBM_GBS = 6650.0


def log(*a):
    print(*a, file=sys.stderr, flush=True)


def parse():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=20)
    p.add_argument("--warmup", type=int, default=5)
    p.add_argument("--workload", default="atax",
                   choices=["bicg_mvt", "kmeans", "kmeans_iter", "gesummv", "syrk", "syr2k", "corr", "gemm", "atax256", "atax"])
    p.add_argument("--variant", default=None,
                   help="fused (default for bicg_mvt/atax), fused1, coop, staged, vec4, literal, regs (kmeans)")
    p.add_argument("--impl", default="catt", choices=["catt", "reference"])
    p.add_argument("--no-study", action="store_true", help="skip the throttle sweep")
    p.add_argument("--no-e2e", action="store_true")
    p.add_argument("--flush-order", default="flush_sleep", choices=["flush_sleep", "sleep_flush"],
                   help="order of the L2 flush and the enqueue-cover GPU sleep before each timed step")
    p.add_argument("--cpu-seconds", type=float, default=8.0, help="CPU-oracle sample budget")
    p.add_argument("--no-l1", action="store_true", help="skip the ncu L1-hit-rate pass over the study picks")
    p.add_argument("--l1-child", default=None, help=argparse.SUPPRESS)   # internal: the ncu-profiled launches
    return p.parse_args()


# ------------------------------------------------------------------ distributed plumbing
def dist_env():
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return world, rank, local


def peak_hbm():
    try:
        return float(json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"]), "measured"
    except Exception:
        return FALLBACK_HBM_GBS, "fallback"


class ClockSampler:
    """nvidia-smi clocks and throttle reasons sampled during the timed region."""

    FIELDS = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,"
              "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
              "clocks_event_reasons.sw_power_cap")

    def __init__(self, index):
        self.index, self.samples, self.proc = index, [], None

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.FIELDS}",
                                          "--format=csv,noheader,nounits", "-lms", "100"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.thread = threading.Thread(target=self._read, daemon=True)
            self.thread.start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            parts = [x.strip() for x in line.split(",")]
            if len(parts) >= 8:
                self.samples.append(parts)

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        time.sleep(0.25)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=2)
        except Exception:
            self.proc.kill()
        sms = []
        reasons = set()
        mx = None
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for s in self.samples:
            try:
                sms.append(float(s[0]))
                mx = float(s[1])
            except ValueError:
                continue
            for nm, v in zip(names, s[4:8]):
                if v.lower() == "active":
                    reasons.add(nm)
        return {"sm_mhz": statistics.median(sms) if sms else None, "sm_max_mhz": mx, "reasons": sorted(reasons),
                "samples": len(sms)}


# ------------------------------------------------------------------ workloads
class Loop:
    def __init__(self, name, fn, nbytes, kind, prob=None, launch=None, plans=None):
        self.name, self.fn, self.nbytes, self.kind = name, fn, nbytes, kind
        self.prob, self.launch = prob, launch
        self.plans = plans or [name]          # keys of Workload.plans behind this launch


class Workload:
    """Device arrays + the loops of one step (all launched through the C ABI)."""
    name = ""
    desc = ""
    variant = "coop"
    scaling = "weak"          # every rank's work is fixed as N grows (the JSON line's "scaling")
    parallelism = "independent problem per rank"   # how N > 1 splits the work (config.parallelism)

    def __init__(self, catt, torch, rank, world, variant):
        self.catt, self.torch, self.rank, self.world = catt, torch, rank, world
        self.variant = variant or self.variant
        self.hw = catt.hw_query()
        self.plans = {}

    def plan(self, key, prob, launch):
        """The CATT analysis (a1-a5) for one loop; returns the throttle to
        launch with. analysis_us = the median of 21 analyses (catt_plan: the
        kernel's attributes, the descriptor, Eq 1-9), first_us = the first
        (it also queries the device); the paper reports 1-2 s."""
        ts = []
        for _ in range(21):
            t0 = time.perf_counter()
            t, r = self.catt.plan(prob, launch, self.hw)
            ts.append(1e6 * (time.perf_counter() - t0))
        self.plans[key] = dict(throttle=[t.active_warps or r["base_warps"], t.active_ctas or r["base_ctas"]],
                               base=[r["base_warps"], r["base_ctas"]], flags=self.catt.FLAG_NAMES[r["flags"]],
                               footprint_lines=r["footprint_lines_full"], l1d_lines=r["l1d_bytes"] // 128,
                               carveout_kb=r["carveout_kb"], analysis_us=round(statistics.median(ts), 1),
                               analysis_first_us=round(ts[0], 1))
        return t

    def collective(self):
        pass

    def inputs(self):
        return []

    def outputs(self):
        return []


class BicgMvt(Workload):
    parallelism = "row-shard"
    name = "bicg_mvt"
    variant = "fused"
    desc = "BICG and MVT 4096x4096 fp32 row-per-thread (memory-divergent) on 1 B200 (BASELINE configs[1])"

    def __init__(self, catt, torch, rank, world, variant):
        super().__init__(catt, torch, rank, world, variant)
        import seeded_inputs as si
        n = 4096
        rows = n                                     # rows per rank (weak scaling)
        self.rows = rows
        dev = torch.device("cuda")
        T = lambda *s: torch.empty(*s, device=dev)
        self.Ab, self.Am = T(rows, n), T(rows, n)
        catt.fill_hash(self.Ab, si.SEED_BICG, offset=rank * rows * n)
        catt.fill_hash(self.Am, si.SEED_MVT, offset=rank * rows * n)
        self.p, self.r, self.y1, self.y2 = T(n), T(rows), T(n), T(rows)
        self.x1, self.x2, self.q, self.s = T(rows), T(n), T(rows), T(n)
        for k, v in enumerate((self.p, self.y1, self.x2)):
            catt.fill_hash(v, si.sub_seed(si.SEED_BICG, k + 1))
        for k, v in enumerate((self.r, self.y2, self.x1)):
            catt.fill_hash(v, si.sub_seed(si.SEED_MVT, k + 1), offset=rank * rows)
        var = self.variant
        mat = rows * n * 4
        acc2 = rank == 0                 # x2 = x2 + sum_g A_g^T y2_g: only rank 0 adds the initial x2
        P = catt.problem
        if var == "fused_peer":
            # the grouped single-read launch with s and x2 all-reduced inside
            # the kernel through peer memory: no NCCL
            # call; x2's initial value is replicated and added after the sum
            from paper_conf_icpp_kimhlsh19_b200 import dist as cdist
            self.desc = ("BICG and MVT 4096x4096 fp32 per rank, row-sharded, column partials all-reduced inside "
                         "the fused kernel through peer memory (configs[1] weak-scaled, SURVEY 8(f) f4)")
            self.peer = cdist.peer_setup(2 * n)
            group = [dict(A=self.Ab, xr=self.p, xc=self.r, yr=self.q, yc=self.s),
                     dict(A=self.Am, xr=self.y1, xc=self.y2, yr=self.x1, yc=self.x2, row_accumulate=True,
                          col_accumulate=True)]
            self.loops = [Loop("bicg+mvt fused + peer all-reduce", lambda: cdist.bicg_mvt_rowshard_peer(group, self.peer),
                               mat + 4 * 2 * (rows + n) + mat + 4 * (3 * rows + 3 * n), "fused")]
            self.study = None
            return
        if var in ("fused", "fused1"):
            # both loops of each application in one pass over A (A read once);
            # "fused" also groups BICG and MVT into one launch (one 128 MiB
            # stream instead of two 64 MiB ones), "fused1" is one launch each
            tf = self.plan("bicg fused", P(catt.K_BICG_2, m=rows, n=n), catt.Throttle(variant="fused"))
            tg = self.plan("mvt fused", P(catt.K_MVT_1, n=n), catt.Throttle(variant="fused"))
            bicg_b = mat + 4 * 2 * (rows + n)
            mvt_b = mat + 4 * (3 * rows + (3 if acc2 else 2) * n)
            if var == "fused":
                group = [dict(A=self.Ab, xr=self.p, xc=self.r, yr=self.q, yc=self.s),
                         dict(A=self.Am, xr=self.y1, xc=self.y2, yr=self.x1, yc=self.x2, row_accumulate=True,
                              col_accumulate=acc2)]
                self.loops = [Loop("bicg+mvt fused (one launch)", lambda: catt.dual_group(group, t=tf),
                                   bicg_b + mvt_b, "fused", plans=["bicg fused", "mvt fused"])]
            else:
                self.loops = [
                    Loop("bicg fused", lambda: catt.dual(self.Ab, self.p, self.q, self.s, xc=self.r, t=tf),
                         bicg_b, "fused"),
                    Loop("mvt fused", lambda: catt.dual(self.Am, self.y1, self.x1, self.x2, xc=self.y2,
                                                        row_accumulate=True, col_accumulate=acc2, t=tg),
                         mvt_b, "fused"),
                ]
            self.study = dict(name="bicg2 q=A p (literal, row per thread)", prob=P(catt.K_BICG_2, m=rows, n=n),
                              A=self.Ab, x=self.p, y=self.q,
                              launches=[(1024, 132), (1024, 196), (1024, 228), (256, 196), (256, 228)])
            self._app_study_setup(catt, P, rows, n)
            return
        self._app_study_setup(catt, P, rows, n)
        col_var = var if var in ("coop", "staged") else "literal"
        cta_row = {"coop": 256, "staged": 32, "vec4": 32, "literal": 32}[var]
        cta_col = {"coop": 1024, "staged": 32, "literal": 256}[col_var]
        P = catt.problem
        tb1 = self.plan("bicg1 s=A^T r", P(catt.K_BICG_1, m=rows, n=n), catt.Throttle(cta_threads=cta_col, variant=col_var))
        tb2 = self.plan("bicg2 q=A p", P(catt.K_BICG_2, m=rows, n=n), catt.Throttle(cta_threads=cta_row, variant=var))
        tm1 = self.plan("mvt1 x1+=A y1", P(catt.K_MVT_1, n=n), catt.Throttle(cta_threads=cta_row, variant=var))
        tm2 = self.plan("mvt2 x2+=A^T y2", P(catt.K_MVT_2, n=n), catt.Throttle(cta_threads=cta_col, variant=col_var))
        self.loops = [
            Loop("bicg1 s=A^T r", lambda: catt.cols(self.Ab, self.r, self.s, False, tb1), mat + 4 * (rows + n), "cols"),
            Loop("bicg2 q=A p", lambda: catt.rows(self.Ab, self.p, self.q, catt.ROWS_STORE, t=tb2), mat + 4 * (rows + n),
                 "rows"),
            Loop("mvt1 x1+=A y1", lambda: catt.rows(self.Am, self.y1, self.x1, catt.ROWS_ACCUM, t=tm1),
                 mat + 4 * (2 * rows + n), "rows"),
            Loop("mvt2 x2+=A^T y2", lambda: catt.cols(self.Am, self.y2, self.x2, acc2, tm2),
                 mat + 4 * (rows + (2 if acc2 else 1) * n), "cols"),
        ]
        self.study = dict(name="bicg2 q=A p (literal, row per thread)", prob=P(catt.K_BICG_2, m=rows, n=n),
                          A=self.Ab, x=self.p, y=self.q,
                          launches=[(1024, 132), (1024, 196), (1024, 228), (256, 196), (256, 228)])

    def _app_study_setup(self, catt, P, rows, n):
        """BICG's two literal loops for the per-application BFTT vs per-loop
        CATT comparison (P:7)."""
        self.app_study = dict(
            name="BICG (s = A^T r, q = A p), literal loops",
            loops=[(P(catt.K_BICG_1, m=rows, n=n), lambda th: catt.cols(self.Ab, self.r, self.s, False, th)),
                   (P(catt.K_BICG_2, m=rows, n=n), lambda th: catt.rows(self.Ab, self.p, self.q, catt.ROWS_STORE, t=th))],
            launches=[(1024, 196), (1024, 228), (1024, 132)])

    def collective(self):
        if self.world > 1 and self.variant != "fused_peer":   # fused_peer reduces inside its kernel
            import torch.distributed as dist
            dist.all_reduce(self.s)
            dist.all_reduce(self.x2)

    def step_bytes(self):
        n, rows = 4096, self.rows
        # BICG: A, p, r, q, s; MVT: A, y1, y2, x1 (in/out), x2 (in/out on rank 0)
        return 2 * rows * n * 4 + 4 * (n + rows + rows + n) + 4 * (n + rows + 2 * rows + 2 * n)

    def inputs(self):
        return [self.Ab, self.Am, self.p, self.r, self.y1, self.y2, self.x1, self.x2]

    def outputs(self):
        return [self.q, self.s, self.x1, self.x2]

    def cpu_oracle_step(self, oracle, host):
        oracle.bicg(host["Ab"], host["p"], host["r"])
        oracle.mvt(host["Am"], host["y1"], host["y2"], host["x1"], host["x2"])

    def host_copy(self):
        return {k: getattr(self, k).cpu().numpy() for k in ("Ab", "Am", "p", "r", "y1", "y2", "x1", "x2")}


class Kmeans(Workload):
    name = "kmeans"
    desc = "KMEANS assign step, Rodinia shape 494020 points x 34 features, k=5, feature-major (configs[2])"
    variant = "staged"

    def __init__(self, catt, torch, rank, world, variant):
        super().__init__(catt, torch, rank, world, variant)
        import seeded_inputs as si
        self.np_, self.nf, self.k, self.ld = 494020, 34, 5, 494020
        dev = torch.device("cuda")
        self.feat = torch.empty(self.nf * self.ld, device=dev)
        catt.fill_hash(self.feat, si.SEED_KMEANS + rank)
        self.clusters = self.feat.view(self.nf, self.ld)[:, : self.k].t().contiguous()
        self.memb = torch.empty(self.np_, dtype=torch.int32, device=dev)
        prob = catt.problem(catt.K_KMEANS, m=self.np_, n=self.nf, k=self.k, ld=self.ld)
        t = self.plan("kmeans assign", prob, catt.Throttle(cta_threads=256, variant=self.variant))
        nbytes = self.np_ * self.nf * 4 + self.np_ * 4 + self.k * self.nf * 4
        self.loops = [Loop("kmeans assign", lambda: catt.kmeans_assign(self.feat, self.ld, self.np_, self.nf,
                                                                         self.clusters, self.memb, t=t), nbytes, "kmeans")]
        self.study = dict(name="kmeans assign (literal, feature-major)", prob=prob, kmeans=True,
                          launches=[(256, 0), (256, 100), (256, 228)])

    def inputs(self):
        return [self.feat]

    def outputs(self):
        return [self.memb]

    def host_copy(self):
        return {"feat": self.feat.cpu().numpy(), "clusters": self.clusters.cpu().numpy()}

    def cpu_oracle_step(self, oracle, host):
        oracle.kmeans_assign(host["feat"], self.ld, self.np_, self.nf, host["clusters"])


class KmeansIter(Workload):
    parallelism = "point-shard"
    name = "kmeans_iter"
    desc = ("KMEANS full iteration (assign + exact centroid update), 494020 points x 34 features, k=5, "
            "feature-major, points sharded per rank (SURVEY 8(f) f2)")
    variant = "fused"

    def __init__(self, catt, torch, rank, world, variant):
        super().__init__(catt, torch, rank, world, variant)
        import seeded_inputs as si
        self.np_, self.nf, self.k, self.ld = 494020, 34, 5, 494020
        dev = torch.device("cuda")
        self.feat = torch.empty(self.nf * self.ld, device=dev)
        catt.fill_hash(self.feat, si.SEED_KMEANS, offset=rank * self.nf * self.ld)
        self.clusters = self.feat.view(self.nf, self.ld)[:, : self.k].t().contiguous()
        self.memb = torch.full((self.np_,), -1, dtype=torch.int32, device=dev)
        self.acc = torch.zeros(catt.kmeans_acc_words(self.k, self.nf), dtype=torch.int64, device=dev)
        nbytes = self.np_ * self.nf * 4 + 8 * self.np_ + self.k * self.nf * 4
        if world == 1:                   # one launch: the last CTA rounds the centres (catt_kmeans_step)
            self.loops = [Loop("kmeans iteration (one launch)", lambda: catt.kmeans_step(
                                   self.feat, self.ld, self.np_, self.nf, self.clusters, self.memb, self.acc),
                               nbytes + self.k * self.nf * 4, "kmeans_acc")]
        else:                            # the iteration's one exchange: integer sums, between the two kernels
            import torch.distributed as dist
            self.loops = [Loop("kmeans assign+sums", lambda: catt.kmeans_accumulate(
                                   self.feat, self.ld, self.np_, self.nf, self.clusters, self.memb, self.acc),
                               nbytes, "kmeans_acc"),
                          Loop("kmeans all-reduce of the sums", lambda: dist.all_reduce(self.acc),
                               self.acc.numel() * 8, "collective"),
                          Loop("kmeans finalize", lambda: catt.kmeans_finalize(self.acc, self.clusters),
                               self.acc.numel() * 8 * 2 + self.k * self.nf * 4, "kmeans_fin")]
        # the KM transpose loop (Rodinia invert_mapping), CATT-planned and studied
        self.pm = torch.empty(self.np_ * self.nf, device=dev)
        catt.fill_hash(self.pm, si.sub_seed(si.SEED_KMEANS, 3))
        self.fm = torch.empty(self.nf * self.ld, device=dev)
        probt = catt.problem(catt.K_KMEANS_T, m=self.np_, n=self.nf, ld=self.ld)
        self.plan("kmeans transpose (literal)", probt, catt.Throttle(cta_threads=256))
        self.study = dict(name="kmeans transpose (literal, point-major -> feature-major)", prob=probt,
                          launches=[(256, 0), (256, 228), (1024, 196)], reps=3,
                          fn=lambda th: (lambda: catt.kmeans_transpose(self.pm, self.np_, self.nf, self.fm, self.ld,
                                                                       t=th)))

    def step_bytes(self):
        return self.np_ * self.nf * 4 + 8 * self.np_

    def inputs(self):
        return [self.feat]

    def outputs(self):
        return [self.memb, self.clusters]

    def host_copy(self):
        return {"feat": self.feat.cpu().numpy(), "clusters": self.clusters.cpu().numpy()}

    def cpu_oracle_step(self, oracle, host):
        from oracle import kmeans as okm
        memb, _ = oracle.kmeans_assign(host["feat"], self.ld, self.np_, self.nf, host["clusters"])
        okm.update(host["feat"], self.ld, self.np_, self.nf, memb, host["clusters"])


class Gesummv(Workload):
    parallelism = "row-shard"
    name = "gesummv"
    desc = "GESUMMV 8192 fp32 (configs[3])"

    def __init__(self, catt, torch, rank, world, variant):
        super().__init__(catt, torch, rank, world, variant)
        import seeded_inputs as si
        n = 8192
        dev = torch.device("cuda")
        self.A, self.B = torch.empty(n, n, device=dev), torch.empty(n, n, device=dev)
        catt.fill_hash(self.A, si.SEED_GESUMMV, offset=rank * n * n)
        catt.fill_hash(self.B, si.sub_seed(si.SEED_GESUMMV, 1), offset=rank * n * n)
        self.x = torch.empty(n, device=dev)
        catt.fill_hash(self.x, si.sub_seed(si.SEED_GESUMMV, 2))
        self.y, self.tmp = torch.empty(n, device=dev), torch.empty(n, device=dev)
        t = self.plan("gesummv", catt.problem(catt.K_GESUMMV, n=n),
                      catt.Throttle(cta_threads=256 if self.variant == "coop" else 64, variant=self.variant))
        self.loops = [Loop("gesummv", lambda: catt.rows(self.A, self.x, self.y, catt.ROWS_GESUMMV, self.B, self.tmp,
                                                         1.5, 1.2, t), 2 * n * n * 4 + 12 * n, "rows")]
        self.study = dict(name="gesummv (literal, row per thread)", prob=catt.problem(catt.K_GESUMMV, n=n),
                          gesummv=True, launches=[(1024, 0), (1024, 196), (256, 196), (256, 228),
                                                  # CTA- vs warp-level on SM partitions (SURVEY 8(d) [3]):
                                                  # 32 CTAs on 8 SMs = 4 per SM, on 16 SMs = 2 per SM
                                                  (256, 8, 8), (256, 196, 8), (256, 228, 8), (256, 228, 16)])

    def inputs(self):
        return [self.A, self.B, self.x]

    def outputs(self):
        return [self.y, self.tmp]

    def host_copy(self):
        return {k: getattr(self, k).cpu().numpy() for k in ("A", "B", "x")}

    def cpu_oracle_step(self, oracle, host):
        oracle.gesummv(host["A"], host["B"], host["x"], 1.5, 1.2)


class Syrk(Workload):
    name = "syrk"
    desc = "SYRK 2048 fp32 (configs[3])"
    variant = "staged"

    def __init__(self, catt, torch, rank, world, variant):
        super().__init__(catt, torch, rank, world, variant)
        import seeded_inputs as si
        n = 2048
        dev = torch.device("cuda")
        self.A, self.C = torch.empty(n, n, device=dev), torch.empty(n, n, device=dev)
        catt.fill_hash(self.A, si.SEED_SYRK + rank)
        catt.fill_hash(self.C, si.sub_seed(si.SEED_SYRK, 1) + rank)
        t = self.plan("syrk", catt.problem(catt.K_SYRK, n=n, k=n), catt.Throttle(variant=self.variant))
        self.flops = 2 * n * n * n
        self.loops = [Loop("syrk", lambda: catt.syrk(self.A, self.C, 1.5, 1.2, t=t), 3 * n * n * 4, "syrk")]
        # SURVEY 8(d) [3]: the discriminating experiment. Paper mode predicts a
        # throttle at the 8 KB carveout, union mode none; the measurement decides.
        Cs = self.C.clone()
        self.study = dict(name="syrk (literal, 2-D block 32 x 8)", prob=catt.problem(catt.K_SYRK, n=n, k=n),
                          launches=[(256, 8), (256, 100), (256, 228)], reps=2,
                          fn=lambda th: (lambda: catt.syrk(self.A, Cs, 1.5, 1.2, t=th)))

    def inputs(self):
        return [self.A, self.C]

    def outputs(self):
        return [self.C]

    def host_copy(self):
        return {k: getattr(self, k).cpu().numpy() for k in ("A", "C")}

    def cpu_oracle_step(self, oracle, host):
        import numpy as np
        oracle.syrk_rows(host["A"], host["C"], 1.5, 1.2, np.arange(16))


class Syr2k(Workload):
    name = "syr2k"
    desc = "SYR2K 2048 fp32 (Table 2 P:77 size; SURVEY 8(f) f3)"
    variant = "staged"

    def __init__(self, catt, torch, rank, world, variant):
        super().__init__(catt, torch, rank, world, variant)
        import seeded_inputs as si
        n = 2048
        dev = torch.device("cuda")
        self.A, self.B, self.C = (torch.empty(n, n, device=dev) for _ in range(3))
        catt.fill_hash(self.A, si.SEED_SYR2K + rank)
        catt.fill_hash(self.B, si.sub_seed(si.SEED_SYR2K, 1) + rank)
        catt.fill_hash(self.C, si.sub_seed(si.SEED_SYR2K, 2) + rank)
        t = self.plan("syr2k", catt.problem(catt.K_SYR2K, n=n, k=n), catt.Throttle(variant=self.variant))
        self.flops = 4 * n * n * n
        self.loops = [Loop("syr2k", lambda: catt.syr2k(self.A, self.B, self.C, 1.5, 1.2, t=t), 4 * n * n * 4, "syr2k")]
        Cs = self.C.clone()
        self.study = dict(name="syr2k (literal, 2-D block 32 x 8)", prob=catt.problem(catt.K_SYR2K, n=n, k=n),
                          launches=[(256, 228), (256, 100)], reps=2,
                          fn=lambda th: (lambda: catt.syr2k(self.A, self.B, Cs, 1.5, 1.2, t=th)))

    def inputs(self):
        return [self.A, self.B, self.C]

    def outputs(self):
        return [self.C]

    def host_copy(self):
        return {k: getattr(self, k).cpu().numpy() for k in ("A", "B", "C")}

    def cpu_oracle_step(self, oracle, host):
        import numpy as np
        oracle.syr2k_rows(host["A"], host["B"], host["C"], 1.5, 1.2, np.arange(16))


class Corr(Workload):
    name = "corr"
    desc = "CORR 2048 x 2048 fp32 (Table 2 P:81; the give-up case of P:395; SURVEY 8(f) f3)"
    variant = "staged"

    def __init__(self, catt, torch, rank, world, variant):
        super().__init__(catt, torch, rank, world, variant)
        import seeded_inputs as si
        n = m = 2048
        self.n, self.m = n, m
        dev = torch.device("cuda")
        self.data = torch.empty(n, m, device=dev)
        catt.fill_hash(self.data, si.SEED_CORR + rank)
        self.mean, self.std = torch.empty(m, device=dev), torch.empty(m, device=dev)
        self.sym = torch.empty(m, m, device=dev)
        self.work = torch.empty(n * m, device=dev)
        prob = catt.problem(catt.K_CORR, n=m, k=n)
        t = self.plan("corr", prob, catt.Throttle(variant=self.variant))
        self.flops = m * m * n                               # the symmetric half, 2 flop per fmaf
        self.loops = [Loop("corr", lambda: catt.corr(self.data, self.mean, self.std, self.sym, self.work, t=t),
                           n * m * 4 * 2 + m * m * 4, "corr")]
        d2 = self.data.clone()
        self.study = dict(name="corr loop (literal, thread per column j1)", prob=prob,
                          launches=[(256, 8), (256, 228)], reps=2,
                          fn=lambda th: (lambda: catt.corr(d2, self.mean, self.std, self.sym, t=th)))

    def inputs(self):
        return [self.data]

    def outputs(self):
        return [self.sym]

    def host_copy(self):
        return {"data": self.data.cpu().numpy()[:256, :256].copy()}

    def cpu_oracle_step(self, oracle, host):
        oracle.corr(host["data"])


class Gemm(Workload):
    name = "gemm"
    desc = "GEMM 512 x 512 fp32 (Table 2 CI group: the cache-insensitive negative control, P:397)"
    variant = "staged"

    def __init__(self, catt, torch, rank, world, variant):
        super().__init__(catt, torch, rank, world, variant)
        import seeded_inputs as si
        n = 512
        dev = torch.device("cuda")
        self.A, self.B, self.C = (torch.empty(n, n, device=dev) for _ in range(3))
        for q, x in enumerate((self.A, self.B, self.C)):
            catt.fill_hash(x, si.sub_seed(si.SEED_GEMM, q) + rank)
        prob = catt.problem(catt.K_GEMM, m=n, n=n, k=n)
        t = self.plan("gemm", prob, catt.Throttle(variant=self.variant))
        self.flops = 2 * n * n * n
        self.loops = [Loop("gemm", lambda: catt.gemm(self.A, self.B, self.C, 1.5, 1.2, t=t), 4 * n * n * 4, "gemm")]
        Cs = self.C.clone()
        self.study = dict(name="gemm (literal, 2-D block 32 x 8)", prob=prob,
                          launches=[(256, 8), (256, 228), (1024, 196)], reps=3,
                          fn=lambda th: (lambda: catt.gemm(self.A, self.B, Cs, 1.5, 1.2, t=th)))

    def inputs(self):
        return [self.A, self.B, self.C]

    def outputs(self):
        return [self.C]

    def host_copy(self):
        return {k: getattr(self, k).cpu().numpy() for k in ("A", "B", "C")}

    def cpu_oracle_step(self, oracle, host):
        oracle.gemm(host["A"], host["B"], host["C"], 1.5, 1.2)


class Atax(Workload):
    parallelism = "row-shard"
    name = "atax"
    variant = "fused"
    desc = "ATAX 65536x16384 fp32 row-sharded with NCCL all-reduce of A^T partials (configs[4])"

    def __init__(self, catt, torch, rank, world, variant, m=65536, n=16384):
        super().__init__(catt, torch, rank, world, variant)
        import seeded_inputs as si
        rows = m // world if m >= 1024 else m          # configs[4]: the global matrix is split across ranks
        self.scaling = "strong" if m >= 1024 else "weak"  # the 65536 x 16384 total is fixed as N grows
        self.m, self.n, self.rows = m, n, rows
        dev = torch.device("cuda")
        seed = si.SEED_ATAX_SHARDED if m >= 1024 else si.SEED_ATAX
        self.A = torch.empty(rows, n, device=dev)
        catt.fill_hash(self.A, seed, offset=rank * rows * n)
        self.x = torch.empty(n, device=dev)
        catt.fill_hash(self.x, si.sub_seed(seed, 1))
        self.tmp, self.y = torch.empty(rows, device=dev), torch.empty(n, device=dev)
        var = self.variant
        mat = rows * n * 4
        self.study = dict(name="atax1 tmp=A x (literal, row per thread)", prob=catt.problem(catt.K_ATAX_1, m=rows, n=n),
                          A=self.A, x=self.x, y=self.tmp, launches=[(256, 228), (256, 196), (1024, 196)])
        # both loops in one kernel, a throttle per loop
        self.kernel_study = dict(m=4096, n=4096, launches=[(1024, 196), (1024, 228), (512, 196)])
        if var == "fused_peer":
            # the A^T partials all-reduced inside the fused kernel through peer
            # memory: no NCCL call, one launch per step
            from paper_conf_icpp_kimhlsh19_b200 import dist as cdist
            self.desc = ("ATAX 65536x16384 fp32 row-sharded, A^T partials all-reduced inside the fused kernel "
                         "through peer memory (configs[4], SURVEY 8(f) f4)")
            self.peer = cdist.peer_setup(n)
            self.loops = [Loop("atax fused + peer all-reduce",
                               lambda: cdist.atax_rowshard_peer(self.A, self.x, self.peer, self.tmp, self.y),
                               mat + 4 * 2 * (rows + n), "fused")]
            return
        if var == "fused":
            tf = self.plan("atax fused", catt.problem(catt.K_ATAX_1, m=rows, n=n), catt.Throttle(variant="fused"))
            self.loops = [Loop("atax fused", lambda: catt.dual(self.A, self.x, self.tmp, self.y, dependent=True, t=tf),
                               mat + 4 * 2 * (rows + n), "fused")]
            return
        t1 = self.plan("atax1 tmp=A x", catt.problem(catt.K_ATAX_1, m=rows, n=n),
                       catt.Throttle(cta_threads=256 if var == "coop" else 32, variant=var))
        cv = var if var in ("coop", "staged") else "literal"
        t2 = self.plan("atax2 y=A^T tmp", catt.problem(catt.K_ATAX_2, m=rows, n=n),
                       catt.Throttle(cta_threads={"coop": 1024, "staged": 32, "literal": 256}[cv], variant=cv))
        self.loops = [Loop("atax1 tmp=A x", lambda: catt.rows(self.A, self.x, self.tmp, catt.ROWS_STORE, t=t1),
                           mat + 4 * (rows + n), "rows"),
                      Loop("atax2 y=A^T tmp", lambda: catt.cols(self.A, self.tmp, self.y, False, t2),
                           mat + 4 * (rows + n), "cols")]

    def collective(self):
        if self.world > 1 and self.variant != "fused_peer":   # fused_peer reduces inside its kernel
            import torch.distributed as dist
            dist.all_reduce(self.y)

    def step_bytes(self):
        # A once, x, tmp, y
        return self.rows * self.n * 4 + 4 * (2 * self.n + self.rows)

    def inputs(self):
        return [self.A, self.x]

    def outputs(self):
        return [self.tmp, self.y]

    def host_copy(self):
        return {k: getattr(self, k).cpu().numpy() for k in ("A", "x")}

    def cpu_oracle_step(self, oracle, host):
        oracle.atax(host["A"][: min(self.rows, 8192)], host["x"])


class Atax256(Atax):
    name = "atax256"
    desc = "ATAX N=M=256 fp32 (configs[0])"

    def __init__(self, catt, torch, rank, world, variant):
        super().__init__(catt, torch, rank, world, variant, m=256, n=256)


WORKLOADS = {"bicg_mvt": BicgMvt, "kmeans": Kmeans, "kmeans_iter": KmeansIter, "gesummv": Gesummv, "syrk": Syrk, "syr2k": Syr2k,
             "corr": Corr, "gemm": Gemm, "atax256": Atax256,
             "atax": Atax}


# ------------------------------------------------------------------ measurement
def time_loops(torch, w, flush, steps, warmup, barrier):
    """Per step: flush L2, then events around every loop (and the collective)."""
    st = torch.cuda.current_stream()
    n = len(w.loops)
    for _ in range(warmup):
        flush()
        for lp in w.loops:
            lp.fn()
        w.collective()
    torch.cuda.synchronize()
    barrier()
    torch.cuda.synchronize()
    per_loop = [[] for _ in range(n)]
    coll, steps_ms = [], []
    evs = []
    for _ in range(steps):
        flush()
        e = [torch.cuda.Event(enable_timing=True) for _ in range(n + 2)]
        e[0].record(st)
        for i, lp in enumerate(w.loops):
            lp.fn()
            e[i + 1].record(st)
        w.collective()
        e[n + 1].record(st)
        evs.append(e)
    torch.cuda.synchronize()
    barrier()
    for e in evs:
        for i in range(n):
            per_loop[i].append(e[i].elapsed_time(e[i + 1]))
        coll.append(e[n].elapsed_time(e[n + 1]))
        steps_ms.append(e[0].elapsed_time(e[n + 1]))
    return steps_ms, per_loop, coll


def study_fn(catt, w, th):
    """The study loop of workload w launched with throttle th (a callable)."""
    S = w.study
    if S.get("fn"):
        return S["fn"](th)
    if S.get("kmeans"):
        return lambda: catt.kmeans_assign(w.feat, w.ld, w.np_, w.nf, w.clusters, w.memb, t=th)
    if S.get("gesummv"):
        return lambda: catt.rows(w.A, w.x, w.y, catt.ROWS_GESUMMV, w.B, w.tmp, 1.5, 1.2, th)
    return lambda: catt.rows(S["A"], S["x"], S["y"], catt.ROWS_STORE, t=th)


def throttle_study(catt, torch, w, flush):
    """CATT's pick vs full TLP vs the exhaustively swept best static throttle
    for the paper's literal loop at launches where the union model says the
    L1D is contended (Fig 9)."""
    if not w.study:
        return None
    hw = w.hw

    def med(fn, reps=5):
        ts = []
        for _ in range(reps + 1):
            flush()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record()
            fn()
            b.record()
            torch.cuda.synchronize()
            ts.append(a.elapsed_time(b))
        ts = sorted(ts[1:])
        return ts[len(ts) // 2]

    out = []
    S = w.study
    parts = {}
    import contextlib
    for spec in S["launches"]:
        cta, carve = spec[0], spec[1]
        # a third entry: run on an SM partition of that many SMs (green
        # context), planned with num_sms = the partition's SM count
        sms = spec[2] if len(spec) > 2 else 0
        if sms and sms not in parts:
            parts[sms] = catt.SmPartition(sms)
        part = parts.get(sms)
        hw_l = part.hw(hw) if part else hw
        with (torch.cuda.stream(part.stream) if part else contextlib.nullcontext()):
            row = _study_launch(catt, w, S, cta, carve, hw_l, med)
        if part:
            row["sm_partition"] = part.sms
        out.append(row)
    for p in parts.values():
        p.close()
    return out


def _study_launch(catt, w, S, cta, carve, hw, med):
    paper_hw = catt.paper_rule(hw)
    launch = catt.Throttle(cta_threads=cta, carveout_kb=carve, variant="literal")
    ts = []
    for _ in range(11):                                   # the analysis' latency (1-2 s per application)
        t0 = time.perf_counter()
        t, r = catt.plan(S["prob"], launch, hw)           # B200 rule (guards on)
        ts.append(1e6 * (time.perf_counter() - t0))
    tp, rp = catt.plan(S["prob"], launch, paper_hw)       # the paper's Eq 9 rule
    W, T = r["base_warps"], r["base_ctas"]
    cands = []
    for a in [d for d in range(W, 0, -1) if W % d == 0]:
        for m in range(T, 0, -1):
            cands.append((a, m))
    times = {}
    for a, m in cands:
        th = launch.copy(active_warps=a, active_ctas=m if m < T else 0)
        times[(a, m)] = med(study_fn(catt, w, th), S.get("reps", 5))
    pick = (t.active_warps or W, t.active_ctas or T)
    pick_p = (tp.active_warps or W, tp.active_ctas or T)
    best = min(times, key=times.get)
    # the bypass alternative: the same literal row loop with L2-only
    # matrix loads at full TLP (row-loop studies only)
    byp = None
    if not S.get("fn") and not S.get("kmeans"):
        byp = med(study_fn(catt, w, launch.copy(variant=catt.VAR_BYPASS)), S.get("reps", 5))
    return dict(loop=S["name"], cta_threads=cta, carveout_kb=r["carveout_kb"], base=[W, T],
                    analysis_us=round(statistics.median(ts), 1),
                    footprint_lines=r["footprint_lines_full"], l1d_lines=r["l1d_bytes"] // 128,
                    contended=rp["flags"] != catt.FIT_NONE_NEEDED,
                    catt=list(pick), catt_rule=catt.FLAG_NAMES.get(r["flags"], r["flags"]),
                    catt_ms=round(times[pick], 4),
                    catt_paper=list(pick_p), catt_paper_ms=round(times[pick_p], 4),
                    full_ms=round(times[(W, T)], 4), best=list(best), best_ms=round(times[best], 4),
                    catt_over_best=round(times[pick] / times[best], 3),
                    catt_over_full=round(times[pick] / times[(W, T)], 3),
                    paper_over_best=round(times[pick_p] / times[best], 3),
                    bypass_ms=round(byp, 4) if byp is not None else None,
                    bypass_over_best=round(byp / times[best], 3) if byp is not None else None,
                    swept={f"{a},{m}": round(v, 4) for (a, m), v in times.items()})


def app_study(catt, torch, w, flush):
    """Per-loop CATT vs per-application BFTT (the paper's comparison, P:377,
    P:395): BFTT applies one static (a, m) to every loop of the application
    (the best such setting for the sum); CATT picks each loop's throttle."""
    S = getattr(w, "app_study", None)
    if not S:
        return None

    def med(fn, reps=3):
        ts = []
        for _ in range(reps + 1):
            flush()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record()
            fn()
            b.record()
            torch.cuda.synchronize()
            ts.append(a.elapsed_time(b))
        ts = sorted(ts[1:])
        return ts[len(ts) // 2]

    out = []
    paper_hw = catt.paper_rule(w.hw)
    for cta, carve in S["launches"]:
        launch = catt.Throttle(cta_threads=cta, carveout_kb=carve, variant="literal")
        per_loop, picks, picks_p = [], [], []
        for prob, mk in S["loops"]:
            t, r = catt.plan(prob, launch, w.hw)
            tp, rp = catt.plan(prob, launch, paper_hw)
            W, T = r["base_warps"], r["base_ctas"]
            times = {}
            for a in [d for d in range(W, 0, -1) if W % d == 0]:
                for m in range(T, 0, -1):
                    times[(a, m)] = med(lambda a=a, m=m: mk(launch.copy(active_warps=a, active_ctas=m if m < T else 0)))
            per_loop.append(times)
            picks.append((t.active_warps or W, t.active_ctas or T))
            picks_p.append((tp.active_warps or W, tp.active_ctas or T))
        common = set(per_loop[0])
        for tms in per_loop[1:]:
            common &= set(tms)
        bftt = min(common, key=lambda am: sum(tms[am] for tms in per_loop))
        bftt_ms = sum(tms[bftt] for tms in per_loop)
        catt_ms = sum(tms[pk] for tms, pk in zip(per_loop, picks))
        paper_ms = sum(tms[pk] for tms, pk in zip(per_loop, picks_p))
        full = [max(tms) for tms in per_loop]
        full_ms = sum(tms[f] for tms, f in zip(per_loop, full))
        out.append(dict(application=S["name"], cta_threads=cta, carveout_kb=carve,
                        catt_picks=[list(p) for p in picks], catt_ms=round(catt_ms, 4),
                        paper_picks=[list(p) for p in picks_p], paper_ms=round(paper_ms, 4),
                        bftt=list(bftt), bftt_ms=round(bftt_ms, 4), full_ms=round(full_ms, 4),
                        catt_speedup_over_bftt=round(bftt_ms / catt_ms, 4),
                        paper_speedup_over_bftt=round(bftt_ms / paper_ms, 4),
                        catt_speedup_over_full=round(full_ms / catt_ms, 4)))
    return out


def kernel_study(catt, torch, w, flush):
    """Per-loop throttles inside ONE kernel: ATAX's two literal
    loops in one cooperative kernel (catt_atax_onekernel). CATT gives each
    loop its own warp gate (a1, a2) and the kernel one CTA cap m (the
    tighter of the loops' caps); BFTT is the best single (a, m) for both
    loops; the sweep covers every (a1, a2, m)."""
    S = getattr(w, "kernel_study", None)
    if not S:
        return None
    import seeded_inputs as si
    mm, nn = S["m"], S["n"]
    A = torch.empty(mm, nn, device="cuda")
    catt.fill_hash(A, si.SEED_ATAX, offset=0)
    x = torch.empty(nn, device="cuda")
    catt.fill_hash(x, si.sub_seed(si.SEED_ATAX, 1))
    tmp, y = torch.empty(mm, device="cuda"), torch.empty(nn, device="cuda")

    def med(fn, reps=3):
        ts = []
        for _ in range(reps + 1):
            flush()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record()
            fn()
            b.record()
            torch.cuda.synchronize()
            ts.append(a.elapsed_time(b))
        ts = sorted(ts[1:])
        return ts[len(ts) // 2]

    out = []
    P = catt.problem
    for cta, carve in S["launches"]:
        launch = catt.Throttle(cta_threads=cta, carveout_kb=carve, variant="literal")
        t1, r1 = catt.plan(P(catt.K_ATAX_1, m=mm, n=nn), launch, w.hw)
        t2, r2 = catt.plan(P(catt.K_ATAX_2, m=mm, n=nn), launch, w.hw)
        W = cta // 32
        T = min(r1["base_ctas"], r2["base_ctas"])
        divs = [d for d in range(W, 0, -1) if W % d == 0]
        times = {}
        for m in range(T, 0, -1):
            for a1 in divs:
                for a2 in divs:
                    k1 = launch.copy(active_warps=a1, active_ctas=m if m < T else 0)
                    k2 = catt.Throttle(active_warps=a2, active_ctas=m if m < T else 0)
                    times[(a1, a2, m)] = med(lambda k1=k1, k2=k2: catt.atax_onekernel(A, x, tmp, y, k1=k1, k2=k2))
        pick = (t1.active_warps or W, t2.active_warps or W, min(t1.active_ctas or T, t2.active_ctas or T))
        bftt = min(((a, a, m) for a in divs for m in range(1, T + 1)), key=lambda k: times[k])
        best = min(times, key=times.get)
        full = (W, W, T)
        out.append(dict(kernel=f"ATAX {mm}x{nn}, both literal loops in one kernel", cta_threads=cta, carveout_kb=carve,
                        catt=list(pick), catt_ms=round(times[pick], 4), bftt=list(bftt), bftt_ms=round(times[bftt], 4),
                        full_ms=round(times[full], 4), best=list(best), best_ms=round(times[best], 4),
                        catt_speedup_over_bftt=round(times[bftt] / times[pick], 4),
                        catt_speedup_over_full=round(times[full] / times[pick], 4),
                        catt_over_best=round(times[pick] / times[best], 4),
                        swept={f"{a1},{a2},{m}": round(v, 4) for (a1, a2, m), v in times.items()}))
    return out


NCU_L1_METRICS = ("l1tex__t_sector_hit_rate.pct", "dram__bytes_read.sum", "dram__bytes_write.sum",
                  "gpu__time_duration.sum")


def l1_spec(study):
    """The launches the ncu pass profiles: each study row's CATT pick, paper
    pick, full TLP and best swept throttle (duplicates once)."""
    spec = []
    for i, row in enumerate(study or []):
        if row.get("sm_partition"):
            continue                          # ncu cannot profile a green-context launch
        roles = {}
        for role, am in (("catt", row["catt"]), ("paper", row["catt_paper"]), ("full", row["base"]),
                         ("best", row["best"])):
            roles.setdefault(tuple(am), []).append(role)
        for (a, m), rl in roles.items():
            spec.append(dict(row=i, cta=row["cta_threads"], carve=row["carveout_kb"], a=a, m=m, T=row["base"][1],
                             roles=rl))
    return spec


def l1_child(args, catt, torch, w):
    """--l1-child: launch the study loop once per spec entry between
    cudaProfilerStart/Stop (ncu --profile-from-start off sees only these)."""
    spec = json.loads(args.l1_child)
    fns = []
    for e in spec:
        th = catt.Throttle(cta_threads=e["cta"], carveout_kb=e["carve"], variant="literal", active_warps=e["a"],
                           active_ctas=e["m"] if e["m"] < e["T"] else 0)
        fns.append(study_fn(catt, w, th))
    torch.cuda.synchronize()
    torch.cuda.profiler.start()
    for f in fns:
        f()
    torch.cuda.synchronize()
    torch.cuda.profiler.stop()
    return 0


def l1_pass(args, study):
    """The L1 half of the metric (Fig 6): ncu's L1 sector hit
    rate, DRAM bytes and duration of the study loop at each pick, one cold
    launch each (ncu flushes the caches before every profiled kernel), in a
    subprocess after the timed region. Adds row["l1"][role] to the study rows."""
    import csv
    import io
    import shutil
    spec = l1_spec(study)
    ncu = shutil.which("ncu") or "/usr/local/cuda/bin/ncu"
    if not spec or not os.path.exists(ncu):
        return {"status": "skipped", "why": "no study launches" if not spec else "ncu not found"}
    cmd = [ncu, "--profile-from-start", "off", "--metrics", ",".join(NCU_L1_METRICS), "--csv", "--print-units", "base",
           sys.executable, os.path.join(ROOT, "bench.py"), "--workload", args.workload, "--l1-child", json.dumps(spec)]
    if args.variant:
        cmd += ["--variant", args.variant]
    t0 = time.perf_counter()
    try:
        out = subprocess.run(cmd, capture_output=True, text=True, timeout=600, cwd=ROOT)
    except Exception as ex:                   # pragma: no cover
        return {"status": "failed", "why": str(ex)[:200]}
    rows = [r for r in csv.reader(io.StringIO("\n".join(l for l in out.stdout.splitlines() if l.startswith('"'))))]
    if not rows:
        return {"status": "failed", "rc": out.returncode, "why": (out.stderr or out.stdout)[-300:]}
    head = rows[0]
    ci = {k: head.index(k) for k in ("ID", "Kernel Name", "Metric Name", "Metric Value")}
    per = {}
    for r in rows[1:]:
        per.setdefault(int(r[ci["ID"]]), {})[r[ci["Metric Name"]]] = float(r[ci["Metric Value"]].replace(",", ""))
    ids = sorted(per)
    if len(ids) != len(spec):
        return {"status": "failed", "why": f"{len(ids)} profiled kernels for {len(spec)} launches"}
    for e, k in zip(spec, ids):
        m = per[k]
        res = {"throttle": [e["a"], e["m"]], "l1_hit_pct": round(m["l1tex__t_sector_hit_rate.pct"], 2),
               "dram_bytes": int(m["dram__bytes_read.sum"] + m["dram__bytes_write.sum"]),
               "ncu_us": round(m["gpu__time_duration.sum"] / 1e3, 1)}
        for role in e["roles"]:
            study[e["row"]].setdefault("l1", {})[role] = res
    return {"status": "ok", "launches": len(spec), "seconds": round(time.perf_counter() - t0, 1),
            "metrics": list(NCU_L1_METRICS), "cache_control": "all (ncu default: caches flushed before each kernel)"}


def ncu_traffic(workload):
    """DRAM bytes per launch of the workload's dominant kernel from the committed ncu summary."""
    path = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    try:
        return json.load(open(path)).get(workload)
    except Exception:
        return None


def run_reference(args):
    """--impl reference: the CPU oracle (as it stands) on this box's host cores."""
    world, rank, _ = dist_env()
    if rank != 0:
        return 0
    import numpy as np
    import oracle
    import seeded_inputs as si
    if world > 1:            # torchrun exports OMP_NUM_THREADS=1; rank 0 alone runs, on every host core
        oracle.set_num_threads(os.cpu_count() or 1)
    wl = args.workload
    t0 = time.perf_counter()
    if wl == "bicg_mvt":
        n = 4096
        host = {"Ab": oracle.fill(si.SEED_BICG, n * n).reshape(n, n), "Am": oracle.fill(si.SEED_MVT, n * n).reshape(n, n)}
        for k, nm in enumerate(("p", "y1", "x2")):
            host[nm] = oracle.fill(si.sub_seed(si.SEED_BICG, k + 1), n)
        for k, nm in enumerate(("r", "y2", "x1")):
            host[nm] = oracle.fill(si.sub_seed(si.SEED_MVT, k + 1), n)
        step = lambda: (oracle.bicg(host["Ab"], host["p"], host["r"]),
                        oracle.mvt(host["Am"], host["y1"], host["y2"], host["x1"], host["x2"]))
        # the same minimal-bytes definition as the GPU arm (A once per application)
        nbytes = 2 * n * n * 4 + 4 * (4 * n) + 4 * (6 * n)
        cfg = BicgMvt.desc
        sample = "the full BICG+MVT 4096^2 step (4 loop nests) per step"
    elif wl == "kmeans":
        npts, nf, k, ld = 494020, 34, 5, 494020
        feat = oracle.fill(si.SEED_KMEANS, nf * ld)
        cl = feat.reshape(nf, ld)[:, :k].T.copy()
        step = lambda: oracle.kmeans_assign(feat, ld, npts, nf, cl)
        nbytes = npts * nf * 4 + npts * 4
        cfg = Kmeans.desc
        sample = "the full assign step per step"
    elif wl == "atax":
        # configs[4]: the oracle on a bounded sample of the 65536 x 16384 matrix
        # (its first 2048 rows, all 16384 columns: 128 MiB, the same generator
        # and seed as the GPU arm), tmp = A x and y = A^T tmp per step
        rows, n = 2048, 16384
        A = oracle.fill(si.SEED_ATAX_SHARDED, rows * n).reshape(rows, n)
        x = oracle.fill(si.sub_seed(si.SEED_ATAX_SHARDED, 1), n)
        step = lambda: oracle.atax(A, x)
        nbytes = rows * n * 4 + 4 * (2 * n + rows)
        cfg = Atax.desc
        sample = f"ATAX on the first {rows} of the 65536 rows (x 16384 columns) per step"
    else:
        print(json.dumps({"impl": "reference", "unavailable": f"reference arm implemented for atax, bicg_mvt and kmeans, not {wl}"}))
        return 0
    for _ in range(max(args.warmup, 1)):
        step()
    ts = []
    for _ in range(args.steps):
        a = time.perf_counter()
        step()
        ts.append(time.perf_counter() - a)
    ms = 1e3 * statistics.mean(ts)
    gbs = nbytes / (ms * 1e-3) / 1e9
    cores = oracle.num_threads()
    line = {"metric": METRIC, "value": round(gbs, 3), "unit": "GB/s", "n_gpus": args.gpus, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": round(ms, 4), "higher_is_better": True,
            "scaling": "strong" if args.workload == "atax" else "weak",
            "vs_baseline": None, "dtype": "f32", "data": "synthetic (seeded counter hash)",
            "config": {"workload": cfg, "l2": "n/a (CPU)"}, "impl": "reference",
            "cpu_baseline": {"value": round(gbs, 3), "unit": "GB/s", "cores": cores, "kind": "oracle",
                             "sample": sample},
            "e2e": {"value": round(gbs, 3), "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
            "setup_s": round(time.perf_counter() - t0, 2)}
    print(json.dumps(line), flush=True)
    return 0


def main():
    args = parse()
    if args.warmup < 3:
        log("warmup raised to 3 (timing rule)")
        args.warmup = 3
    if args.impl == "reference":
        return run_reference(args)
    world, rank, local = dist_env()
    import torch
    if not torch.cuda.is_available():
        raise SystemExit("bench.py needs a CUDA device (no CPU fallback)")
    # CATT_BENCH_SHARE_GPU=1 (tests only): every rank on cuda:0 over gloo, so
    # the N > 1 path can be exercised on a one-GPU box; never a bench number
    share = os.environ.get("CATT_BENCH_SHARE_GPU") == "1"
    if share:
        local = 0
    torch.cuda.set_device(local)
    if world > 1:
        import torch.distributed as dist
        # NCCL's own report of the communicator (ranks, NVLink / NVLS paths)
        # lands in stderr for the driver's rank check
        os.environ.setdefault("NCCL_DEBUG", "INFO")
        if share:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        barrier = lambda: dist.barrier()
    else:
        barrier = lambda: None
    log(f"bench: rank {rank} of world {world} on cuda:{local} ({torch.cuda.get_device_name(local)}), "
        f"workload {args.workload}")
    import paper_conf_icpp_kimhlsh19_b200 as catt

    w = WORKLOADS[args.workload](catt, torch, rank, world, args.variant)
    if args.l1_child:
        return l1_child(args, catt, torch, w)
    # L2 flush between steps: write 256 MiB (> 126 MB L2), then read another
    # 256 MiB so the lines left in L2 are clean (a write-only flush leaves
    # ~126 MB of dirty lines whose write-back would land in the timed region)
    flush_buf = torch.empty(64 * 1024 * 1024, dtype=torch.int32, device="cuda")
    clean_buf = torch.zeros(64 * 1024 * 1024, dtype=torch.int32, device="cuda")

    def flush():
        # keep the GPU busy ~0.2 ms while the host enqueues the timed launches,
        # so host-side enqueue cost never lands between the CUDA events. Order
        # "sleep_flush" sleeps first, so HBM is busy with the flush right up to
        # the timed kernels; "flush_sleep" leaves it idle for the sleep.
        if args.flush_order == "sleep_flush":
            torch.cuda._sleep(400_000)
        flush_buf.zero_()
        clean_buf.sum()
        if args.flush_order == "flush_sleep":
            torch.cuda._sleep(400_000)
    torch.cuda.synchronize()

    clocks = ClockSampler(local)
    clocks.start()
    steps_ms, per_loop, coll = time_loops(torch, w, flush, args.steps, args.warmup, barrier)
    clk = clocks.stop()

    ms_local = statistics.mean(steps_ms)
    loop_ms = [statistics.mean(x) for x in per_loop]
    t = torch.tensor([ms_local], device="cuda", dtype=torch.float64)
    if world > 1:
        import torch.distributed as dist
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    ms = float(t.item())
    # the step's algorithmic bytes: the minimal traffic of the computation (A
    # read once per application, vectors once), whatever the variant does
    step_bytes = w.step_bytes() if hasattr(w, "step_bytes") else sum(lp.nbytes for lp in w.loops)
    total_bytes = step_bytes * world
    value = total_bytes / (ms * 1e-3) / 1e9

    # ---- end to end through the public API: pinned host inputs -> device -> loops -> host outputs
    e2e = None
    if not args.no_e2e:
        ins = [x for x in w.inputs()]
        outs = [x for x in w.outputs()]
        h_in = [torch.empty(x.shape, dtype=x.dtype, pin_memory=True) for x in ins]
        for h, d in zip(h_in, ins):
            h.copy_(d)
        h_out = [torch.empty(x.shape, dtype=x.dtype, pin_memory=True) for x in outs]
        st = torch.cuda.current_stream()

        def e2e_step():
            for h, d in zip(h_in, ins):
                d.copy_(h, non_blocking=True)
            for lp in w.loops:
                lp.fn()
            w.collective()
            for h, d in zip(h_out, outs):
                h.copy_(d, non_blocking=True)

        for _ in range(args.warmup):
            e2e_step()
        torch.cuda.synchronize()
        barrier()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(st)
        for _ in range(args.steps):
            e2e_step()
        b.record(st)
        torch.cuda.synchronize()
        e2e_ms = a.elapsed_time(b) / args.steps
        tt = torch.tensor([e2e_ms], device="cuda", dtype=torch.float64)
        if world > 1:
            import torch.distributed as dist
            dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        e2e_ms = float(tt.item())
        h2d = sum(x.numel() * x.element_size() for x in ins)
        d2h = sum(x.numel() * x.element_size() for x in outs)
        e2e = {"value": round(total_bytes / (e2e_ms * 1e-3) / 1e9, 3), "unit": "GB/s", "ms_per_step": round(e2e_ms, 4),
               "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h}

    study = app = kst = l1 = None
    if rank == 0 and world == 1 and not args.no_study:   # N > 1 (SCALE runs): the studies are per-GPU, done at N = 1
        study = throttle_study(catt, torch, w, flush)
        app = app_study(catt, torch, w, flush)
        kst = kernel_study(catt, torch, w, flush)
        if world == 1 and not args.no_l1:
            l1 = l1_pass(args, study)

    # ---- roofline of the dominant loop
    dom = max((i for i in range(len(w.loops)) if w.loops[i].kind != "collective"), key=lambda i: loop_ms[i])
    lp = w.loops[dom]
    peak, peak_src = peak_hbm()
    if lp.kind in ("syrk", "syr2k", "corr", "gemm"):
        # FP32 CUDA-core bound: 148 SMs x 128 FP32 lanes x 2 flop x clock
        clk_mhz = clk.get("sm_mhz") or 1965.0
        peak_t = 148 * 128 * 2 * clk_mhz * 1e6 / 1e12
        ach = w.flops / (loop_ms[dom] * 1e-3) / 1e12
        roof = {"bound": "alu", "kernel": lp.name, "achieved": round(ach, 3), "peak": round(peak_t, 3),
                "unit": "TFLOP/s", "frac": round(ach / peak_t, 4), "traffic": ncu_traffic(w.name) if w.variant == type(w).variant else None,
                "peak_source": f"derived: 148 SM x 128 FP32 lanes x 2 x {clk_mhz:.0f} MHz (median under load)",
                # the highest FP32 FMA rate measured on this pool's B200 (tools/ffma_probe.cu:
                # independent FFMA chains, 512-thread CTAs, 1965 MHz; profiles/r2/tiles/ffma_probe.txt)
                "measured_peak": FP32_MEASURED_TFLOPS, "frac_of_measured": round(ach / FP32_MEASURED_TFLOPS, 4),
                "measured_peak_source": "tools/ffma_probe.cu, profiles/r2/tiles/ffma_probe.txt"}
    else:
        ach = lp.nbytes / (loop_ms[dom] * 1e-3) / 1e9
        roof = {"bound": "hbm", "kernel": lp.name, "achieved": round(ach, 2), "peak": peak, "unit": "GB/s",
                "frac": round(ach / peak, 4), "traffic": ncu_traffic(w.name) if w.variant == type(w).variant else None,
                "peak_source": f"{peak_src} (MEASURED_PEAKS.json hbm_gbs)" if peak_src == "measured" else "fallback"}

    # ---- the dominant loop's rate on every rank (max-over-ranks timing above
    # is the job's; this is each GPU's own roofline)
    if world > 1:
        import torch.distributed as dist
        mine = torch.tensor([loop_ms[dom]], device="cuda", dtype=torch.float64)
        allr = [torch.zeros_like(mine) for _ in range(world)]
        dist.all_gather(allr, mine)
        roof["per_rank"] = []
        for r_, t_ in enumerate(allr):
            ms_r = float(t_.item())
            a_r = (w.flops / (ms_r * 1e-3) / 1e12) if roof["unit"] == "TFLOP/s" else lp.nbytes / (ms_r * 1e-3) / 1e9
            roof["per_rank"].append({"rank": r_, "ms": round(ms_r, 5), "achieved": round(a_r, 2),
                                     "frac": round(a_r / roof["peak"], 4)})

    # ---- context: a plain device copy moving the same bytes as the dominant
    # loop, timed the same way (flush, queued events). At 64 MiB a single
    # kernel cannot reach the 2 GiB copy peak of MEASURED_PEAKS.json.
    if lp.kind not in ("syrk", "syr2k", "corr", "gemm"):
        half = max(1, lp.nbytes // 8)                # floats per side: read + write = nbytes
        src = torch.empty(half, device="cuda")
        dst = torch.empty(half, device="cuda")
        cts = []
        for r in range(6):
            flush()
            a_, b_ = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a_.record()
            dst.copy_(src)
            b_.record()
            torch.cuda.synchronize()
            if r:
                cts.append(a_.elapsed_time(b_))
        cgbs = 2 * half * 4 / (statistics.median(cts) * 1e-3) / 1e9
        roof["same_size_copy_gbs"] = round(cgbs, 1)
        roof["frac_of_same_size_copy"] = round(roof["achieved"] / cgbs, 4)
        # and a read-only stream of the same bytes (torch sum): most loops here
        # only read, and a read-only stream of <= 128 MB is far from the copy peak
        rd = torch.empty(max(1, lp.nbytes // 4), device="cuda").fill_(1.0)
        rts = []
        for r in range(6):
            flush()
            a_, b_ = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a_.record()
            rd.sum()
            b_.record()
            torch.cuda.synchronize()
            if r:
                rts.append(a_.elapsed_time(b_))
        rgbs = rd.numel() * 4 / (statistics.median(rts) * 1e-3) / 1e9
        roof["same_size_read_gbs"] = round(rgbs, 1)
        roof["frac_of_same_size_read"] = round(roof["achieved"] / rgbs, 4)
        del src, dst, rd

    # ---- CPU oracle baseline (rank 0, N = 1)
    cpu = None
    if rank == 0 and world == 1 and args.cpu_seconds > 0:
        try:
            import oracle
            host = w.host_copy()
            w.cpu_oracle_step(oracle, host)
            reps, t0 = 0, time.perf_counter()
            while time.perf_counter() - t0 < args.cpu_seconds:
                w.cpu_oracle_step(oracle, host)
                reps += 1
            sec = (time.perf_counter() - t0) / reps
            cpu_bytes = step_bytes
            if w.name in ("syrk", "syr2k"):
                cpu_bytes = step_bytes * 16 / 2048
            if w.name == "corr":                         # the oracle runs a 256 x 256 sample of the data
                cpu_bytes = 256 * 256 * 4 * 3
            if w.name == "atax":
                cpu_bytes = step_bytes * min(w.rows, 8192) / w.rows
            cpu = {"value": round(cpu_bytes / sec / 1e9, 3), "unit": "GB/s", "cores": oracle.num_threads(),
                   "kind": "oracle", "sample": f"{reps} x one oracle step ({w.name}), {1e3 * sec:.1f} ms each"}
            # the same oracle on one host thread (SURVEY 8(d) oracle timing (i))
            nthr = oracle.num_threads()
            oracle.set_num_threads(1)
            try:
                reps1, t0 = 0, time.perf_counter()
                while reps1 < 1 or time.perf_counter() - t0 < args.cpu_seconds / 2:
                    w.cpu_oracle_step(oracle, host)
                    reps1 += 1
                sec1 = (time.perf_counter() - t0) / reps1
            finally:
                oracle.set_num_threads(nthr)
            cpu["single_thread"] = {"value": round(cpu_bytes / sec1 / 1e9, 3), "unit": "GB/s", "cores": 1,
                                    "sample": f"{reps1} x the same step, {1e3 * sec1:.1f} ms each"}
        except Exception as ex:                     # pragma: no cover
            cpu = {"value": None, "unit": "GB/s", "cores": None, "kind": "oracle", "sample": f"failed: {ex}"}

    if rank == 0:
        line = {
            "metric": METRIC, "value": round(value, 2), "unit": "GB/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": round(ms, 5), "higher_is_better": True, "scaling": w.scaling,
            "vs_baseline": None, "dtype": "f32", "data": "synthetic (seeded counter hash, generated on device)",
            "config": {"workload": w.desc, "variant": w.variant, "l2": "flushed before every step (256 MiB write, then 256 MiB clean read)", "flush_order": args.flush_order,
                       "rows_per_rank": getattr(w, "rows", None), "parallelism": f"{w.parallelism} x{world}"},
            "loops": {lp.name: {"ms": round(loop_ms[i], 5),
                                "gbs": round(lp.nbytes / (loop_ms[i] * 1e-3) / 1e9, 1),
                                "plan": [dict(w.plans[k], loop=k) for k in lp.plans if k in w.plans] or None}
                      for i, lp in enumerate(w.loops)},
            "analysis_us": max([p_["analysis_us"] for p_ in w.plans.values()] +
                               [r_.get("analysis_us", 0) for r_ in (study or [])] or [None]),
            "collective_ms": round(statistics.mean(coll), 5) if world > 1 else 0.0,
            "roofline": roof,
            "cpu_baseline": cpu,
            "e2e": e2e,
            "gpu_launches": len(w.loops) * args.steps,
            "clocks": clk,
            "l1_hit_pct": ({role: study[0]["l1"][role]["l1_hit_pct"] for role in ("catt", "paper", "full", "best")
                            if role in study[0].get("l1", {})} if study and l1 and l1.get("status") == "ok" else None),
            "l1_pass": l1,
            "throttle_study": study,
            "bftt_vs_catt": app,
            "per_loop_in_one_kernel": kst,
        }
        print(json.dumps(line), flush=True)
    if world > 1:
        import torch.distributed as dist
        dist.barrier()
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
