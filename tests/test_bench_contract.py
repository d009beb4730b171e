"""The bench.py JSON contract the driver parses (one line, required keys and
types), on a short run of the default workload and of the reference arm."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _run(args, timeout=900):
    env = dict(os.environ, PYTHONPATH=ROOT)
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py")] + args, capture_output=True, text=True,
                         timeout=timeout, cwd=ROOT, env=env)
    assert out.returncode == 0, out.stderr[-2000:]
    lines = [l for l in out.stdout.strip().splitlines() if l.startswith("{")]
    assert len(lines) == 1, out.stdout
    return json.loads(lines[0])


@pytest.mark.gpu
def test_default_bench_line():
    d = _run(["--steps", "3", "--warmup", "3", "--no-study", "--cpu-seconds", "1"])
    for k, t in (("metric", str), ("value", (int, float)), ("unit", str), ("n_gpus", int), ("steps", int),
                 ("warmup", int), ("ms_per_step", (int, float)), ("higher_is_better", bool), ("scaling", str),
                 ("dtype", str), ("data", str), ("config", dict), ("gpu_launches", int), ("clocks", dict),
                 ("roofline", dict), ("cpu_baseline", dict), ("e2e", dict)):
        assert isinstance(d.get(k), t), k
    assert "vs_baseline" in d and d["n_gpus"] == 1 and d["steps"] == 3 and d["warmup"] >= 3
    assert "workload" in d["config"] and d["value"] > 0 and d["gpu_launches"] > 0
    r = d["roofline"]
    assert r["bound"] in ("hbm", "tensor", "alu") and r["peak"] > 0 and abs(r["frac"] - r["achieved"] / r["peak"]) < 1e-3
    c = d["cpu_baseline"]
    assert c["kind"] == "oracle" and c["cores"] >= 1 and c["value"] > 0 and c["sample"]
    e = d["e2e"]
    assert e["value"] > 0 and e["h2d_bytes_per_step"] > 0 and e["d2h_bytes_per_step"] > 0
    assert {"sm_mhz", "sm_max_mhz", "reasons"} <= set(d["clocks"])


def test_reference_arm_line():
    """--impl reference runs the CPU oracle (no GPU needed)."""
    d = _run(["--impl", "reference", "--steps", "1", "--warmup", "3"])
    assert d["impl"] == "reference" and d["value"] > 0 and d["cpu_baseline"]["kind"] == "oracle"
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["e2e"]["d2h_bytes_per_step"] == 0
    assert d["unit"] == "GB/s" and d["higher_is_better"] is True


def _run_torchrun(args, nproc=2, timeout=900, extra_env=None):
    env = dict(os.environ, PYTHONPATH=ROOT, **(extra_env or {}))
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes", "1", "--nproc-per-node", str(nproc),
           "--master-addr", "127.0.0.1", "--master-port", str(29600 + os.getpid() % 300),
           os.path.join(ROOT, "bench.py"), "--gpus", str(nproc)] + args
    out = subprocess.run(cmd, capture_output=True, text=True, timeout=timeout, cwd=ROOT, env=env)
    assert out.returncode == 0, out.stderr[-3000:]
    lines = [l for l in out.stdout.strip().splitlines() if l.startswith("{")]
    assert len(lines) == 1, out.stdout          # rank 0 alone prints
    return json.loads(lines[0])


def test_reference_arm_under_torchrun_rank0_only():
    """The driver launches --impl reference through torchrun for N > 1: rank 0
    runs the oracle and prints the one line, the other ranks exit 0."""
    d = _run_torchrun(["--impl", "reference", "--steps", "1", "--warmup", "3"])
    assert d["impl"] == "reference" and d["value"] > 0 and d["e2e"]["h2d_bytes_per_step"] == 0


@pytest.mark.gpu
@pytest.mark.parametrize("workload,variant,par", [("atax", None, "row-shard"), ("atax", "fused_peer", "row-shard"),
                                                  ("bicg_mvt", None, "row-shard"),
                                                  ("kmeans_iter", None, "point-shard"),
                                                  ("syrk", None, "independent problem per rank")])
def test_bench_two_ranks_share_one_gpu(workload, variant, par):
    """The N > 1 bench path end to end (row shards with the A^T all-reduce
    between the ranks or inside the fused kernel, k-means points with the
    exact-sum all-reduce, independent replicas; max-over-ranks timing, one
    line from rank 0), with both ranks on cuda:0 over gloo
    (CATT_BENCH_SHARE_GPU, tests only: NCCL refuses two ranks on one device).
    Not a bench number."""
    args = ["--workload", workload, "--steps", "2", "--warmup", "3", "--no-study", "--no-l1", "--cpu-seconds", "0"]
    if variant:
        args += ["--variant", variant]
    d = _run_torchrun(args, extra_env={"CATT_BENCH_SHARE_GPU": "1"})
    assert d["n_gpus"] == 2 and d["value"] > 0 and d["gpu_launches"] > 0
    assert d["config"]["parallelism"] == f"{par} x2"
    if workload == "atax":
        assert d["config"]["rows_per_rank"] == 65536 // 2
    assert isinstance(d["roofline"], dict) and d["roofline"]["achieved"] > 0
