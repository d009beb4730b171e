#!/bin/bash
# SM partitions (green contexts): GPU tests, then the GESUMMV study with
# CTA- vs warp-level throttling at 4 / 2 CTAs per SM
export PYTHONPATH=.
O=gpurun_out/r1g2; mkdir -p $O
timeout 600 python -m pytest tests/test_gpu.py -q -x -k "sm_partition or dual or residency" > $O/pytest.txt 2>&1; echo "rc=$?" >> $O/pytest.txt
timeout 1500 python bench.py --workload gesummv > $O/bench_gesummv.json 2> $O/bench_gesummv.err
