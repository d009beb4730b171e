#!/bin/bash
# fused BICG+MVT tail: phase trace and bench per grid-barrier form
# (1: ordered atomics + last arriver, 2: per-problem arrival counters)
export PYTHONPATH=.
O=gpurun_out/r1t3; mkdir -p $O
timeout 600 python -m pytest tests/test_gpu.py -q -x -k "fused or dual" > $O/pytest_fused.txt 2>&1; echo "rc=$?" >> $O/pytest_fused.txt
for B in 1 2; do
  CATT_FUSED_BARRIER=$B CATT_FUSED_TRACE=1 timeout 300 python tools/fused_trace.py 4096 8 > $O/trace_bar$B.txt 2>&1
  CATT_FUSED_BARRIER=$B timeout 300 python bench.py --steps 50 --warmup 5 --no-study --no-e2e --cpu-seconds 0 > $O/bench_bar$B.json 2>&1
done
