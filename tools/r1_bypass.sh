#!/bin/bash
export PYTHONPATH=.
O=gpurun_out/bypass; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu.py -q -m gpu -k "bypass or rows or bicg or gesummv" > $O/tests.txt 2>&1; echo "rc=$?" >> $O/tests.txt
for w in bicg_mvt gesummv atax256 atax; do
  timeout 1200 python bench.py --workload $w --steps 10 --warmup 3 --no-e2e --cpu-seconds 0 > $O/bench_$w.json 2> $O/bench_$w.err
done
