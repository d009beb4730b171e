#!/bin/bash
export PYTHONPATH=.
O=gpurun_out/corr; mkdir -p $O
timeout 1200 python -m pytest tests/test_gpu.py -q -m gpu -k "gemm or corr or syrk" > $O/tests.txt 2>&1; echo "rc=$?" >> $O/tests.txt
for w in gemm corr syrk; do
  timeout 900 python bench.py --workload $w --steps 10 --warmup 3 --no-study --no-e2e --cpu-seconds 0 > $O/bench_$w.json 2> $O/bench_$w.err
done
