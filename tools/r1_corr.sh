#!/bin/bash
export PYTHONPATH=.
O=gpurun_out/corr; mkdir -p $O
timeout 900 python bench.py --workload corr --steps 5 --warmup 3 > $O/bench_corr.json 2> $O/bench_corr.err
