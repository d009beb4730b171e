#!/bin/bash
# CORR staged: batched loads for the sequential statistics chains
export PYTHONPATH=.
O=gpurun_out/r1c3; mkdir -p $O
timeout 900 python -m pytest tests -m gpu -q -x -k "corr" > $O/pytest.txt 2>&1; echo "rc=$?" >> $O/pytest.txt
timeout 600 python bench.py --workload corr --no-study --steps 20 --cpu-seconds 0 > $O/bench_corr.json 2> $O/bench_corr.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_corr.csv python bench.py --workload corr --steps 2 --warmup 3 --no-study --no-e2e --cpu-seconds 0 > /dev/null 2>&1
