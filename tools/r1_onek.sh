#!/bin/bash
# ATAX in one kernel with a throttle per loop: GPU tests, the one-kernel study
export PYTHONPATH=.
O=gpurun_out/r1ok; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu.py -q -x -k "onekernel" > $O/pytest.txt 2>&1; echo "rc=$?" >> $O/pytest.txt
timeout 1500 python bench.py --workload atax256 --steps 10 --cpu-seconds 0 --no-e2e > $O/bench_atax256.json 2> $O/bench_atax256.err
