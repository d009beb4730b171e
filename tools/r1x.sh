#!/bin/bash
export PYTHONPATH=.
O=gpurun_out/r1x; mkdir -p $O
timeout 1500 python -m pytest tests -q -m gpu -p no:cacheprovider > $O/pytest_gpu.txt 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.txt 2>&1; echo "smoke rc=$?" >> $O/smoke.txt
timeout 600 python bench.py --workload kmeans --cpu-seconds 2 > $O/bench_kmeans.json 2> $O/bench_kmeans.err
timeout 600 python bench.py --cpu-seconds 2 > $O/bench_bicg_mvt.json 2> $O/bench.err
