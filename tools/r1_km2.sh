#!/bin/bash
# KMEANS iteration: ballot phase 2 (default) vs the sorted form (CATT_KM_SORT=1)
export PYTHONPATH=.
O=gpurun_out/r1km2; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_kmeans.py -q -x > $O/pytest.txt 2>&1; echo "rc=$?" >> $O/pytest.txt
timeout 600 python bench.py --workload kmeans_iter --no-study --steps 30 > $O/bench_bal.json 2> $O/bench_bal.err
CATT_KM_SORT=1 timeout 600 python bench.py --workload kmeans_iter --no-study --steps 30 --no-e2e --cpu-seconds 0 > $O/bench_sort.json 2> $O/bench_sort.err
timeout 600 ncu --set full --clock-control none --import-source on -k regex:km_accumulate -s 3 -c 1 -o $O/ncu_km -f python bench.py --workload kmeans_iter --steps 1 --warmup 3 --no-study --no-e2e --cpu-seconds 0 > $O/ncu.log 2>&1
