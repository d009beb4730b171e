#!/bin/bash
export PYTHONPATH=.
O=gpurun_out/r1kmf; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_kmeans.py tests/test_gpu.py tests/test_dist.py -q -x -k "kmeans" > $O/pytest.txt 2>&1; echo "rc=$?" >> $O/pytest.txt
for i in 1 2; do
  timeout 600 python bench.py --workload kmeans_iter --no-study --steps 30 --no-e2e --cpu-seconds 0 > $O/bench_new_$i.json 2> /dev/null
  CATT_KM_FENCE_ALL=1 timeout 600 python bench.py --workload kmeans_iter --no-study --steps 30 --no-e2e --cpu-seconds 0 > $O/bench_old_$i.json 2> /dev/null
done
