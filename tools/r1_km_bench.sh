#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_kmeans.py -q -x > gpurun_out/km_tests.log 2>&1; echo "rc=$?" >> gpurun_out/km_tests.log
timeout 600 python bench.py --workload kmeans_iter --steps 20 --warmup 5 --no-study --cpu-seconds 0 > gpurun_out/kmi_bench.json 2> gpurun_out/kmi_bench.err
PYTHONPATH=. timeout 600 ncu --set full --clock-control none --import-source on -k regex:km_acc -o gpurun_out/km_full -f python tools/ncu_km.py > gpurun_out/ncu_km.log 2>&1
