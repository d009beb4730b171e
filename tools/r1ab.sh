#!/bin/bash
export PYTHONPATH=.
O=gpurun_out/r1ab; mkdir -p $O
ncu --set full --clock-control none --import-source on -k regex:km_accumulate -s 3 -c 1 -o $O/prof_km_acc python bench.py --workload kmeans_iter --steps 1 --warmup 3 --no-study --no-e2e --cpu-seconds 0 > $O/ncu_km.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:tiled_kernel -s 3 -c 1 -o $O/prof_syrk python bench.py --workload syrk --steps 1 --warmup 3 --no-study --no-e2e --cpu-seconds 0 > $O/ncu_syrk.log 2>&1
