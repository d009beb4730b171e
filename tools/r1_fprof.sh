#!/bin/bash
export PYTHONPATH=.
O=gpurun_out/fprof; mkdir -p $O
CATT_FUSED_STAGE_KB=16 timeout 600 ncu --set full --clock-control none --import-source on -k regex:fused_nd -s 3 -c 1 -o $O/nd16 -f python bench.py --steps 1 --warmup 3 --no-study --no-e2e --cpu-seconds 0 > $O/nd16.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:fused_nd -s 3 -c 1 -o $O/nd64 -f python bench.py --steps 1 --warmup 3 --no-study --no-e2e --cpu-seconds 0 > $O/nd64.log 2>&1
