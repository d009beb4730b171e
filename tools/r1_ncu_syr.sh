#!/bin/bash
mkdir -p gpurun_out
PYTHONPATH=. ncu --set full --clock-control none --import-source on -k regex:tiled -o gpurun_out/syr_full -f python tools/ncu_syr.py > gpurun_out/ncu_syr.log 2>&1
CATT_SYR2K_MINB=2 PYTHONPATH=. ncu --set full --clock-control none --import-source on -k regex:syr2k_tiled -o gpurun_out/syr2k_minb2 -f python tools/ncu_syr.py >> gpurun_out/ncu_syr.log 2>&1
