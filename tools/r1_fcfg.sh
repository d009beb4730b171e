#!/bin/bash
export PYTHONPATH=.
O=gpurun_out/fcfg; mkdir -p $O; : > $O/cfg.txt
timeout 900 python -m pytest tests/test_gpu.py tests/test_dist.py -q -m gpu -k "fused or dual or bicg or mvt or rowshard" > $O/tests.txt 2>&1; echo "rc=$?" >> $O/tests.txt
for cfg in "200 64" "200 32" "200 16" "220 32" "200 48" "180 16"; do set -- $cfg
  r=$(CATT_FUSED_SMEM_KB=$1 CATT_FUSED_STAGE_KB=$2 timeout 300 python bench.py --no-study --no-e2e --cpu-seconds 0 --steps 20 2>/dev/null | python -c "import json,sys; d=json.load(sys.stdin); print(d['ms_per_step'], d['value'])")
  echo "smem=$1 stage=$2  bicg_mvt $r" >> $O/cfg.txt
done
