#!/bin/bash
export PYTHONPATH=.
O=gpurun_out/fcfg; mkdir -p $O; : > $O/cfg.txt
for cfg in "200 64" "100 32" "110 48" "100 16" "72 32" "200 96"; do set -- $cfg
  r=$(CATT_FUSED_SMEM_KB=$1 CATT_FUSED_STAGE_KB=$2 timeout 300 python bench.py --no-study --no-e2e --cpu-seconds 0 --steps 20 2>/dev/null | python -c "import json,sys; d=json.load(sys.stdin); print(d['ms_per_step'], d['value'])")
  a=$(CATT_FUSED_SMEM_KB=$1 CATT_FUSED_STAGE_KB=$2 timeout 300 python bench.py --workload atax --no-study --no-e2e --cpu-seconds 0 --steps 5 2>/dev/null | python -c "import json,sys; d=json.load(sys.stdin); print(d['ms_per_step'], d['value'])")
  echo "smem=$1 stage=$2  bicg_mvt $r  atax $a" >> $O/cfg.txt
done
