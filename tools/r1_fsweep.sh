#!/bin/bash
# fused BICG+MVT stage size x ring budget, with the per-problem arrival counters
export PYTHONPATH=.
O=gpurun_out/r1fs; mkdir -p $O
for KB in 32 48 64 96; do for B in 140 180 220; do
  echo "KB=$KB BUDGET=$B $(CATT_FUSED_STAGE_KB=$KB CATT_FUSED_SMEM_KB=$B timeout 120 python bench.py --steps 40 --warmup 5 --no-study --no-e2e --cpu-seconds 0 2>/dev/null | python -c 'import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(d["ms_per_step"], [(k, v["ms"]) for k, v in d["loops"].items()])')" >> $O/fused_sweep.txt
done; done
