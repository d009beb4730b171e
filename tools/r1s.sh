#!/bin/bash
# fused phase trace; KMEANS COOP (FFMA2, 16-byte lanes) parity + bench vs staged
export PYTHONPATH=.
O=gpurun_out/r1s; mkdir -p $O
timeout 300 python tools/fused_trace.py 4096 6 > $O/fused_trace.txt 2>&1
CATT_FUSED_SMEM_KB=220 timeout 300 python tools/fused_trace.py 4096 4 > $O/fused_trace_s3.txt 2>&1
timeout 600 python -m pytest tests/test_gpu.py -q -x -k "kmeans" -p no:cacheprovider > $O/pytest_kmeans.txt 2>&1
for V in staged coop regs; do
  echo "$V $(timeout 120 python bench.py --workload kmeans --variant $V --steps 30 --warmup 5 --no-study --no-e2e --cpu-seconds 0 2>/dev/null | python -c 'import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(d["ms_per_step"], [(k, v["ms"]) for k, v in d["loops"].items()])')" >> $O/kmeans_variants.txt
done
for B in 200 220; do
  echo "B=$B $(CATT_FUSED_SMEM_KB=$B timeout 120 python bench.py --steps 30 --warmup 5 --no-study --no-e2e --cpu-seconds 0 2>/dev/null | python -c 'import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(d["ms_per_step"], [(k, v["ms"]) for k, v in d["loops"].items()])')" >> $O/fused_budget.txt
done
