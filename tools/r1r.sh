#!/bin/bash
# fused BICG+MVT: interleaved vs banded stage chunks x stage size x ring budget;
# packed-FP32 throughput probe; read ceiling with interleaved bulk copies
export PYTHONPATH=.
O=gpurun_out/r1r; mkdir -p $O
timeout 120 ./tools/ffma_probe > $O/ffma_probe.txt 2>&1
timeout 400 ./tools/read_probe 7 > $O/read_probe.txt 2>&1
for IL in 1 0; do
  CATT_FUSED_INTERLEAVE=$IL timeout 600 python -m pytest tests/test_gpu.py -q -x -k "fused or dual" -p no:cacheprovider > $O/pytest_fused_il$IL.txt 2>&1
done
for IL in 1 0; do for KB in 16 32 48 64; do for B in 100 140 200; do
  echo "IL=$IL KB=$KB BUDGET=$B $(CATT_FUSED_INTERLEAVE=$IL CATT_FUSED_STAGE_KB=$KB CATT_FUSED_SMEM_KB=$B timeout 120 python bench.py --steps 30 --warmup 5 --no-study --no-e2e --cpu-seconds 0 2>/dev/null | python -c 'import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(d["ms_per_step"], [(k, v["ms"]) for k, v in d["loops"].items()])')" >> $O/fused_sweep.txt
done; done; done
