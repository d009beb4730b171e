#!/bin/bash
export PYTHONPATH=.
O=gpurun_out/r1t; mkdir -p $O
timeout 120 ./tools/launch_probe > $O/launch_probe.txt 2>&1
for FB in 0 1; do for B in 200 220; do
  echo "== barrier=$FB budget=$B" >> $O/fused_trace.txt
  CATT_FUSED_BARRIER=$FB CATT_FUSED_SMEM_KB=$B timeout 300 python tools/fused_trace.py 4096 4 >> $O/fused_trace.txt 2>&1
  echo "FB=$FB B=$B $(CATT_FUSED_BARRIER=$FB CATT_FUSED_SMEM_KB=$B timeout 120 python bench.py --steps 30 --warmup 5 --no-study --no-e2e --cpu-seconds 0 2>/dev/null | python -c 'import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(d["ms_per_step"], [(k, v["ms"]) for k, v in d["loops"].items()])')" >> $O/fused_bench.txt
done; done
timeout 600 python -m pytest tests/test_gpu.py -q -x -k "fused or dual or kmeans" -p no:cacheprovider > $O/pytest.txt 2>&1
for V in staged coop; do
  echo "$V $(timeout 120 python bench.py --workload kmeans --variant $V --steps 30 --warmup 5 --no-study --no-e2e --cpu-seconds 0 2>$O/km_$V.err | python -c 'import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(d["ms_per_step"], [(k, v["ms"]) for k, v in d["loops"].items()])')" >> $O/kmeans_variants.txt
done
