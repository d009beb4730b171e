#!/bin/bash
export PYTHONPATH=.
O=gpurun_out/r1aa; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu.py -q -x -k "fused or dual or atax" -p no:cacheprovider > $O/pytest.txt 2>&1
for W in atax256 atax; do
  echo "$W $(timeout 300 python bench.py --workload $W --steps 30 --warmup 5 --no-study --no-e2e --cpu-seconds 0 2>$O/$W.err | python -c 'import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(d["ms_per_step"], [(k, v["ms"]) for k, v in d["loops"].items()])')" >> $O/bench.txt
done
echo "atax256 no-cluster $(CATT_FUSED_NO_CLUSTER=1 timeout 300 python bench.py --workload atax256 --steps 30 --warmup 5 --no-study --no-e2e --cpu-seconds 0 2>/dev/null | python -c 'import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(d["ms_per_step"], [(k, v["ms"]) for k, v in d["loops"].items()])')" >> $O/bench.txt
