#!/bin/bash
export PYTHONPATH=.
O=gpurun_out/r1ad; mkdir -p $O
for E in "X=0" "CATT_TILED_SMALL=1" "CATT_TILED_LEAN=1"; do
  echo "$E $(env $E timeout 300 python bench.py --workload syrk --steps 20 --warmup 3 --no-study --no-e2e --cpu-seconds 0 2>/dev/null | python -c 'import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(d["ms_per_step"], d["roofline"]["achieved"])')" >> $O/bench.txt
  echo "gemm $E $(env $E timeout 300 python bench.py --workload gemm --steps 20 --warmup 3 --no-study --no-e2e --cpu-seconds 0 2>/dev/null | python -c 'import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(d["ms_per_step"], d["roofline"]["achieved"])')" >> $O/bench.txt
done
CATT_TILED_SMALL=1 timeout 900 python -m pytest tests/test_gpu.py -q -x -k "syrk or gemm or corr" -p no:cacheprovider > $O/pytest_small.txt 2>&1
