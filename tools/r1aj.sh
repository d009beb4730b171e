#!/bin/bash
export PYTHONPATH=.
O=gpurun_out/r1aj; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu.py tests/test_gpu_peer.py -q -x -k "fused or dual or atax or peer" -p no:cacheprovider > $O/pytest.txt 2>&1
for E in "X=0" "CATT_FUSED_NO_SMALL=1"; do
echo "$E atax256 $(env $E timeout 300 python bench.py --workload atax256 --steps 30 --warmup 5 --no-study --no-e2e --cpu-seconds 0 2>/dev/null | python -c 'import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(d["ms_per_step"], [(k, v["ms"]) for k, v in d["loops"].items()])')" >> $O/bench.txt
done
