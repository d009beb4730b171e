#!/bin/bash
export PYTHONPATH=.
O=gpurun_out/r1ag; mkdir -p $O
timeout 600 python -m pytest tests/test_gpu_peer.py -q -x -p no:cacheprovider > $O/pytest_peer.txt 2>&1
timeout 900 python -m pytest tests/test_gpu.py -q -x -k "fused or dual or atax" -p no:cacheprovider > $O/pytest_fused.txt 2>&1
echo "atax fused $(timeout 300 python bench.py --workload atax --steps 20 --warmup 3 --no-study --no-e2e --cpu-seconds 0 2>/dev/null | python -c 'import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(d["ms_per_step"], [(k, v["ms"]) for k, v in d["loops"].items()])')" >> $O/bench.txt
echo "atax fused_peer $(timeout 300 python bench.py --workload atax --variant fused_peer --steps 20 --warmup 3 --no-study --no-e2e --cpu-seconds 0 2>$O/peer.err | python -c 'import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(d["ms_per_step"], [(k, v["ms"]) for k, v in d["loops"].items()])')" >> $O/bench.txt
