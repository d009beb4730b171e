#!/bin/bash
export PYTHONPATH=.
O=gpurun_out/r1ac; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu.py -q -x -k "syrk or syr2k or gemm or corr" -p no:cacheprovider > $O/pytest.txt 2>&1
for W in syrk syr2k corr gemm; do
  echo "$W $(timeout 300 python bench.py --workload $W --steps 20 --warmup 3 --no-study --no-e2e --cpu-seconds 0 2>$O/$W.err | python -c 'import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(d["ms_per_step"], [(k, v["ms"]) for k, v in d["loops"].items()], d["roofline"]["achieved"], d["roofline"]["frac"])')" >> $O/bench.txt
done
echo "syrk lean=0 $(CATT_TILED_LEAN=0 timeout 300 python bench.py --workload syrk --steps 20 --warmup 3 --no-study --no-e2e --cpu-seconds 0 2>/dev/null | python -c 'import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(d["ms_per_step"], d["roofline"]["achieved"])')" >> $O/bench.txt
