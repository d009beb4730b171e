#!/bin/bash
export PYTHONPATH=.
O=gpurun_out/r1ai; mkdir -p $O
for C in 0 1; do for M in 2 1; do
  echo "contig=$C ctas_per_sm=$M $(CATT_KMEANS_CONTIG=$C CATT_KMEANS_CTAS_PER_SM=$M timeout 300 python bench.py --workload kmeans --steps 30 --warmup 5 --no-study --no-e2e --cpu-seconds 0 2>/dev/null | python -c 'import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(d["ms_per_step"], [(k, v["ms"]) for k, v in d["loops"].items()])')" >> $O/bench.txt
done; done
CATT_KMEANS_CONTIG=1 timeout 600 python -m pytest tests/test_gpu.py -q -x -k "kmeans" -p no:cacheprovider > $O/pytest.txt 2>&1
