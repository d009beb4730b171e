#!/bin/bash
export PYTHONPATH=.
O=gpurun_out/kma; mkdir -p $O; : > $O/cfg.txt
timeout 900 python -m pytest tests/test_gpu.py -q -m gpu -k "kmeans" > $O/tests.txt 2>&1; echo "rc=$?" >> $O/tests.txt
for m in 2 1; do
  r=$(CATT_KMEANS_CTAS_PER_SM=$m timeout 300 python bench.py --workload kmeans --no-study --no-e2e --cpu-seconds 0 --steps 20 2>/dev/null | python -c "import json,sys; d=json.load(sys.stdin); print(d['ms_per_step'], d['value'], d['loops'])")
  echo "ctas/sm=$m $r" >> $O/cfg.txt
done
