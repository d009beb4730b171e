#!/bin/bash
export PYTHONPATH=.
O=gpurun_out/lean; mkdir -p $O; : > $O/cfg.txt
timeout 900 python -m pytest tests/test_gpu.py -q -m gpu -k "syrk or corr or gemm or syr2k" > $O/tests.txt 2>&1; echo "rc=$?" >> $O/tests.txt
for w in syrk corr gemm syr2k; do
  r=$(timeout 300 python bench.py --workload $w --no-study --no-e2e --cpu-seconds 0 --steps 10 2>/dev/null | python -c "import json,sys; d=json.load(sys.stdin); print(d['ms_per_step'], d['roofline']['achieved'], d['roofline']['frac'])")
  echo "$w $r" >> $O/cfg.txt
done
