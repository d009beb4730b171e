#!/bin/bash
export PYTHONPATH=.
O=gpurun_out/fnd; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu.py tests/test_dist.py -q -m gpu -k "fused or dual or bicg or mvt or atax or rowshard" > $O/tests.txt 2>&1; echo "rc=$?" >> $O/tests.txt
for ord in flush_sleep sleep_flush; do
  timeout 600 python bench.py --no-study --cpu-seconds 0 --steps 20 --flush-order $ord > $O/bench_nd_$ord.json 2>> $O/err.txt
  CATT_FUSED_ND=1 timeout 600 python bench.py --no-study --cpu-seconds 0 --steps 20 --flush-order $ord > $O/bench_old_$ord.json 2>> $O/err.txt
done
timeout 300 python tools/read_order.py > $O/read_order.txt 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:fused_nd -s 3 -c 1 -o $O/ncu_nd -f python bench.py --steps 1 --warmup 3 --no-study --no-e2e --cpu-seconds 0 > $O/ncu.log 2>&1
