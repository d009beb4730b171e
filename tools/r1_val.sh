#!/bin/bash
# Re-entry validation of HEAD: smoke, all GPU tests, the default bench line, the
# workloads changed since profiles/r1f (kmeans_iter, atax256), the launch list.
export PYTHONPATH=.
O=gpurun_out/r1v
mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw,temperature.gpu --format=csv > $O/nvsmi.txt 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.txt 2>&1; echo "smoke rc=$?" >> $O/smoke.txt
timeout 1800 python -m pytest tests -m gpu -q > $O/pytest_gpu.txt 2>&1; echo "rc=$?" >> $O/pytest_gpu.txt
timeout 900 python bench.py > $O/bench_default.json 2> $O/bench_default.err
for w in kmeans kmeans_iter atax256; do
  timeout 900 python bench.py --workload $w --no-study > $O/bench_$w.json 2> $O/bench_$w.err
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_bicg_mvt.csv python bench.py --steps 2 --warmup 3 --no-study --no-e2e --cpu-seconds 0 > /dev/null 2>&1
ls -la $O
