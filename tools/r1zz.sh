#!/bin/bash
# Round-1 closing measurement pass (third session): smoke, every GPU test,
# every bench workload (throttle studies included), the reference arm, the
# default bench's launch list, one ncu --set full capture of each
# workload's dominant kernel.
export PYTHONPATH=.
O=gpurun_out/r1zz
mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw,temperature.gpu --format=csv > $O/nvsmi.txt 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.txt 2>&1; echo "smoke rc=$?" >> $O/smoke.txt
timeout 1800 python -m pytest tests -m gpu -q > $O/pytest_gpu.txt 2>&1; echo "rc=$?" >> $O/pytest_gpu.txt
timeout 900 python bench.py > $O/bench_bicg_mvt.json 2> $O/bench_bicg_mvt.err
for w in kmeans kmeans_iter gesummv syrk syr2k corr gemm atax atax256; do
  timeout 1500 python bench.py --workload $w > $O/bench_$w.json 2> $O/bench_$w.err
done
timeout 900 python bench.py --impl reference --steps 3 --warmup 3 > $O/bench_reference.json 2> $O/bench_reference.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_bicg_mvt.csv python bench.py --steps 2 --warmup 3 --no-study --no-e2e --cpu-seconds 0 > /dev/null 2>&1
for pair in "bicg_mvt:fused_nd" "kmeans:kmeans_tma" "kmeans_iter:km_accumulate" "gesummv:row_warp" "syrk:tiled_kernel" "syr2k:tiled_kernel" "corr:tiled_kernel" "gemm:tiled_kernel" "atax:fused_kernel" "atax256:atax_small"; do
  w=${pair%%:*}; k=${pair##*:}
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:$k -s 3 -c 1 -o $O/ncu_$w -f python bench.py --workload $w --steps 1 --warmup 3 --no-study --no-e2e --cpu-seconds 0 > $O/ncu_$w.log 2>&1
done
ls -la $O
