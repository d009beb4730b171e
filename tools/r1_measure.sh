#!/bin/bash
# Round-1 measurement set (run under gpurun). Outputs land in gpurun_out/r1/.
export PYTHONPATH=.
O=gpurun_out/r1; mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > $O/nvsmi.txt
timeout 1200 python -m pytest tests -q -m gpu -p no:cacheprovider > $O/pytest_gpu.txt 2>&1
python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.txt 2>&1
python bench.py > $O/bench_bicg_mvt.json 2> $O/bench.err
for w in kmeans gesummv syrk atax256 atax; do python bench.py --workload $w --cpu-seconds 3 > $O/bench_$w.json 2>> $O/bench.err; done
python bench.py --variant coop --no-study --cpu-seconds 0 > $O/bench_bicg_mvt_coop.json 2>> $O/bench.err
python bench.py --variant staged --no-study --cpu-seconds 0 > $O/bench_bicg_mvt_staged.json 2>> $O/bench.err
python bench.py --impl reference --steps 3 > $O/bench_reference.json 2>> $O/bench.err
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_bicg_mvt.csv python bench.py --steps 2 --warmup 3 --no-study --no-e2e --cpu-seconds 0 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:"fused_kernel" -s 2 -c 2 -o $O/prof_fused python bench.py --steps 1 --warmup 3 --no-study --no-e2e --cpu-seconds 0 > $O/prof_fused.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:"fused_kernel" -s 3 -c 1 -o $O/prof_fused_atax python bench.py --workload atax --steps 1 --warmup 3 --no-study --no-e2e --cpu-seconds 0 > $O/prof_fused_atax.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:"kmeans_kernel|row_warp|syrk_tiled" -s 3 -c 1 -o $O/prof_kmeans python bench.py --workload kmeans --steps 1 --warmup 3 --no-study --no-e2e --cpu-seconds 0 > $O/prof_kmeans.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:"row_warp" -s 3 -c 1 -o $O/prof_gesummv python bench.py --workload gesummv --steps 1 --warmup 3 --no-study --no-e2e --cpu-seconds 0 > $O/prof_gesummv.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:"syrk_tiled" -s 3 -c 1 -o $O/prof_syrk python bench.py --workload syrk --steps 1 --warmup 3 --no-study --no-e2e --cpu-seconds 0 > $O/prof_syrk.log 2>&1
ls -la $O
