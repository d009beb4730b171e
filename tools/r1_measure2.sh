#!/bin/bash
export PYTHONPATH=.
O=gpurun_out/r1b; mkdir -p $O
timeout 1200 python -m pytest tests -q -m gpu -p no:cacheprovider > $O/pytest_gpu.txt 2>&1
python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.txt 2>&1
python bench.py > $O/bench_bicg_mvt.json 2> $O/bench.err
python bench.py --workload atax --cpu-seconds 3 > $O/bench_atax.json 2>> $O/bench.err
python bench.py --workload kmeans --cpu-seconds 3 > $O/bench_kmeans.json 2>> $O/bench.err
python bench.py --workload gesummv --cpu-seconds 3 > $O/bench_gesummv.json 2>> $O/bench.err
python bench.py --impl reference --steps 3 > $O/bench_reference.json 2>> $O/bench.err
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_bicg_mvt.csv python bench.py --steps 2 --warmup 3 --no-study --no-e2e --cpu-seconds 0 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:"fused_kernel" -s 2 -c 2 -o $O/prof_fused python bench.py --steps 1 --warmup 3 --no-study --no-e2e --cpu-seconds 0 > $O/prof_fused.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:"fused_kernel" -s 3 -c 1 -o $O/prof_fused_atax python bench.py --workload atax --steps 1 --warmup 3 --no-study --no-e2e --cpu-seconds 0 > $O/prof_fused_atax.log 2>&1
