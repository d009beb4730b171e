export PYTHONPATH=.
python bench.py > gpurun_out/bench_r1e.json 2> gpurun_out/bench_r1e.err
python bench.py --workload kmeans --no-e2e --cpu-seconds 3 > gpurun_out/bench_kmeans_r1e.json 2>> gpurun_out/bench_r1e.err
python bench.py --workload gesummv --no-e2e --cpu-seconds 3 > gpurun_out/bench_gesummv_r1e.json 2>> gpurun_out/bench_r1e.err
ncu --set full --clock-control none --import-source on -k regex:"row_tma|col_tma|col_cluster|col_warp" -c 4 -o gpurun_out/prof_r1e python tools/explore_one.py > gpurun_out/prof_r1e.log 2>&1
