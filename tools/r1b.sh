export PYTHONPATH=.
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_r1b.txt 2>&1
python bench.py > gpurun_out/bench_r1b.json 2> gpurun_out/bench_r1b.err
python bench.py --workload kmeans --no-e2e > gpurun_out/bench_kmeans_r1b.json 2> gpurun_out/bench_kmeans_r1b.err
python bench.py --impl reference --steps 3 > gpurun_out/bench_ref_r1b.json 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_r1b.csv python bench.py --steps 2 --warmup 3 --no-study --no-e2e --cpu-seconds 0 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:"row_warp|col_warp" -s 4 -c 2 -o gpurun_out/prof_r1b python bench.py --steps 1 --warmup 3 --no-study --no-e2e --cpu-seconds 0 > gpurun_out/prof_r1b.log 2>&1
ls -la gpurun_out
