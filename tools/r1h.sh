export PYTHONPATH=.
timeout 900 python -m pytest tests/test_gpu.py -q -x -p no:cacheprovider -k "fused or dual" > gpurun_out/gpu_tests_r1h.txt 2>&1
python bench.py --variant fused --no-study --cpu-seconds 1 > gpurun_out/bench_fused_r1h.json 2>> gpurun_out/bench_r1h.err
python bench.py --workload atax --variant fused --no-study --no-e2e --cpu-seconds 1 > gpurun_out/bench_atax_fused_r1h.json 2>> gpurun_out/bench_r1h.err
ncu --set full --clock-control none --import-source on -k regex:"fused_kernel" -s 2 -c 1 -o gpurun_out/prof_fused_r1h python bench.py --variant fused --steps 1 --warmup 3 --no-study --no-e2e --cpu-seconds 0 > gpurun_out/prof_fused_r1h.log 2>&1
