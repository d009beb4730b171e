export PYTHONPATH=.
timeout 900 python -m pytest tests/test_gpu.py tests/test_dist.py -q -x -p no:cacheprovider > gpurun_out/gpu_tests_r1g.txt 2>&1
for v in fused coop staged; do python bench.py --variant $v --no-study --cpu-seconds 1 > gpurun_out/bench_${v}_r1g.json 2>> gpurun_out/bench_r1g.err; done
python bench.py --workload atax --variant fused --no-study --no-e2e --cpu-seconds 1 > gpurun_out/bench_atax_fused_r1g.json 2>> gpurun_out/bench_r1g.err
python bench.py --workload atax --variant coop --no-study --no-e2e --cpu-seconds 1 > gpurun_out/bench_atax_coop_r1g.json 2>> gpurun_out/bench_r1g.err
ncu --set full --clock-control none --import-source on -k regex:"fused_kernel" -s 2 -c 2 -o gpurun_out/prof_fused_r1g python bench.py --variant fused --steps 1 --warmup 3 --no-study --no-e2e --cpu-seconds 0 > gpurun_out/prof_fused_r1g.log 2>&1
