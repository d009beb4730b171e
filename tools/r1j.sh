export PYTHONPATH=.
timeout 900 python -m pytest tests/test_gpu.py tests/test_dist.py -q -x -p no:cacheprovider > gpurun_out/gpu_tests_r1j.txt 2>&1
rm -f gpurun_out/fused_skip.txt; bash tools/r1i.sh
python bench.py --variant fused --cpu-seconds 2 > gpurun_out/bench_fused_r1j.json 2> gpurun_out/bench_r1j.err
python bench.py --workload atax --variant fused --no-study --no-e2e --cpu-seconds 1 > gpurun_out/bench_atax_fused_r1j.json 2>> gpurun_out/bench_r1j.err
