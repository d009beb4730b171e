export PYTHONPATH=.
timeout 900 python -m pytest tests/test_gpu.py -q -x -p no:cacheprovider -k "fused or dual" > gpurun_out/gpu_tests_r1l.txt 2>&1
for cl in 1 2 4 8; do echo "cluster=$cl" >> gpurun_out/fused_cl.txt; CATT_FUSED_CLUSTER=$cl python bench.py --variant fused --no-study --no-e2e --cpu-seconds 0 2>>gpurun_out/fused_cl.err | python -c "import json,sys; d=json.load(sys.stdin); print(d['ms_per_step'], {k:v['ms'] for k,v in d['loops'].items()})" >> gpurun_out/fused_cl.txt; done
echo "atax cl8" >> gpurun_out/fused_cl.txt; python bench.py --workload atax --variant fused --no-study --no-e2e --cpu-seconds 0 --steps 5 2>>gpurun_out/fused_cl.err | python -c "import json,sys; d=json.load(sys.stdin); print(d['ms_per_step'], d['value'])" >> gpurun_out/fused_cl.txt
