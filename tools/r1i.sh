export PYTHONPATH=.
for sk in 0 1 2 3 4 7; do echo "skip=$sk" >> gpurun_out/fused_skip.txt; CATT_DEBUG_FUSED_SKIP=$sk python bench.py --variant fused --no-study --no-e2e --cpu-seconds 0 2>/dev/null | python -c "import json,sys; d=json.load(sys.stdin); print(d['ms_per_step'], {k:v['ms'] for k,v in d['loops'].items()})" >> gpurun_out/fused_skip.txt; done
python bench.py --variant coop --no-study --no-e2e --cpu-seconds 0 2>/dev/null | python -c "import json,sys; d=json.load(sys.stdin); print('coop', d['ms_per_step'], {k:v['ms'] for k,v in d['loops'].items()})" >> gpurun_out/fused_skip.txt
