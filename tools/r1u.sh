#!/bin/bash
export PYTHONPATH=.
O=gpurun_out/r1u; mkdir -p $O
timeout 600 python -m pytest tests/test_gpu.py -q -x -k "fused or dual or kmeans" -p no:cacheprovider > $O/pytest.txt 2>&1
for V in staged coop; do
  echo "$V $(timeout 120 python bench.py --workload kmeans --variant $V --steps 30 --warmup 5 --no-study --no-e2e --cpu-seconds 0 2>$O/km_$V.err | python -c 'import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(d["ms_per_step"], [(k, v["ms"]) for k, v in d["loops"].items()])')" >> $O/kmeans_variants.txt
done
echo "fused default $(timeout 120 python bench.py --steps 30 --warmup 5 --no-study --no-e2e --cpu-seconds 0 2>/dev/null | python -c 'import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(d["ms_per_step"], [(k, v["ms"]) for k, v in d["loops"].items()])')" >> $O/kmeans_variants.txt
ncu --set full --clock-control none -k regex:kmeans_coop -s 3 -c 1 -o $O/prof_km_coop python bench.py --workload kmeans --variant coop --steps 1 --warmup 3 --no-study --no-e2e --cpu-seconds 0 > $O/ncu.log 2>&1
