#!/bin/bash
export PYTHONPATH=.
O=gpurun_out/r1al; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_kmeans.py tests/test_gpu.py -q -x -k "kmeans" -p no:cacheprovider > $O/pytest.txt 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.txt 2>&1; echo "rc=$?" >> $O/smoke.txt
echo "kmeans_iter $(timeout 300 python bench.py --workload kmeans_iter --steps 20 --warmup 3 --no-study --no-e2e --cpu-seconds 0 2>$O/ki.err | python -c 'import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(d["ms_per_step"], [(k, v["ms"]) for k, v in d["loops"].items()], d["roofline"]["frac"])')" >> $O/bench.txt
