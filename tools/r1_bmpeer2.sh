#!/bin/bash
export PYTHONPATH=.
O=gpurun_out/r1bp2; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_peer.py -q -x > $O/pytest.txt 2>&1; echo "rc=$?" >> $O/pytest.txt
for v in 0 1; do
  if [ $v = 1 ]; then export CATT_PEER_FENCE_ALL=1; fi
  timeout 600 python bench.py --variant fused_peer --no-study --no-e2e --steps 30 --cpu-seconds 0 > $O/bench_peer_fa$v.json 2> $O/bench_peer_fa$v.err
  timeout 600 python bench.py --workload atax --variant fused_peer --no-study --no-e2e --steps 10 --cpu-seconds 0 > $O/bench_atax_peer_fa$v.json 2> $O/bench_atax_peer_fa$v.err
done
unset CATT_PEER_FENCE_ALL
timeout 600 python bench.py --workload atax --no-study --no-e2e --steps 10 --cpu-seconds 0 > $O/bench_atax_fused.json 2> $O/bench_atax_fused.err
