#!/bin/bash
# BICG+MVT with the column partials all-reduced inside the fused kernel
# (catt_dual_group_peer): GPU tests (processes sharing cuda:0), bench N=1,
# and N=2 on one shared GPU (functional only)
export PYTHONPATH=.
O=gpurun_out/r1bp; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_peer.py tests/test_gpu.py -q -x -k "peer or dual" > $O/pytest.txt 2>&1; echo "rc=$?" >> $O/pytest.txt
timeout 600 python bench.py --variant fused_peer --no-study --steps 30 --cpu-seconds 0 > $O/bench_peer_n1.json 2> $O/bench_peer_n1.err
CATT_BENCH_SHARE_GPU=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29613 bench.py --gpus 2 --variant fused_peer --steps 5 --warmup 3 --no-study --no-e2e --cpu-seconds 0 > $O/bench_peer_n2.json 2> $O/bench_peer_n2.err
CATT_BENCH_SHARE_GPU=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29614 bench.py --gpus 2 --steps 5 --warmup 3 --no-study --no-e2e --cpu-seconds 0 > $O/bench_fused_n2.json 2> $O/bench_fused_n2.err
