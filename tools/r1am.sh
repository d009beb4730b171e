#!/bin/bash
# N = 2 bench paths on one GPU (ranks share cuda:0 over gloo): NCCL-free fused peer ATAX and the default
export PYTHONPATH=.
O=gpurun_out/r1am; mkdir -p $O
CATT_BENCH_SHARE_GPU=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29611 bench.py --gpus 2 --workload atax --variant fused_peer --steps 5 --warmup 3 --no-study --no-e2e --cpu-seconds 0 > $O/atax_peer_n2.json 2> $O/atax_peer_n2.err
CATT_BENCH_SHARE_GPU=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29612 bench.py --gpus 2 --workload kmeans_iter --steps 5 --warmup 3 --no-study --no-e2e --cpu-seconds 0 > $O/kmi_n2.json 2> $O/kmi_n2.err
