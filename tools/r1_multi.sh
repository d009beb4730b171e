#!/bin/bash
# The N > 1 bench path on one GPU: 2 ranks sharing cuda:0 over gloo (a correctness smoke, not a measurement).
export PYTHONPATH=. CATT_BENCH_SHARE_GPU=1
O=gpurun_out/multi; mkdir -p $O
for w in bicg_mvt atax gesummv kmeans_iter kmeans; do
  timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29517 \
    bench.py --workload $w --gpus 2 --steps 3 --warmup 3 --no-study --cpu-seconds 0 > $O/$w.json 2> $O/$w.err
  echo "$w rc=$?" >> $O/rc.txt
done
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29518 \
  bench.py --impl reference --gpus 2 --steps 3 --warmup 3 > $O/reference.json 2> $O/reference.err
echo "reference rc=$?" >> $O/rc.txt
