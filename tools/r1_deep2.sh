#!/bin/bash
export PYTHONPATH=.
O=gpurun_out/r1deep2; mkdir -p $O
timeout 900 python -m pytest tests -m gpu -q -x -k "syrk or syr2k or corr or gemm or tiled" > $O/pytest.txt 2>&1; echo "rc=$?" >> $O/pytest.txt
timeout 900 python bench.py --workload syr2k > $O/bench_syr2k.json 2> $O/bench_syr2k.err
timeout 600 ncu --set full --clock-control none --import-source on -k regex:tiled_kernel -s 3 -c 1 -o $O/ncu_syr2k -f python bench.py --workload syr2k --steps 1 --warmup 3 --no-study --no-e2e --cpu-seconds 0 > $O/ncu.log 2>&1
