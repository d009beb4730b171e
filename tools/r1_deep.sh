#!/bin/bash
# tiled FP32 kernel: BK = 32 (SYR2K 16) stages in dynamic shared memory vs the default
export PYTHONPATH=.
O=gpurun_out/r1deep; mkdir -p $O
CATT_TILED_DEEP=1 timeout 900 python -m pytest tests -m gpu -q -x -k "syrk or syr2k or corr or gemm or tiled" > $O/pytest_deep.txt 2>&1; echo "rc=$?" >> $O/pytest_deep.txt
for w in syrk syr2k corr gemm; do
  for D in 0 1; do
    CATT_TILED_DEEP=$D timeout 600 python bench.py --workload $w --no-study --steps 20 --no-e2e --cpu-seconds 0 > $O/bench_${w}_deep$D.json 2> $O/bench_${w}_deep$D.err
  done
done
