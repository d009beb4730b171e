#!/bin/bash
# SYRK/SYR2K tiled: parity tests, then bench with both register budgets.
mkdir -p gpurun_out
python -m pytest tests/test_gpu.py -x -q -k "syr2k or syrk" > gpurun_out/syr2k_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/syr2k_tests.log
for w in syrk syr2k; do for mb in 1 2; do
CATT_TILED_MINB=$mb timeout 300 python bench.py --workload $w --steps 10 --warmup 3 --no-study --cpu-seconds 0 > gpurun_out/${w}_mb$mb.json 2> gpurun_out/${w}_mb$mb.err
done; done
