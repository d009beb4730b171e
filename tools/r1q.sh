#!/bin/bash
# session-3 check: GPU tests, smoke, default bench, read-only HBM ceiling probe
export PYTHONPATH=.
O=gpurun_out/r1q; mkdir -p $O
nvidia-smi > $O/nvsmi.txt 2>&1
timeout 300 ./tools/read_probe 7 > $O/read_probe.txt 2>&1
timeout 1500 python -m pytest tests -q -m gpu -p no:cacheprovider > $O/pytest_gpu.txt 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.txt 2>&1; echo "smoke rc=$?" >> $O/smoke.txt
timeout 600 python bench.py > $O/bench_bicg_mvt.json 2> $O/bench.err
