#!/bin/bash
export PYTHONPATH=.
O=gpurun_out/r1z; mkdir -p $O
timeout 2400 python tools/heldout2_study.py --set3 > $O/heldout3.log 2>&1
cp gpurun_out/heldout3_study.json $O/ 2>/dev/null
timeout 900 python -m pytest tests -q -m gpu -p no:cacheprovider > $O/pytest_gpu.txt 2>&1
