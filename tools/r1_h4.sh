#!/bin/bash
export PYTHONPATH=.
O=gpurun_out/r1h4; mkdir -p $O
timeout 2400 python tools/heldout2_study.py --set4 > $O/heldout4.log 2>&1
cp gpurun_out/heldout4_study.json $O/ 2>/dev/null
