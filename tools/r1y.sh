#!/bin/bash
export PYTHONPATH=.
O=gpurun_out/r1y; mkdir -p $O
timeout 2400 python tools/heldout2_study.py > $O/heldout2.log 2>&1
cp gpurun_out/heldout2_study.json $O/ 2>/dev/null
