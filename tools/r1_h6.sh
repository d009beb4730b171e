#!/bin/bash
export PYTHONPATH=.
O=gpurun_out/r1h6; mkdir -p $O
timeout 2400 python tools/heldout2_study.py --set6 > $O/heldout6.log 2>&1
cp gpurun_out/heldout6_study.json $O/ 2>/dev/null
