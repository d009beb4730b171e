#!/bin/bash
export PYTHONPATH=.
O=gpurun_out/r1h7; mkdir -p $O
timeout 2400 python tools/heldout2_study.py --set7 > $O/heldout7.log 2>&1
cp gpurun_out/heldout7_study.json $O/ 2>/dev/null
