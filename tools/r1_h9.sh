#!/bin/bash
export PYTHONPATH=.
O=gpurun_out/r1h9; mkdir -p $O
timeout 2400 python tools/heldout2_study.py --set9 > $O/heldout9.log 2>&1
cp gpurun_out/heldout9_study.json $O/ 2>/dev/null
