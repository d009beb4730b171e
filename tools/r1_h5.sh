#!/bin/bash
export PYTHONPATH=.
O=gpurun_out/r1h5; mkdir -p $O
timeout 2400 python tools/heldout2_study.py --set5 > $O/heldout5.log 2>&1
cp gpurun_out/heldout5_study.json $O/ 2>/dev/null
