#!/bin/bash
export PYTHONPATH=.
O=gpurun_out/r1h8; mkdir -p $O
timeout 2400 python tools/heldout2_study.py --set8 > $O/heldout8.log 2>&1
cp gpurun_out/heldout8_study.json $O/ 2>/dev/null
