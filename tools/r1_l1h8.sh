#!/bin/bash
export PYTHONPATH=.
O=gpurun_out/r1l1h8; mkdir -p $O
timeout 1500 ncu --metrics l1tex__t_sector_hit_rate.pct,dram__bytes_read.sum,gpu__time_duration.sum --clock-control none \
  -k regex:"row_thread" --csv --log-file $O/l1.csv python tools/l1_heldout.py profiles/r1h8/heldout8_study.json > $O/l1_cases.txt 2> $O/l1_err.txt
python tools/l1_parse.py $O/l1_cases.txt $O/l1.csv > $O/l1_table.txt 2>&1
