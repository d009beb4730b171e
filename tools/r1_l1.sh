#!/bin/bash
export PYTHONPATH=.
O=gpurun_out/l1; mkdir -p $O
timeout 2400 ncu --metrics l1tex__t_sector_hit_rate.pct,dram__bytes_read.sum,gpu__time_duration.sum --clock-control none \
  -k regex:"row_thread|kmeans_kernel|syrk_thread|syr2k_thread|km_transpose_thread" --csv --log-file $O/l1.csv \
  python tools/l1_study.py profiles/r1n bicg_mvt kmeans gesummv syr2k kmeans_iter atax256 > $O/cases.txt 2> $O/err.txt
python tools/l1_parse.py $O/cases.txt $O/l1.csv > $O/l1_table.txt 2>&1
