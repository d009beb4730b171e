#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_kmeans.py -q -x > gpurun_out/km_tests.log 2>&1; echo "rc=$?" >> gpurun_out/km_tests.log
