#!/bin/bash
# One parameterised runner for gpurun calls (replaces round 1's r1*.sh):
#   /usr/local/graft/bin/gpurun --timeout S -- 'bash tools/gpu_jobs.sh <job> [<job> ...]'
# Every job writes under gpurun_out/$TAG/ (TAG defaults to the job list).
# Jobs:
#   smoke     __graft_entry__.smoke()
#   tests     pytest -m gpu (all)
#   occ       the occupancy-API and residency-probe tests only
#   sanitize  compute-sanitizer memcheck / racecheck / synccheck on tools/sanitize_cases.py
#   bench     default bench line (+ the reference arm)
#   benchall  every workload's bench line
#   launches  ncu launch list of the default bench (gpu__time_duration)
#   ncu       ncu --set full of the default bench's dominant kernel
#   tiles     FP32 tile kernels: bit-exact tests, T2 vs tiled_kernel timing, FFMA2 peak probe
#   ncutile   ncu --set full of one tile kernel (NCU_KERNEL, TILE_ONLY)
#   ncut2     ncu --set full of the T2 tile kernel for syrk / syr2k / corr (details csv)
#   sass      per-kernel SASS opcode summary of libcatt.so
#   mcprobe   NVLS multicast support with one visible GPU (tools/multicast_probe)
export PYTHONPATH=.
TAG=${TAG:-$(echo "$@" | tr ' ' '_')}
O=gpurun_out/$TAG
mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw,temperature.gpu --format=csv > $O/nvsmi.txt 2>&1
CS="compute-sanitizer --kernel-name kns=catt --print-limit 50 --error-exitcode 9"
for job in "$@"; do
  case $job in
    smoke)
      timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.txt 2>&1; echo "rc=$?" >> $O/smoke.txt ;;
    tests)
      timeout 2400 python -m pytest tests -m gpu -q -x > $O/pytest_gpu.txt 2>&1; echo "rc=$?" >> $O/pytest_gpu.txt ;;
    occ)
      timeout 600 python -m pytest tests/test_gpu.py -m gpu -q -k "occupancy or residency" > $O/pytest_occ.txt 2>&1; echo "rc=$?" >> $O/pytest_occ.txt ;;
    sanitize_t2)
      S=$O/sanitizer; mkdir -p $S
      for tool in memcheck racecheck synccheck; do
        timeout 1200 $CS --tool $tool python tools/sanitize_cases.py tiles2 > $S/${tool}_tiles2.txt 2>&1; echo "rc=$?" >> $S/${tool}_tiles2.txt
      done ;;
    sanitize|sanitize_mem)
      S=$O/sanitizer; mkdir -p $S
      timeout 1500 $CS --tool memcheck python tools/sanitize_cases.py > $S/memcheck_all.txt 2>&1; echo "rc=$?" >> $S/memcheck_all.txt
      timeout 1200 $CS --tool synccheck python tools/sanitize_cases.py > $S/synccheck_all.txt 2>&1; echo "rc=$?" >> $S/synccheck_all.txt
      # initcheck without the kernel filter: torch's fills (zeros) must be seen as writes
      timeout 1500 compute-sanitizer --print-limit 50 --error-exitcode 9 --tool initcheck python tools/sanitize_cases.py > $S/initcheck_all.txt 2>&1; echo "rc=$?" >> $S/initcheck_all.txt
      [ $job = sanitize_mem ] && continue
      for c in ${SAN_CASES:-gate_sem gate_barrier cta_counter smem_pad staged coop fused fused_graph onekernel kmeans km_iter tiles tiles2}; do
        timeout 900 $CS --tool racecheck --racecheck-report analysis python tools/sanitize_cases.py $c > $S/racecheck_$c.txt 2>&1; echo "rc=$?" >> $S/racecheck_$c.txt
      done
      timeout 900 python -m torch.distributed.run --nnodes 1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 \
        --no-python $CS --tool memcheck python tools/sanitize_cases.py peer > $S/memcheck_peer.txt 2>&1; echo "rc=$?" >> $S/memcheck_peer.txt
      timeout 900 python -m torch.distributed.run --nnodes 1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29534 \
        --no-python $CS --tool racecheck python tools/sanitize_cases.py peer > $S/racecheck_peer.txt 2>&1; echo "rc=$?" >> $S/racecheck_peer.txt
      ;;
    bench)
      timeout 1200 python bench.py > $O/bench.json 2> $O/bench.err; echo "rc=$?" >> $O/bench.err
      timeout 900 python bench.py --impl reference --steps 3 --warmup 3 > $O/bench_reference.json 2> $O/bench_reference.err ;;
    benchall)
      for w in atax bicg_mvt kmeans kmeans_iter gesummv syrk syr2k corr gemm atax256; do
        timeout 1500 python bench.py --workload $w > $O/bench_$w.json 2> $O/bench_$w.err
      done ;;
    launches)
      timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches.csv \
        python bench.py --steps 2 --warmup 3 --no-study --no-e2e --cpu-seconds 0 > $O/launches.log 2>&1 ;;
    ncu)
      timeout 900 ncu --set full --clock-control none --import-source on -k regex:${NCU_KERNEL:-fused} -s 3 -c 1 -o $O/ncu_default -f \
        python bench.py --steps 1 --warmup 3 --no-study --no-e2e --cpu-seconds 0 > $O/ncu_default.log 2>&1 ;;
    mcprobe)
      nvidia-smi topo -m > $O/topo.txt 2>&1
      timeout 120 ./tools/multicast_probe > $O/multicast_probe.txt 2>&1; echo "rc=$?" >> $O/multicast_probe.txt ;;
    tiles)
      timeout 300 python -m pytest tests/test_gpu.py -m gpu -q -k "syrk or syr2k or corr or gemm" > $O/pytest_tiles.txt 2>&1; echo "rc=$?" >> $O/pytest_tiles.txt
      for v in 0 1; do
        CATT_TILED_T2=$v timeout 300 python tools/tile_bench.py > $O/tile_bench_t2_$v.json 2> $O/tile_bench_t2_$v.err
      done
      [ -x tools/ffma_probe ] && timeout 120 ./tools/ffma_probe > $O/ffma_probe.txt 2>&1 ;;
    ncutile)
      timeout 600 ncu --set full --clock-control none --import-source on -k regex:${NCU_KERNEL:-tile2} -s 1 -c 1 -o $O/ncu_tile -f \
        python tools/tile_bench.py --reps 1 --only ${TILE_ONLY:-syrk} > $O/ncu_tile.log 2>&1 ;;
    ncut2)
      for w in syrk syr2k corr; do
        timeout 600 ncu --set full --clock-control none --import-source on -k regex:tile2 -s 1 -c 1 -o $O/ncu_t2_$w -f \
          python tools/tile_bench.py --reps 1 --only $w > $O/ncu_t2_$w.log 2>&1
        ncu -i $O/ncu_t2_$w.ncu-rep --page details --csv > $O/ncu_t2_${w}_details.csv 2>/dev/null
      done ;;
    sass)
      python tools/sass_summary.py paper_conf_icpp_kimhlsh19_b200/libcatt.so > $O/sass_summary.txt 2>&1 ;;
    *)
      echo "unknown job $job" >> $O/errors.txt ;;
  esac
done
ls -la $O > $O/ls.txt
