#!/usr/bin/env bash
# One gpurun call: GPU tests, the default bench line, the ncu launch list of the bench
# workload and `ncu --set full` captures of its count kernels (read back here with
# tools/ncu_summary.py).  Usage: STEPS="tests bench launches full" bash tools/gpu_round.sh
set -u
OUT=gpurun_out
mkdir -p $OUT
STEPS=${STEPS:-"tests bench launches full"}
CFG=${CFG:-4}
case $CFG in 3) D=paper; R=none;; 4) D=degree; R=paper;; 5) D=paper; R=paper;; *) D=degree; R=none;; esac
TAG=${TAG:-r02}
for S in $STEPS; do
  case $S in
    tests)
      timeout ${TEST_TIMEOUT:-1800} python -m pytest tests -m gpu -q ${PYTEST_ARGS:-} > $OUT/${TAG}_pytest_gpu.log 2>&1
      echo "pytest rc=$?" >> $OUT/${TAG}_pytest_gpu.log ;;
    bench)
      timeout 1200 python bench.py ${BENCH_ARGS:-} > $OUT/${TAG}_bench_cfg$CFG.json 2> $OUT/${TAG}_bench_cfg$CFG.err ;;
    aorder)
      # host A-order greedy micro-benchmark on the box's idle cores (d~ of the bench workload)
      g++ -O3 -std=c++17 -pthread -Iinclude tools/aorder_bench.cpp -o /tmp/aorder_bench && \
      python tools/dump_od.py $CFG $D /tmp/od.u32 && /tmp/aorder_bench /tmp/od.u32 5 > $OUT/${TAG}_aorder_bench.txt 2>&1
      cat $OUT/${TAG}_aorder_bench.txt ;;
    launches)
      timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/${TAG}_launches_cfg$CFG.csv \
        python bench.py --config $CFG --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > $OUT/${TAG}_launches_cfg$CFG.log 2>&1 ;;
    full)
      for K in ${KERNELS:-count_large count_small}; do
        ITERS=1 timeout 900 ncu --set full --clock-control none --import-source on -k regex:$K -s 0 -c 1 \
          -o $OUT/${TAG}_full_cfg${CFG}_$K python tools/timeline.py $CFG $D $R > $OUT/${TAG}_full_cfg${CFG}_$K.log 2>&1
        if [ -f $OUT/${TAG}_full_cfg${CFG}_$K.ncu-rep ]; then
          ncu -i $OUT/${TAG}_full_cfg${CFG}_$K.ncu-rep --page raw --csv > $OUT/${TAG}_full_cfg${CFG}_$K.raw.csv 2>/dev/null
          ncu -i $OUT/${TAG}_full_cfg${CFG}_$K.ncu-rep --page source --csv > $OUT/${TAG}_full_cfg${CFG}_$K.source.csv 2>/dev/null
          python tools/ncu_summary.py $OUT/${TAG}_full_cfg${CFG}_$K.ncu-rep > $OUT/${TAG}_full_cfg${CFG}_$K.summary.txt 2>&1
          # .ncu-rep files are ~30 MB: gpurun copies back <= 64 MiB, the CSV pages suffice
          [ -n "${KEEP_REP:-}" ] || rm -f $OUT/${TAG}_full_cfg${CFG}_$K.ncu-rep
        fi
      done ;;
  esac
done
du -sh $OUT 2>/dev/null
tail -3 $OUT/${TAG}_pytest_gpu.log 2>/dev/null
cat $OUT/${TAG}_bench_cfg$CFG.json 2>/dev/null | head -c 3000; echo
cat $OUT/${TAG}_full_cfg${CFG}_*.summary.txt 2>/dev/null | head -60
