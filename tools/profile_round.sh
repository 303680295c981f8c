#!/usr/bin/env bash
# Round profile capture (run on the GPU box through gpurun, one GPU, never multi-rank):
#   1. per-launch device times of one bench invocation (cold-cache, serialised: use SHARES)
#   2. one `ncu --set full` capture of each top kernel of the default bench workload
# Outputs land in gpurun_out/; tools/make_profiles.py turns them into profiles/ summaries.
set -u
CFG=${CFG:-2}
# directing / ordering of the bench line for this config (bench.py CONFIG_RULES)
case $CFG in 3) D=paper; R=none;; 4) D=degree; R=paper;; 5) D=paper; R=paper;; *) D=degree; R=none;; esac
OUT=gpurun_out
mkdir -p $OUT
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches_cfg${CFG}.csv \
    python bench.py --config $CFG --steps 2 --warmup 1 --no-e2e --no-cpu-baseline > $OUT/launches_bench.log 2>&1
for K in rs_pass_kernel count_small count_large count_range unique_kernel rs_hist_kernel; do
  ITERS=2 ncu --set full --clock-control none --import-source on -k regex:$K -s 1 -c 1 -o $OUT/full_cfg${CFG}_$K \
      python tools/timeline.py $CFG $D $R > /dev/null 2>&1 || true
done
ls -la $OUT
