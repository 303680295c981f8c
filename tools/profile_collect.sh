#!/usr/bin/env bash
# Round profile collection on the GPU box (one GPU): bench lines for every config, the ncu
# launch list + full captures of configs[1] and configs[2] (tools/profile_round.sh), the
# profiles/ summaries made ON the box (tools/make_profiles.py), the raw pages of every
# capture as CSV; the .ncu-rep files are deleted so gpurun_out/ stays under gpurun's 64 MiB.
set -u
OUT=gpurun_out
mkdir -p $OUT/profiles_new
python bench.py > $OUT/bench_default.json 2> $OUT/bench_default.err
python bench.py --config 3 --no-e2e --no-cpu-baseline > $OUT/bench_cfg3.json 2>&1
python bench.py --config 1 --no-e2e --no-cpu-baseline > $OUT/bench_cfg1.json 2>&1
python bench.py --config 4 --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > $OUT/bench_cfg4.json 2>&1
python bench.py --config 5 --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > $OUT/bench_cfg5.json 2>&1
for C in 2 3; do
  case $C in 3) R=paper:none;; *) R=degree:none;; esac
  CFG=$C timeout 900 bash tools/profile_round.sh > $OUT/prof$C.log 2>&1
  python tools/make_profiles.py --round ${ROUND:-r01} --cfg $C --rules $R > /dev/null 2>&1
  for f in $OUT/full_cfg${C}_*.ncu-rep; do
    [ -f "$f" ] && ncu -i "$f" --page raw --csv > "${f%.ncu-rep}.raw.csv" 2>/dev/null
    rm -f "$f"
  done
  cp profiles/${ROUND:-r01}_ncu_cfg$C.md $OUT/profiles_new/
done
cp profiles/traffic.json $OUT/profiles_new/
du -sh $OUT
