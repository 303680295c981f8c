set -u
OUT=gpurun_out; mkdir -p $OUT
TAG=r02d STEPS="tests bench launches full" bash tools/gpu_round.sh
for c in 3 2 5; do timeout 900 python bench.py --config $c --no-e2e --no-cpu-baseline --steps 3 --warmup 2 > $OUT/r02d_bench_cfg$c.json 2>&1; python -c "
import json; d=json.load(open('$OUT/r02d_bench_cfg$c.json')); print($c, d['value'], d['count_ms'], d['whole_path'], d['stages_ms'])"; done
