set -u
OUT=gpurun_out; mkdir -p $OUT
TAG=r02j STEPS="tests bench launches full" bash tools/gpu_round.sh
for c in 3 2 1 5; do timeout 900 python bench.py --config $c --no-cpu-baseline --steps 5 --warmup 3 > $OUT/r02j_bench_cfg$c.json 2>&1; python -c "
import json; d=json.load(open('$OUT/r02j_bench_cfg$c.json')); print($c, d['value'], d['count_ms'], d['whole_path']['value'], d['e2e']['value'], d['stages_ms'])"; done
