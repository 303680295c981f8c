set -u
OUT=gpurun_out; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_configs.py -x -q > $OUT/r02b_pytest.log 2>&1; echo "rc=$?" >> $OUT/r02b_pytest.log
tail -3 $OUT/r02b_pytest.log
for c in 4 3 2; do timeout 600 python bench.py --config $c --no-e2e --no-cpu-baseline --steps 5 --warmup 2 > $OUT/r02b_bench_cfg$c.json 2>&1; python -c "
import json; d=json.load(open('$OUT/r02b_bench_cfg$c.json')); print($c, d['value'], d['count_ms'], d['kernels_ms_per_step'].get('count'), d['stages_ms'])"; done
TAG=r02b STEPS=full bash tools/gpu_round.sh > /dev/null 2>&1
cat $OUT/r02b_full_cfg4_*.summary.txt
