set -u
OUT=gpurun_out; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "shorter or closed or random or config1 or multi_piece or schedules" > $OUT/r02h_pytest.log 2>&1; echo "rc=$?" >> $OUT/r02h_pytest.log
tail -2 $OUT/r02h_pytest.log
python tools/kprof.py --config 4 --rule degree:paper --reps 2 2>&1 | head -3
python tools/kprof.py --config 3 --rule paper:none --reps 3 2>&1 | head -3
python tools/kprof.py --config 5 --rule paper:paper --reps 1 2>&1 | head -3
