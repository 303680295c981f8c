set -u
OUT=gpurun_out; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q > $OUT/r02i_pytest.log 2>&1; echo "rc=$?" >> $OUT/r02i_pytest.log
tail -2 $OUT/r02i_pytest.log
for lib in "" build_variant/sub32/libtc_b200.so build_variant/minb6/libtc_b200.so build_variant/sub32minb6/libtc_b200.so; do
  echo "== lib $lib"
  TC_B200_LIB=$lib python tools/kprof.py --config 4 --rule degree:paper --reps 2 2>&1 | sed -n 2,2p
  TC_B200_LIB=$lib python tools/kprof.py --config 3 --rule paper:none --reps 3 2>&1 | sed -n 2,2p
  TC_B200_LIB=$lib python tools/kprof.py --config 5 --rule paper:paper --reps 1 2>&1 | sed -n 2,2p
done
python tools/ab_option.py --config 2 --option vtiles --values 1,2,4,8 --rule degree:none --reps 3
