OUT=gpurun_out/r01zb; mkdir -p $OUT
for v in a4dt1 a4dt2 a4dt4; do
  for wl in c2 c3; do TOASTB200_LIB=build/variants/libtoastb200_$v.so timeout 600 python scripts/bench_ops.py --workload $wl --reps 10 --only "build_noise" > $OUT/ops_${v}_$wl.jsonl 2>&1; done
done
TOASTB200_LIB=build/variants/libtoastb200_a4dt2.so timeout 900 python -m pytest tests/test_parity_gpu.py -x -q -k "build_noise or round_trip" > $OUT/pytest_a4.log 2>&1; echo "rc=$?" >> $OUT/pytest_a4.log
