OUT=gpurun_out/r02r; mkdir -p $OUT
bash scripts/fp64_peak.sh r02r > $OUT/fp64.log 2>&1
timeout 300 python -m pytest tests/test_synth_gpu.py -q > $OUT/synth_test.log 2>&1
free -g > $OUT/free.txt
/usr/bin/time -v timeout 900 python bench.py > $OUT/bench_c4.json 2> $OUT/bench_c4.err
timeout 600 python bench.py --workload c5m --steps 5 --warmup 3 --no-cpu-baseline > $OUT/bench_c5m.json 2> $OUT/bench_c5m.err
timeout 600 python bench.py --workload c3rt --steps 10 --warmup 3 --no-cpu-baseline > $OUT/bench_c3rt.json 2> $OUT/bench_c3rt.err
tail -3 $OUT/synth_test.log
