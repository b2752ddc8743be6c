export PYTHONPATH=.
OUT=gpurun_out/$1; shift; mkdir -p $OUT
timeout 900 python -m pytest tests -m gpu -x -q -k "tod or round_trip or scan or should_zero or fp32 or gamma or wide or non_power" > $OUT/pytest.txt 2>&1; tail -2 $OUT/pytest.txt
for lib in paper_conf_sc_demeurekktbb23_b200/libtoastb200.so "$@"; do
  v=$(basename $lib .so)
  for w in c2 c3 c5; do
    TOASTB200_LIB=$(readlink -f $lib) timeout 300 python scripts/bench_ops.py --workload $w --only "pointing_to_tod,pointing_to_map" 2>&1 | python -c "
import sys, json
for l in sys.stdin:
    try: d=json.loads(l); print('$v', d['workload'], d['entry'][:28], '%.4f ms'%d['ms'])
    except Exception: pass"
  done
done | tee $OUT/variants.txt
