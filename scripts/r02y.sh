OUT=gpurun_out/r02y; mkdir -p $OUT
export PYTHONPATH=.
timeout 600 python -m pytest tests -m gpu -x -q -k "tod or round_trip or scan or should_zero" > $OUT/pytest_scan.txt 2>&1
timeout 300 python bench.py --workload c5m --steps 5 --warmup 3 --no-cpu-baseline > $OUT/bench_c5m.json 2> $OUT/bench_c5m.err
timeout 300 python bench.py --workload c3rt --steps 10 --warmup 3 --no-cpu-baseline > $OUT/bench_c3rt.json 2> $OUT/bench_c3rt.err
for w in c2 c5; do timeout 300 python scripts/bench_ops.py --workload $w > $OUT/ops_$w.jsonl 2>&1; done
tail -3 $OUT/pytest_scan.txt
for f in c5m c3rt; do python -c "
import json; d=json.loads(open('$OUT/bench_$f.json').read().strip().splitlines()[-1]); r=d['roofline']
print('$f', '%.3e'%d['value'], 'ms/step %.4f'%d['ms_per_step'], 'frac %.3f'%r['frac'], 'kern %.4f'%r['kernel_ms'])"; done
cat $OUT/ops_*.jsonl | python -c "
import sys, json
for l in sys.stdin:
    try: d=json.loads(l); print(d['workload'], d['entry'][:34], '%.4f ms'%d['ms'], 'hbm %.2f'%d.get('hbm_frac',0))
    except Exception: pass"
