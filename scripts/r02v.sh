OUT=gpurun_out/r02v; mkdir -p $OUT
export PYTHONPATH=.
timeout 900 python -m pytest tests -m gpu -x -q -k "pointing_detector or stokes or unwrapped or gamma or noise_weighted or round_trip" > $OUT/pytest.txt 2>&1; tail -2 $OUT/pytest.txt
for w in c2 c3 c5; do timeout 300 python scripts/bench_ops.py --workload $w > $OUT/ops_$w.jsonl 2>&1; done
timeout 600 python bench.py --workload c5 --steps 10 --warmup 3 --no-cpu-baseline --reduce scatter > $OUT/bench_c5_compact.json 2> $OUT/bench_c5_compact.err
timeout 600 python bench.py --workload c3 --steps 10 --warmup 3 --no-cpu-baseline > $OUT/bench_c3.json 2> $OUT/bench_c3.err
for f in c5_compact c3; do python -c "
import json; d=json.loads([l for l in open('$OUT/bench_$f.json') if l.startswith('{')][-1]); r=d['roofline']
print('$f', '%.3e'%d['value'], 'ms/step %.4f'%d['ms_per_step'], 'kern %.4f'%r['kernel_ms'], d['clocks'], d['config'].get('map_domain'), 'e2e %.3e'%d['e2e']['value'])"; done
cat $OUT/ops_*.jsonl | python -c "
import sys, json
for l in sys.stdin:
    try: d=json.loads(l); print(d['workload'], d['entry'][:34], '%.4f ms'%d['ms'], 'hbm %.2f'%d.get('hbm_frac',0))
    except Exception: pass"
