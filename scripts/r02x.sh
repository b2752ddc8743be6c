OUT=gpurun_out/r02x; mkdir -p $OUT
timeout 300 python bench.py --workload c1 --steps 50 --warmup 5 --no-cpu-baseline > $OUT/bench_c1.json 2> $OUT/bench_c1.err
timeout 300 python bench.py --workload c1 --graph 10 --steps 50 --warmup 5 --no-cpu-baseline > $OUT/bench_c1g.json 2> $OUT/bench_c1g.err
for w in c2 c3; do timeout 300 python scripts/bench_ops.py --workload $w > $OUT/ops_$w.jsonl 2>&1; done
for f in c1 c1g; do python -c "
import json; d=json.loads(open('$OUT/bench_$f.json').read().strip().splitlines()[-1]); r=d['roofline']
print('$f', '%.3e'%d['value'], 'ms/step %.4f'%d['ms_per_step'], 'kern %.4f'%r['kernel_ms'], 'frac %.3f'%r['frac'], 'e2e %.3e'%d['e2e']['value'])"; done
cat $OUT/ops_c2.jsonl | python -c "
import sys, json
for l in sys.stdin:
    try: d=json.loads(l); print(d['workload'], d['entry'][:34], '%.4f ms'%d['ms'], 'hbm %.2f'%d.get('hbm_frac',0))
    except Exception: pass"
