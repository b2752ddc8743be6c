# GPU box: per-entry timings of variant libraries on C2 and C3 (A1, A4 and the fused pair).
for v in u0 u1 u2 u3 u4 u5; do
  for w in c2 c3; do
    TOASTB200_LIB=vbuild/libtoastb200_$v.so timeout 300 python scripts/bench_ops.py --workload $w --only "(A1),(A4),(A2),(A3),(A5)" 2>&1 | python -c "
import sys, json
for l in sys.stdin:
    try: d=json.loads(l); print('$v', d['workload'], d['entry'][:28], '%.4f ms'%d['ms'], 'hbm %.2f'%d.get('hbm_frac',0))
    except Exception: pass"
  done
done
