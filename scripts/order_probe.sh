# GPU box: item-order variants — time (tune_fused) and DRAM bytes of one fused launch at C5.
# Usage: bash scripts/order_probe.sh TAG lib1.so lib2.so ...
TAG=$1; shift; OUT=gpurun_out/$TAG; mkdir -p $OUT
export PYTHONPATH=.
for w in c5 c2; do timeout 900 python scripts/tune_fused.py --workload $w "$@" >> $OUT/tune.jsonl 2>&1; done
for lib in "$@"; do
  n=$(basename $lib .so)
  TOASTB200_LIB=$(readlink -f $lib) timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum \
    --clock-control none -k regex:pointing_to_map -s 3 -c 1 --csv --log-file $OUT/dram_$n.csv \
    python bench.py --workload c5 --steps 1 --warmup 3 --soak 0 --no-e2e --no-cpu-baseline > /dev/null 2>&1
  grep -h "dram__bytes\|gpu__time" $OUT/dram_$n.csv | awk -F'","' -v n=$n '{print n, $(NF-2), $(NF-1), $NF}'
done
cat $OUT/tune.jsonl | python -c "
import sys, json
for l in sys.stdin:
    try: d=json.loads(l); print(d.get('wl'), d['lib'].split('/')[-1], '%.4f ms'%d['ms'] if 'ms' in d else d.get('error','')[-300:])
    except Exception as e: print(l[:200])"
