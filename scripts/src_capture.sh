# GPU box: ncu source-page (SASS) CSV of the fused map kernel for the given workloads.
# Usage: bash scripts/src_capture.sh TAG "c5 c2"
OUT=gpurun_out/$1; mkdir -p $OUT /tmp/rep_$1
export PYTHONPATH=.
for w in $2; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:pointing_to_map -s 3 -c 1 \
    -o /tmp/rep_$1/p_$w python bench.py --workload $w --steps 1 --warmup 3 --soak 0 --no-e2e --no-cpu-baseline > $OUT/ncu_$w.log 2>&1
  ncu -i /tmp/rep_$1/p_$w.ncu-rep --page source --csv --print-source sass > $OUT/src_$w.csv 2>/dev/null
  gzip -f $OUT/src_$w.csv
done
ls -la $OUT
