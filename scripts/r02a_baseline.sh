set -u
OUT=gpurun_out/r02a; mkdir -p $OUT
nproc > $OUT/host.txt; free -g >> $OUT/host.txt; nvidia-smi >> $OUT/host.txt 2>&1
bash scripts/fp64_peak.sh r02a > $OUT/fp64.log 2>&1
for w in c2 c5; do
timeout 600 ncu --set full --clock-control none --import-source on -k regex:pointing_to_map -s 4 -c 1 \
    -o $OUT/prof_fused_$w python bench.py --workload $w --steps 2 --warmup 3 --soak 0 --no-e2e --no-cpu-baseline > $OUT/ncu_full_$w.log 2>&1
done
echo done
