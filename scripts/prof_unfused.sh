# GPU box: bandwidth probe + ncu --set full of the unfused A1-A5 kernels at C2.  Usage: bash scripts/prof_unfused.sh TAG
OUT=gpurun_out/$1; mkdir -p $OUT
export PYTHONPATH=.
python scripts/bw_probe.py > $OUT/bw_probe.json 2>&1
for k in pointing_detector_kernel:A1 pixels_healpix_kernel:A2 stokes_weights_kernel:A3 build_noise_weighted_kernel:A4 scan_map_kernel:A5; do
  kn=${k%%:*}; e=${k##*:}
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:$kn -s 2 -c 1 \
    -o ${REPDIR:-$OUT}/prof_$e python scripts/bench_ops.py --workload c2 --reps 1 --only "($e)" > $OUT/ncu_$e.log 2>&1
done
