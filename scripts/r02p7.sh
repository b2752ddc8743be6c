#!/bin/bash
# GPU box: C2/C3 A/B (current vs PIPE at every nside) + ncu --set full of the current kernel on C5.
TAG=$1; OUT=gpurun_out/$TAG; mkdir -p $OUT
export PYTHONPATH=.
for w in c2 c3; do timeout 900 python scripts/tune_fused.py --workload $w vbuild/libtoastb200_cur.so vbuild/libtoastb200_pipeall.so >> $OUT/tune.jsonl 2>&1; done
cat $OUT/tune.jsonl
TOASTB200_LIB=$(readlink -f vbuild/libtoastb200_pipeall.so) timeout 900 python -m pytest tests/test_parity_gpu.py -x -q -m gpu -k "fused" > $OUT/pytest_pipeall.log 2>&1; tail -1 $OUT/pytest_pipeall.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:pointing_to_map -s 4 -c 1 \
    -o $OUT/prof_c5 python bench.py --workload c5 --steps 2 --warmup 3 --soak 0 --no-e2e --no-cpu-baseline > $OUT/ncu_c5.log 2>&1
echo done
