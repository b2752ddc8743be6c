export TOASTB200_LIB=vbuild/libtoastb200_s3.so
timeout 600 ncu --set full --clock-control none --import-source on -k regex:pointing_to_map -s 4 -c 1 -o gpurun_out/r02p/prof_c2 python bench.py --workload c2 --steps 2 --warmup 3 --soak 0 --no-e2e --no-cpu-baseline > gpurun_out/r02p/ncu_c2.log 2>&1
