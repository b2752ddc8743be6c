nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/fp64_microbench scripts/fp64_microbench.cu && /tmp/fp64_microbench > gpurun_out/r02i/microbench.txt 2>&1
TOASTB200_LIB=vbuild/libtoastb200_base.so bash scripts/prof2.sh r02i "c2 c5"
