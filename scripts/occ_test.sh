for b in 1 2; do TB_BPS=$b python scripts/tune_fused.py --workload c2 vbuild/libtoastb200_occ.so; TB_BPS=$b python scripts/tune_fused.py --workload c5 vbuild/libtoastb200_occ.so; done
