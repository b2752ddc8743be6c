export PYTHONPATH=.
python scripts/debug_tod.py
bash scripts/tune_run.sh r02o "c2 c3 c5" vbuild/libtoastb200_s3.so vbuild/libtoastb200_s2.so
