export PYTHONPATH=.
python scripts/debug_tod.py
python scripts/tune_fused.py --workload c2; python scripts/tune_fused.py --workload c3; python scripts/tune_fused.py --workload c5
