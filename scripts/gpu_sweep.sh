timeout -s KILL 900 python -m pytest tests -m gpu -q --timeout 200 -x 2>&1 | tail -3
timeout -s KILL 300 python scripts/spmm_sweep.py reddit 256 44 2>&1 | grep -v Warn
timeout -s KILL 300 python scripts/spmm_sweep.py proteins 128 112 8 2>&1 | grep -v Warn
