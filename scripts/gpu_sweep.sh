timeout -s KILL 600 python -m pytest tests/test_gpu_kernels.py -q --timeout 120 -k spmm -x 2>&1 | tail -1
timeout -s KILL 300 python scripts/spmm_sweep.py reddit 256 48 2>&1 | grep "dir 0"
timeout -s KILL 300 python scripts/spmm_sweep.py products 256 104 48 2>&1 | grep "dir 0"
