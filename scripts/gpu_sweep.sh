timeout -s KILL 300 python scripts/spmm_sweep.py reddit 256 44 2>&1 | grep -v Warn
MGGCN_SPMM_CARVEOUT=0 timeout -s KILL 300 python scripts/spmm_sweep.py reddit 256 44 2>&1 | grep -v Warn
PERM_SEED=0 timeout -s KILL 300 python scripts/spmm_sweep.py reddit 256 44 2>&1 | grep -v Warn
