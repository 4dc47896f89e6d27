# SpMM column-window sweep (MGGCN_SPMM_WIN) on Reddit/Products shapes.
for WL in reddit products; do
for WIN in 512 256 128 64 32; do
  MGGCN_SPMM_WIN=$WIN timeout -s KILL 400 python scripts/spmm_sweep.py $WL 256 48 2>&1 | grep -v Warn
done
done
