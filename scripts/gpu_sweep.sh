for L in "" a b c d e f; do
  LIB=""; [ -n "$L" ] && LIB=scratch_libs/libmggcn_$L.so
  echo "VARIANT=$L"; MGGCN_LIB=$LIB timeout -s KILL 300 python scripts/spmm_sweep.py reddit 256 44 2>&1 | grep "dir 0"
done
