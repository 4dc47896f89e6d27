# narrow-width SpMM sweep (shape overrides x occupancy variants)
for lib in "" sweep_libs/minb3.so sweep_libs/minb4.so sweep_libs/w4m8.so; do
  for shp in "" "8,2" "16,1" "32,1"; do
    echo "== lib=${lib:-default} shape=${shp:-auto}"
    MGGCN_LIB=$lib MGGCN_SPMM_SHAPE=$shp timeout -s KILL 300 python scripts/spmm_sweep.py reddit 48 2>&1 | grep "width"
  done
  echo "== lib=${lib:-default} wide"
  MGGCN_LIB=$lib timeout -s KILL 300 python scripts/spmm_sweep.py reddit 256 2>&1 | grep "dir 0"
done
