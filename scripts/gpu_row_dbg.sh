# row GEMM component timing (TIMING ONLY variants, MGGCN_ROW_DBG): launch list of the gemm_rows kernels
for L in sweep_libs/lib_dbg*.so; do
  MGGCN_LIB=$L timeout -s KILL 300 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:gemm_rows -c 10 --csv \
     python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --no-cache-l0 2>/dev/null > gpurun_out/rowdbg_$(basename $L .so).csv
done
