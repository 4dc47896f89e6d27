# row GEMM variants: B_lo loaded vs recomputed (MGGCN_ROW_RAWB) x transform warps (MGGCN_ROW_XF_WARPS)
for L in sweep_libs/lib_rb*_xf*.so; do
  for WL in reddit products; do
    MGGCN_LIB=$L timeout -s KILL 300 python bench.py --workload $WL --no-cpu-baseline --no-cache-l0 --no-e2e --steps 10 2>/dev/null \
      | python -c "import sys,json; d=json.loads([l for l in sys.stdin if l.startswith('{')][-1]); print('$L', '$WL', round(d['value'],3), round(d['breakdown_ms_per_epoch']['gemm'],3))"
  done
done
