# SpMM launch-shape variants (launch bounds / warps per block) on the bench workloads
for L in sweep_libs/lib_*.so; do
  for WL in reddit products; do
    MGGCN_LIB=$L timeout -s KILL 300 python bench.py --workload $WL --no-cpu-baseline --no-cache-l0 --no-e2e --steps 10 2>/dev/null \
      | python -c "import sys,json; d=json.loads([l for l in sys.stdin if l.startswith('{')][-1]); print('$L', '$WL', round(d['value'],3), round(d['breakdown_ms_per_epoch']['spmm'],3), round(d['breakdown_ms_per_epoch']['gemm'],3))"
  done
done
