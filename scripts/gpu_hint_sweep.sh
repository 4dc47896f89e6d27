# SpMM L2 cache-policy variants (MGGCN_SPMM_HINT: 1 = index stream evict_first, 2 = + gathers evict_last),
# with the column windows on: epoch/SpMM ms and the DRAM bytes of one wide Reddit SpMM launch.
for L in sweep_libs/lib_base.so sweep_libs/lib_hint1.so sweep_libs/lib_hint2.so; do
  for WL in reddit products; do
    MGGCN_LIB=$L timeout -s KILL 300 python bench.py --workload $WL --no-cpu-baseline --no-cache-l0 --no-e2e --steps 10 2>/dev/null \
      | python -c "import sys,json; d=json.loads([l for l in sys.stdin if l.startswith('{')][-1]); print('$L', '$WL', round(d['value'],3), round(d['breakdown_ms_per_epoch']['spmm'],3), round(d['breakdown_ms_per_epoch']['gemm'],3))"
  done
  MGGCN_LIB=$L timeout -s KILL 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct \
     -k regex:spmm_stage -s 10 -c 2 --csv python bench.py --workload reddit --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --no-cache-l0 2>/dev/null \
     | grep -E "gpu__time|dram__|lts__" | awk -F'","' -v L=$L '{print L, $(NF-2), $NF}'
done
