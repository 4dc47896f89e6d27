# row GEMM: single-CTA vs CTA-pair (cta_group::2) on the bench workloads + per-kernel launch list
for P in 0 1; do
  for WL in reddit products; do
    MGGCN_ROW_PAIR=$P timeout -s KILL 300 python bench.py --workload $WL --no-cpu-baseline --no-cache-l0 --no-e2e --steps 10 2>/dev/null \
      | python -c "import sys,json; d=json.loads([l for l in sys.stdin if l.startswith('{')][-1]); print('pair=$P', '$WL', round(d['value'],3), round(d['breakdown_ms_per_epoch']['spmm'],3), round(d['breakdown_ms_per_epoch']['gemm'],3))"
  done
  MGGCN_ROW_PAIR=$P timeout -s KILL 300 ncu --metrics gpu__time_duration.sum,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed --clock-control none -k regex:gemm_rows -c 10 --csv \
     python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --no-cache-l0 2>/dev/null > gpurun_out/pair_$P.csv
done
