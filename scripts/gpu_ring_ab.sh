# A/B of the row-GEMM operand ring (MGGCN_ROW_RING=0: ring after the old-C chunks; default: unmasked
# products take those 32 KB too). GEMM parity tests first, then interleaved bench lines.
timeout -s KILL 600 python -m pytest tests -m gpu -q -x -k "gemm or epoch" --timeout 300 > gpurun_out/ring_tests.log 2>&1; echo "tests rc=$?"; tail -2 gpurun_out/ring_tests.log
: > gpurun_out/ring_ab.log
for WL in products reddit; do
  for R in 0 1 0 1; do
    MGGCN_ROW_RING=$R timeout -s KILL 600 python bench.py --workload $WL --steps 20 --warmup 5 --no-e2e --no-cpu-baseline --no-cache-l0 2>/dev/null | tail -1 | \
      python -c "import sys,json; d=json.loads(sys.stdin.read()); print('$WL ring=$R', round(d['value'],3), 'gemm', round(d['breakdown_ms_per_epoch']['gemm'],3), 'spmm', round(d['breakdown_ms_per_epoch']['spmm'],3), 'clk', d['clocks']['sm_mhz'], d['clocks']['reasons'])" >> gpurun_out/ring_ab.log 2>&1
  done
done
cat gpurun_out/ring_ab.log
