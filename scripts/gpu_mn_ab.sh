# Same-box A/B of the weight-gradient ring budget: A = libmggcn.so (192 KB, <= 10 raw stages),
# B = libmggcn_mn224.so (224 KB, <= 16 raw stages). GEMM tests on B first.
P=paper_conf_icpp_balinsc22_b200
MGGCN_LIB=$P/libmggcn_mn224.so timeout -s KILL 600 python -m pytest tests -m gpu -q -x -k "gemm" --timeout 300 > gpurun_out/mn_tests.log 2>&1; echo "tests rc=$?"; tail -1 gpurun_out/mn_tests.log
: > gpurun_out/mn_ab.log
for WL in products reddit; do
  for L in A B A B; do
    if [ $L = A ]; then LIB=$P/libmggcn.so; else LIB=$P/libmggcn_mn224.so; fi
    MGGCN_LIB=$LIB timeout -s KILL 600 python bench.py --workload $WL --steps 20 --warmup 5 --no-e2e --no-cpu-baseline --no-cache-l0 2>/dev/null | tail -1 | \
      python -c "import sys,json; d=json.loads(sys.stdin.read()); print('$WL $L', round(d['value'],3), 'gemm', round(d['breakdown_ms_per_epoch']['gemm'],3), 'spmm', round(d['breakdown_ms_per_epoch']['spmm'],3), 'clk', d['clocks']['sm_mhz'], d['clocks']['reasons'])" >> gpurun_out/mn_ab.log 2>&1
  done
done
cat gpurun_out/mn_ab.log
