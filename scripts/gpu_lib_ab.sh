# Same-box A/B of library builds (MGGCN_LIB): A = 2048-entry segments + warp fix-up, B = adaptive
# segments + one fix-up launch per stage, C = adaptive segments + fix-up fused into the SpMM.
P=paper_conf_icpp_balinsc22_b200
for L in A B C A B C; do
  if [ $L = C ]; then LIB=$P/libmggcn.so; else LIB=$P/libmggcn_ab_$L.so; fi
  X=$(MGGCN_LIB=$LIB timeout -s KILL 600 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-cache-l0 --no-e2e 2>&1 | tail -1 | python -c "
import sys,json; d=json.loads(sys.stdin.read()); b=d['breakdown_ms_per_epoch']; print(round(d['value'],3), 'eager', round(d['eager_ms'],3), 'spmm', round(b['spmm'],3))")
  Y=$(MGGCN_LIB=$LIB timeout -s KILL 600 python scripts/papers_rank.py --workload reddit --parts 8 --rank 0 --steps 10 --warmup 3 2>&1 | grep '^{' | python -c "
import sys,json; d=json.loads(sys.stdin.read()); b=d['breakdown_ms_per_epoch']; print(round(d['compute_ms_per_epoch'],3), 'spmm', round(b['spmm'],3))")
  echo "$L  P=1: $X  | SOLO P=8: $Y"
done
