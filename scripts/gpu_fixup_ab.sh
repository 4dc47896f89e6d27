# Same-box A/B of the fix-up threshold (MGGCN_FIXUP_MANY): 0 = every split row gets a block,
# 1000000 = every split row a warp, default 32; P = 1 bench and SOLO P = 8 Reddit.
for M in 0 1000000 32 8 0 1000000; do
  MGGCN_FIXUP_MANY=$M timeout -s KILL 600 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-cache-l0 --no-e2e > gpurun_out/b_ab.log 2>&1
  A=$(tail -1 gpurun_out/b_ab.log | python -c "
import sys,json; d=json.loads(sys.stdin.read()); b=d['breakdown_ms_per_epoch']; print(round(d['value'],3), 'eager', round(d['eager_ms'],3), 'spmm', round(b['spmm'],3))")
  B=$(MGGCN_FIXUP_MANY=$M timeout -s KILL 600 python scripts/papers_rank.py --workload reddit --parts 8 --rank 0 --steps 10 --warmup 3 2>&1 | grep '^{' | python -c "
import sys,json; d=json.loads(sys.stdin.read()); b=d['breakdown_ms_per_epoch']; print(round(d['compute_ms_per_epoch'],3), 'spmm', round(b['spmm'],3))")
  echo "many=$M  P1: $A  | P8 solo: $B"
done
