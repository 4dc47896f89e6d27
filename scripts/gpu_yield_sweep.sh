# Cost of the SPMM_YIELD grid oversubscription on one GPU (forced with MGGCN_SPMM_YIELD=k):
# epoch and SpMM ms per epoch, Reddit- and Products-shaped, P = 1.
OUT=gpurun_out/yield_sweep.log
: > $OUT
for WL in reddit products; do
for Y in 0 2 4 8 16; do
  MGGCN_SPMM_YIELD=$Y timeout -s KILL 600 python bench.py --workload $WL --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --eager > gpurun_out/ys.log 2>&1
  echo "== $WL yield=$Y rc=$?" >> $OUT
  tail -1 gpurun_out/ys.log | python -c "
import sys,json
try:
  d=json.loads(sys.stdin.read()); b=d.get('breakdown_ms_per_epoch',{})
  print('epoch', round(d['value'],3), 'spmm', round(b.get('spmm'),3), 'gemm', round(b.get('gemm'),3))
except Exception as e: print('parse fail', e)" >> $OUT
done
done
cat $OUT
