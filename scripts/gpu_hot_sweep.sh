# L2 priority-class sweep on the Products-shaped workload (1 GPU): budget of
# evict_last rows (MGGCN_SPMM_HOT_MB) x persisting set-aside (MGGCN_L2_PERSIST_MB).
OUT=gpurun_out/hot_sweep.log
: > $OUT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv >> $OUT
for cfg in "HOTCLS=0" "HOT=0" "HOT=32" "HOT=64" "HOT=96" "HOT=32 PERS=200" "HOT=64 PERS=200" "HOT=96 PERS=200"; do
  unset MGGCN_SPMM_HOT_MB MGGCN_L2_PERSIST_MB MGGCN_SPMM_HOTCLS
  for kv in $cfg; do
    case $kv in
      HOTCLS=*) export MGGCN_SPMM_HOTCLS=${kv#HOTCLS=};;
      HOT=*) export MGGCN_SPMM_HOT_MB=${kv#HOT=};;
      PERS=*) export MGGCN_L2_PERSIST_MB=${kv#PERS=};;
    esac
  done
  timeout -s KILL 600 python bench.py --workload ${WL:-products} --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/hs.log 2>&1
  echo "== $cfg rc=$?" >> $OUT
  grep "persisting" gpurun_out/hs.log >> $OUT
  tail -1 gpurun_out/hs.log | python -c "
import sys,json
try:
  d=json.loads(sys.stdin.read()); b=d.get('breakdown_ms_per_epoch',{})
  print('epoch', d['value'], 'eager', d.get('eager_ms'), 'spmm', b.get('spmm'), 'gemm', b.get('gemm'), 'l2frac', d['roofline'].get('l2_gather',{}).get('frac'))
except Exception as e: print('parse fail', e)" >> $OUT
done
cat $OUT
