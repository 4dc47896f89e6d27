# Adaptive hub-segment length: SOLO per-rank compute at P = 8 (Reddit, Products, Proteins) for
# forced segment lengths vs the adaptive default; P = 1 Reddit bench; kernel + epoch tests.
timeout -s KILL 900 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_epoch.py -q -x > gpurun_out/t_split.log 2>&1; echo "tests rc=$?"; tail -2 gpurun_out/t_split.log
OUT=gpurun_out/split_sweep.log; : > $OUT
for WL in reddit products proteins; do
  for S in 0 2048 512 256 128; do
    R=$(MGGCN_SPMM_SPLIT=$S timeout -s KILL 600 python scripts/papers_rank.py --workload $WL --parts 8 --rank 0 --steps 10 --warmup 3 2>&1 | grep '^{' | python -c "
import sys,json; d=json.loads(sys.stdin.read()); b=d['breakdown_ms_per_epoch']; print(round(d['compute_ms_per_epoch'],3), 'spmm', round(b['spmm'],3))")
    echo "$WL P=8 split=$S compute $R" >> $OUT
  done
done
timeout -s KILL 600 python bench.py --steps 20 --warmup 5 --no-cpu-baseline > gpurun_out/b_split.log 2>&1
tail -1 gpurun_out/b_split.log | python -c "
import sys,json; d=json.loads(sys.stdin.read()); b=d['breakdown_ms_per_epoch']; print('reddit P=1 bench', round(d['value'],3), 'eager', round(d['eager_ms'],3), 'spmm', round(b['spmm'],3))" >> $OUT
cat $OUT
