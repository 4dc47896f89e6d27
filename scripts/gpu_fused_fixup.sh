# Fused hub-row fix-up: kernel/epoch/graph/full-size tests, P = 1 bench (x2), SOLO P = 8 Reddit/Products/Proteins.
timeout -s KILL 1200 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_epoch.py tests/test_gpu_graph.py tests/test_gpu_fullsize.py tests/test_gpu_15d.py -q -x > gpurun_out/t_ff.log 2>&1; echo "tests rc=$?"; tail -2 gpurun_out/t_ff.log
for i in 1 2; do
timeout -s KILL 600 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-cache-l0 --no-e2e > gpurun_out/b_ff.log 2>&1
tail -1 gpurun_out/b_ff.log | python -c "
import sys,json; d=json.loads(sys.stdin.read()); b=d['breakdown_ms_per_epoch']; print('reddit P=1 bench', round(d['value'],3), 'eager', round(d['eager_ms'],3), 'spmm', round(b['spmm'],3), 'launches', d['gpu_launches'])"
done
for WL in reddit products proteins; do
timeout -s KILL 600 python scripts/papers_rank.py --workload $WL --parts 8 --rank 0 --steps 10 --warmup 3 2>&1 | grep '^{' | python -c "
import sys,json; d=json.loads(sys.stdin.read()); b=d['breakdown_ms_per_epoch']; print('$WL P=8 solo', round(d['compute_ms_per_epoch'],3), 'spmm', round(b['spmm'],3))"
done
