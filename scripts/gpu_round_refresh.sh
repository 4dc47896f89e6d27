# End-of-round evidence refresh (1 GPU): bench lines for the three single-GPU workloads,
# then the launch list + ncu --set full captures of scripts/profile_round.sh.
TAG=${1:-r01}
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
for WL in reddit products proteins cora; do
  timeout -s KILL 900 python bench.py --workload $WL > gpurun_out/${TAG}_bench_${WL}.log 2>&1; echo "bench $WL rc=$?"
  tail -1 gpurun_out/${TAG}_bench_${WL}.log | cut -c1-300
done
bash scripts/profile_round.sh $TAG reddit
ls -la gpurun_out
