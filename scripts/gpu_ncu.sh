# ncu evidence for the bench workload (1 GPU).  $1 = tag
TAG=${1:-r01}
shift
ARGS="--steps 1 --warmup 1 --no-e2e --no-cpu-baseline $@"
timeout -s KILL 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 300 --csv \
   --log-file gpurun_out/launches_${TAG}.csv python bench.py $ARGS > gpurun_out/ncu_launch_${TAG}.log 2>&1
echo "launch list rc=$?"
timeout -s KILL 1200 ncu --set full --clock-control none --import-source on -k regex:spmm_stage -s 6 -c 1 \
   -o gpurun_out/prof_spmm_${TAG} -f python bench.py $ARGS > gpurun_out/ncu_spmm_${TAG}.log 2>&1
echo "spmm full rc=$?"
timeout -s KILL 1200 ncu --set full --clock-control none --import-source on -k regex:gemm_tf32 -s 8 -c 1 \
   -o gpurun_out/prof_gemm_${TAG} -f python bench.py $ARGS > gpurun_out/ncu_gemm_${TAG}.log 2>&1
echo "gemm full rc=$?"
ls -la gpurun_out/
