TAG=${1:-r01c}
ARGS="--steps 1 --warmup 1 --no-e2e --no-cpu-baseline"
timeout -s KILL 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 300 --csv \
   --log-file gpurun_out/launches_${TAG}.csv python bench.py $ARGS > gpurun_out/ncu_launch_${TAG}.log 2>&1
echo "launch rc=$?"
timeout -s KILL 1200 ncu --set full --clock-control none --import-source on -k regex:gemm_wgrad -s 3 -c 1 \
   -o gpurun_out/prof_wgrad_${TAG} -f python bench.py $ARGS > gpurun_out/ncu_wgrad_${TAG}.log 2>&1
echo "wgrad rc=$?"
timeout -s KILL 1200 ncu --set full --clock-control none --import-source on -k regex:gemm_rows -s 5 -c 1 \
   -o gpurun_out/prof_rows_${TAG} -f python bench.py $ARGS > gpurun_out/ncu_rows_${TAG}.log 2>&1
echo "rows rc=$?"
