TAG=${1:-r01b}
ARGS="--steps 1 --warmup 1 --no-e2e --no-cpu-baseline"
timeout -s KILL 1200 ncu --set full --clock-control none --import-source on -k regex:spmm_stage -s 6 -c 1 \
   -o gpurun_out/prof_spmm_${TAG} -f python bench.py $ARGS > gpurun_out/ncu_spmm_${TAG}.log 2>&1
echo "spmm full rc=$?"
