# Products-shaped evidence: forced-class parity test, launch list of one epoch, and one
# ncu --set full capture of a width-256 SpMM launch (2nd epoch's 2nd SpMM).
timeout -s KILL 900 python -m pytest tests/test_gpu_kernels.py -q -x -k hot_classes > gpurun_out/t_hot.log 2>&1; echo "hot tests rc=$?"; tail -2 gpurun_out/t_hot.log
ARGS="--workload products --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --no-cache-l0 --eager"
timeout -s KILL 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
   --log-file gpurun_out/r01p_launches.csv python bench.py $ARGS > gpurun_out/r01p_launch.log 2>&1
echo "launch list rc=$?"
timeout -s KILL 900 ncu --set full --clock-control none --import-source on -k regex:spmm_stage -s 6 -c 1 \
   -o gpurun_out/r01p_spmm_wide -f python bench.py $ARGS > gpurun_out/r01p_spmm_wide.log 2>&1
echo "ncu rc=$?"
