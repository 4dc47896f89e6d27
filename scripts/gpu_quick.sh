timeout -s KILL 600 python -m pytest tests/test_gpu_kernels.py -q --timeout 120 -x -k gemm 2>&1 | tail -2
timeout -s KILL 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 300 --csv \
   --log-file gpurun_out/launches_q.csv python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > /dev/null 2>&1
echo "launch rc=$?"
