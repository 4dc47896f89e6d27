set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout -s KILL 300 python -m pytest tests/test_gpu_kernels.py -x -q --timeout 120 -k "gemm_integer_exact" > gpurun_out/t_gemm.log 2>&1; echo "gemm rc=$?"
tail -30 gpurun_out/t_gemm.log
timeout -s KILL 300 python -m pytest tests/test_gpu_kernels.py -q --timeout 120 -k "spmm" > gpurun_out/t_spmm.log 2>&1; echo "spmm rc=$?"
tail -30 gpurun_out/t_spmm.log
