# full GPU test suite with per-test timeouts; logs under gpurun_out/
timeout -s KILL 1200 python -m pytest tests -m gpu -q --timeout 300 -x "$@" > gpurun_out/t_gpu.log 2>&1; echo "gpu tests rc=$?"
tail -40 gpurun_out/t_gpu.log
