timeout -s KILL 1500 python -m pytest tests/test_gpu_dense.py tests/test_gpu_epoch.py tests/test_gpu_graph.py -x -q --timeout 300 > gpurun_out/d24_tests.log 2>&1; echo "tests rc=$?"; tail -2 gpurun_out/d24_tests.log
bash scripts/gpu_round.sh d24 bench reddit --steps 20 --warmup 5
bash scripts/gpu_round.sh d24 bench proteins --steps 20 --warmup 5
