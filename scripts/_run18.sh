timeout -s KILL 900 python -m pytest tests/test_gpu_dense.py -x -q --timeout 300 > gpurun_out/d18_tests.log 2>&1; echo "tests rc=$?"; tail -2 gpurun_out/d18_tests.log
timeout -s KILL 600 python scripts/dense_probe.py --workload reddit --width 256 48 --thr 0.03 --reps 10 2>/dev/null > gpurun_out/d18.jsonl
timeout -s KILL 600 python scripts/dense_probe.py --workload proteins --width 128 112 8 --thr 0.03 --reps 10 2>/dev/null >> gpurun_out/d18.jsonl
