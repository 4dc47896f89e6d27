# Solo-mode parity test, then the Papers-shaped rank-0-of-8 compute timing (scripts/papers_rank.py).
timeout -s KILL 600 python -m pytest tests/test_gpu_epoch.py -q -x -k solo > gpurun_out/t_solo.log 2>&1; echo "solo tests rc=$?"; tail -3 gpurun_out/t_solo.log
free -g; nproc
timeout -s KILL 2400 python scripts/papers_rank.py --rank 0 --parts 8 --steps 5 --warmup 2 > gpurun_out/papers_rank0.log 2>&1; echo "papers rc=$?"
tail -c 3000 gpurun_out/papers_rank0.log
