timeout -s KILL 2400 python scripts/papers_rank.py --rank 0 --parts 8 --steps 5 --warmup 2 > gpurun_out/papers_rank0.log 2>&1; echo "papers rc=$?"
tail -c 2500 gpurun_out/papers_rank0.log
