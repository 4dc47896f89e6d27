# Round-end: full GPU suite, SOLO per-rank compute at P = 2/4/8, bench lines, launch list + ncu.
bash scripts/gpu_tests.sh
: > gpurun_out/solo_scaling.jsonl
for WL in reddit products proteins; do
  for P in 2 4 8; do
    timeout -s KILL 600 python scripts/papers_rank.py --workload $WL --parts $P --rank 0 --steps 10 --warmup 3 2>&1 | grep '^{' >> gpurun_out/solo_scaling.jsonl
  done
done
bash scripts/gpu_round_refresh.sh r01
