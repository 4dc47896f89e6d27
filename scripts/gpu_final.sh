# Round-end evidence: new tests, per-rank SOLO compute for P = 2/4/8, bench lines, launch list + ncu.
timeout -s KILL 900 python -m pytest tests/test_gpu_epoch.py -q -x -k "delay or solo" > gpurun_out/t_delay.log 2>&1; echo "delay/solo tests rc=$?"; tail -2 gpurun_out/t_delay.log
: > gpurun_out/solo_scaling.jsonl
for WL in reddit products proteins; do
  for P in 2 4 8; do
    timeout -s KILL 600 python scripts/papers_rank.py --workload $WL --parts $P --rank 0 --steps 10 --warmup 3 2>&1 | grep '^{' >> gpurun_out/solo_scaling.jsonl
    echo "solo $WL P=$P rc=$?"
  done
done
bash scripts/gpu_round_refresh.sh r01
