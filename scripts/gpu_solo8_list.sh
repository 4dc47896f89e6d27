timeout -s KILL 900 ncu --metrics gpu__time_duration.sum,launch__grid_size --clock-control none -c 400 --csv \
   --log-file gpurun_out/solo8_launches.csv python scripts/papers_rank.py --workload reddit --parts 8 --steps 1 --warmup 1 > gpurun_out/solo8_ncu.log 2>&1
echo "ncu rc=$?"
