# Launch list of one SOLO epoch of Reddit-shaped rank 0 at P = 8 (per-stage kernel times), and
# the same with the yield grid off (MGGCN_SPMM_YIELD=1) for comparison.
timeout -s KILL 900 ncu --metrics gpu__time_duration.sum,launch__grid_size --clock-control none -c 400 --csv \
   --log-file gpurun_out/solo8_launches.csv python scripts/papers_rank.py --workload reddit --parts 8 --steps 1 --warmup 1 > gpurun_out/solo8_ncu.log 2>&1
echo "ncu rc=$?"
for Y in 0 1; do
  MGGCN_SPMM_YIELD=$Y timeout -s KILL 600 python scripts/papers_rank.py --workload reddit --parts 8 --steps 10 --warmup 3 2>&1 | grep '^{' | cut -c1-400
done
