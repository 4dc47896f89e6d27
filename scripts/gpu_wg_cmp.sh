ARGS="--steps 1 --warmup 1 --no-e2e --no-cpu-baseline --no-cache-l0"
for v in x mn; do
  MGGCN_WGRAD=$v timeout -s KILL 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:gemm -c 100 --csv \
     --log-file gpurun_out/wg_${v}.csv python bench.py $ARGS > /dev/null 2>&1
  echo "$v rc=$?"
  grep -o '"gemm_[a-z_]*kernel[^"]*","[^"]*","[^"]*","gpu__time_duration.sum","[^"]*","[0-9.]*"' gpurun_out/wg_${v}.csv | awk -F'","' '{print $1, $NF}' | tail -8
done
MGGCN_WGRAD=mn timeout -s KILL 900 ncu --set full --clock-control none --import-source on -k regex:gemm_wgrad -s 5 -c 1 \
   -o gpurun_out/prof_wgmn -f python bench.py $ARGS > gpurun_out/ncu_wgmn.log 2>&1
echo "full rc=$?"
