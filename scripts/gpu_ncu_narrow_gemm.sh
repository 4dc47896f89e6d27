# ncu --set full of the narrow-N GEMMs of the Reddit epoch (H2·W2 row GEMM, W_G2 wgrad) and the CE kernel
ARGS="--workload reddit --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --no-cache-l0"
for spec in "rows_n41:gemm_rows:7" "wgrad_n41:gemm_wgrad:3" "ce:softmax_ce:1"; do
  NAME=${spec%%:*}; REST=${spec#*:}; K=${REST%%:*}; S=${REST#*:}
  timeout -s KILL 600 ncu --set full --clock-control none --import-source on -k regex:$K -s $S -c 1 \
     -o gpurun_out/n_${NAME} -f python bench.py $ARGS > gpurun_out/n_${NAME}.log 2>&1
  echo "$NAME rc=$?"
done
