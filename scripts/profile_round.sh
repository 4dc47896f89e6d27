# Round profile evidence: launch list of one epoch + ncu --set full of the top kernels.
# usage: bash scripts/profile_round.sh <tag> [workload]
TAG=$1; WL=${2:-reddit}
sha256sum paper_conf_icpp_balinsc22_b200/libmggcn.so > gpurun_out/${TAG}_so.sha
ARGS="--workload $WL --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --no-cache-l0"
timeout -s KILL 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
   --log-file gpurun_out/${TAG}_launches.csv python bench.py $ARGS > gpurun_out/${TAG}_launch.log 2>&1
echo "launch list rc=$?"
for spec in "dense_tile:dense_tile:${DENSE_SKIP:-4}" "spmm_wide:spmm_stage:${WIDE_SKIP:-10}" "spmm_narrow:spmm_stage:${NARROW_SKIP:-14}" "gemm_rows:gemm_rows:5" "gemm_wgrad:gemm_wgrad:5"; do
  NAME=${spec%%:*}; REST=${spec#*:}; K=${REST%%:*}; S=${REST#*:}
  timeout -s KILL 900 ncu --set full --clock-control none --import-source on -k regex:$K -s $S -c 1 \
     -o gpurun_out/${TAG}_${NAME} -f python bench.py $ARGS > gpurun_out/${TAG}_${NAME}.log 2>&1
  echo "$NAME rc=$?"
done
