# ncu --set full of one kernel launch of the bench: $1 tag, $2 kernel regex, $3 skip count
TAG=$1; K=$2; S=$3
ARGS="--steps 1 --warmup 1 --no-e2e --no-cpu-baseline"
timeout -s KILL 1200 ncu --set full --clock-control none --import-source on -k regex:$K -s $S -c 1 \
   -o gpurun_out/prof_${TAG} -f python bench.py $ARGS > gpurun_out/ncu_${TAG}.log 2>&1
echo "$TAG rc=$?"
