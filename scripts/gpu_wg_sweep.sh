ARGS="--steps 1 --warmup 1 --no-e2e --no-cpu-baseline --no-cache-l0"
for lib in "" sweep_libs/mn4.so sweep_libs/mn12.so sweep_libs/mn16.so; do
  MGGCN_LIB=$lib timeout -s KILL 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:gemm_wgrad -c 100 --csv \
     --log-file gpurun_out/wgs.csv python bench.py $ARGS > /dev/null 2>&1
  echo "lib=${lib:-default(8)}: $(python -c "
import csv
rows=list(csv.reader(open('gpurun_out/wgs.csv')))
h=[i for i,r in enumerate(rows) if 'Kernel Name' in r][0]
vi=rows[h].index('Metric Value')
print([r[vi] for r in rows[h+1:]][-3:])")"
done
