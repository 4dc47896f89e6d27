ARGS="--steps 1 --warmup 1 --no-e2e --no-cpu-baseline --no-cache-l0"
timeout -s KILL 600 python -m pytest tests/test_gpu_kernels.py -q -x -k gemm 2>&1 | tail -1
timeout -s KILL 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:gemm -c 100 --csv \
     --log-file gpurun_out/gt.csv python bench.py $ARGS > /dev/null 2>&1
python -c "
import csv
rows=list(csv.reader(open('gpurun_out/gt.csv')))
h=[i for i,r in enumerate(rows) if 'Kernel Name' in r][0]
vi=rows[h].index('Metric Value'); ki=rows[h].index('Kernel Name')
print([(r[ki][11:20],r[vi]) for r in rows[h+1:]][-8:])"
