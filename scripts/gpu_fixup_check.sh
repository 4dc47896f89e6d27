timeout -s KILL 600 python -m pytest tests/test_gpu_kernels.py -q -x -k "rmat_hubs or power_law" > gpurun_out/t_fix.log 2>&1; echo "tests rc=$?"; tail -1 gpurun_out/t_fix.log
timeout -s KILL 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:fixup -c 40 --csv \
   --log-file gpurun_out/fix_launches.csv python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --no-cache-l0 --eager > /dev/null 2>&1
python -c "
import csv
rows=list(csv.reader(open('gpurun_out/fix_launches.csv')))
h=[i for i,r in enumerate(rows) if 'Kernel Name' in r][0]
vi=rows[h].index('Metric Value'); ki=rows[h].index('Kernel Name')
v=[(r[ki][:40],float(r[vi])) for r in rows[h+1:]]
print('fixup launches', len(v), 'total us (last 10)', sum(x[1] for x in v[-10:])/1e3, v[-1][0])"
for i in 1 2; do
timeout -s KILL 600 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-cache-l0 > gpurun_out/b_fix.log 2>&1
tail -1 gpurun_out/b_fix.log | python -c "
import sys,json; d=json.loads(sys.stdin.read()); b=d['breakdown_ms_per_epoch']; print('reddit P=1 bench', round(d['value'],3), 'eager', round(d['eager_ms'],3), 'spmm', round(b['spmm'],3), d['clocks'])"
done
timeout -s KILL 600 python scripts/papers_rank.py --workload reddit --parts 8 --rank 0 --steps 10 --warmup 3 2>&1 | grep '^{' | cut -c1-330
