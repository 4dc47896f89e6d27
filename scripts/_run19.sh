for WL in reddit proteins; do for P in 4 8; do
 for cfg in "MGGCN_DENSE_MIN_ROWS=32768" "MGGCN_DENSE_MIN_ROWS=0 MGGCN_DENSE_MIN_ENTRIES=3000000" "MGGCN_DENSE_MIN_ROWS=0 MGGCN_DENSE_MIN_ENTRIES=5000000"; do
  env $cfg timeout -s KILL 900 python scripts/papers_rank.py --workload $WL --parts $P --rank 0 --steps 10 --warmup 3 2>/dev/null | grep '^{' | python -c "
import json,sys
for l in sys.stdin:
  d=json.loads(l); print(json.dumps({'wl':'$WL','P':$P,'cfg':'$cfg','ms':d['compute_ms_per_epoch'],'spmm':d['breakdown_ms_per_epoch']['spmm'],'dense':d['dense'],'groups':d['stage_groups']}))" >> gpurun_out/d19_solo_ab.jsonl
 done; done; done
