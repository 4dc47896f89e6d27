
MGGCN_LIB=$PWD/sweep_libs/libmggcn_l1pf.so timeout -s KILL 600 python scripts/dense_probe.py --workload reddit --width 256 48 --thr 0,0.03 --reps 5 2>/dev/null | sed 's/^{/{"v": "l1pf", /' >> gpurun_out/d15.jsonl
