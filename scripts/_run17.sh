for v in apf0 default apf16; do
  if [ $v = default ]; then L=""; else L="MGGCN_LIB=$PWD/sweep_libs/libmggcn_$v.so"; fi
  env $L timeout -s KILL 600 python scripts/dense_probe.py --workload reddit --width 256 48 --thr 0.03 --reps 10 2>/dev/null | sed "s/^{/{\"v\": \"$v\", /" >> gpurun_out/d17.jsonl
done
