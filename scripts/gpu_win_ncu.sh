# DRAM / L2 traffic of the width-256 Reddit SpMM per column window (MGGCN_SPMM_WIN).
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sectors_srcunit_tex_op_read.sum,lts__t_sector_hit_rate.pct,l1tex__t_sector_hit_rate.pct,lts__throughput.avg.pct_of_peak_sustained_elapsed,lts__t_requests_srcunit_tex_op_read.sum
for WIN in 512 128 64; do
  MGGCN_SPMM_WIN=$WIN timeout -s KILL 600 ncu --metrics $M --clock-control none -k regex:spmm_stage -c 6 --csv \
     python scripts/spmm_sweep.py reddit 256 > gpurun_out/win_ncu_$WIN.csv 2>&1
  echo "WIN=$WIN rc=$?"
done
