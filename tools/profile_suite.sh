#!/bin/bash
# ncu launch lists (per-kernel time, DRAM bytes, L2 atomic / reduction sectors, issue and
# warp occupancy) of every configs-1..4 workload, the LDPC decoder and the queue
# microbenchmark, under KBK (one kernel per stage per wave) and the megakernel; then
# summarised by tools/ncu_launch_summary.py.  Numbers printed under ncu are not bench values.
mkdir -p gpurun_out/suite
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sectors_op_atom.sum,lts__t_sectors_op_red.sum,smsp__issue_active.avg.pct_of_peak_sustained_active,sm__warps_active.avg.pct_of_peak_sustained_active,launch__registers_per_thread
for wl in reyes1x face8 pyr cfd raster raster_near ldpc qb4 qb16 qb272; do
  for m in kbk mega; do
    extra=""
    [ "$wl" = "pyr" ] && extra="--imgs 32"
    timeout 600 ncu --metrics $M --clock-control none -c 600 --csv --log-file gpurun_out/suite/${wl}_${m}.csv \
      python tools/ncu_wl.py $wl $m $extra > gpurun_out/suite/${wl}_${m}.log 2>&1
  done
done
python tools/ncu_launch_summary.py gpurun_out/suite > gpurun_out/suite_ncu.txt 2>&1
