mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 600 python tools/reyes_sweep.py --reps 3 --no-timers --configs h60b16_16_64_4,mega > gpurun_out/l2_off.log 2>&1
timeout 600 python tools/reyes_sweep.py --reps 3 --no-timers --l2 --configs h60b16_16_64_4,mega > gpurun_out/l2_on.log 2>&1
M=gpu__time_duration.sum,lts__t_sector_hit_rate.pct,lts__t_sectors_op_atom.sum,lts__t_sectors_op_red.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sectors_srcunit_tex_lookup_hit.sum,lts__t_sectors_srcunit_tex_lookup_miss.sum
timeout 600 ncu --metrics $M --clock-control none -k regex:vp_kernel -c 1 --csv python tools/ncu_targets.py mega --frames 64 --runs 1 > gpurun_out/l2_ncu_off.csv 2>&1
timeout 600 ncu --metrics $M --clock-control none -k regex:vp_kernel -c 1 --csv python tools/ncu_targets.py mega --frames 64 --runs 1 --l2 > gpurun_out/l2_ncu_on.csv 2>&1
