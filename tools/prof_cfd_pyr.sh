python -c "import __graft_entry__ as g; g.build()" >/dev/null 2>&1
for m in kbk mega; do timeout 120 python tools/ncu_wl.py cfd $m --outer 2 --runs 3 --timers; timeout 300 python tools/ncu_wl.py pyr $m --runs 3 --timers; done
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/cfd_kbk_launches.csv python tools/ncu_wl.py cfd kbk --outer 1 > /dev/null 2>&1
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/pyr_kbk_launches.csv python tools/ncu_wl.py pyr kbk --imgs 8 > /dev/null 2>&1
timeout 400 ncu --set full --clock-control none --import-source on -k regex:vp_kernel --launch-skip 4 -c 4 -o gpurun_out/cfd_kbk python tools/ncu_wl.py cfd kbk --outer 1 > gpurun_out/ncu_cfd.log 2>&1
