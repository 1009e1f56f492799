# Dev: correctness + A/B timing of build variants (VP_LIB_NAME; "base" = ab_base/, a build of
# the last commit) on the config-5 hybrid.
mkdir -p gpurun_out
for lib in ${VP_AB_TEST_LIBS:-libvp.so}; do
  VP_LIB_NAME=$lib timeout 900 python -m pytest ${VP_AB_TESTS:-tests} -m gpu -x -q > gpurun_out/pytest_$lib.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_$lib.log
done
for rep in 1 2; do
for lib in ${VP_AB_LIBS:-libvp.so}; do
  echo "== $lib" >> gpurun_out/ab.txt
  if [ "$lib" = base ]; then
    (cd ab_base && timeout 300 python tools/reyes_sweep.py --no-timers --reps 5 --configs ${VP_AB_CFGS:-h36,h40,h44}) >> gpurun_out/ab.txt 2>&1
  else
    VP_LIB_NAME=$lib timeout 300 python tools/reyes_sweep.py --no-timers --reps 5 --configs ${VP_AB_CFGS:-h36,h40,h44} >> gpurun_out/ab.txt 2>&1
  fi
done
done
# optional: a full ncu capture of the fused [Dice,Shade] kernel of the default build
if [ -n "$VP_AB_NCU_TAG" ]; then
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:vp_kernel -c 1 -o gpurun_out/rtc_leaf$VP_AB_NCU_TAG python tools/ncu_targets.py rtc_leaf --frames 64 --runs 1 > gpurun_out/ncu_full$VP_AB_NCU_TAG.log 2>&1
  ncu -i gpurun_out/rtc_leaf$VP_AB_NCU_TAG.ncu-rep --page source --csv --print-source cuda,sass > gpurun_out/rtc_leaf_src$VP_AB_NCU_TAG.csv 2>&1
  python tools/ncu_summary.py gpurun_out/rtc_leaf$VP_AB_NCU_TAG.ncu-rep 40 > gpurun_out/rtc_leaf_sum$VP_AB_NCU_TAG.txt 2>&1
fi
