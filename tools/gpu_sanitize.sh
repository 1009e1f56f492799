# Dev: compute-sanitizer memcheck / racecheck / synccheck over tools/sanitize_run.py
mkdir -p gpurun_out
for t in memcheck racecheck synccheck; do
  timeout 1500 compute-sanitizer --tool $t python tools/sanitize_run.py > gpurun_out/r2_sanitize_$t.log 2>&1; echo "rc=$?" >> gpurun_out/r2_sanitize_$t.log
done
