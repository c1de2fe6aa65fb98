# compute-sanitizer memcheck / racecheck / synccheck over tools/sanitize_driver.py (args: tag)
T=${1:-r02}
for tool in memcheck racecheck synccheck; do
  timeout 1500 compute-sanitizer --tool $tool --error-exitcode 9 python tools/sanitize_driver.py > gpurun_out/sanitizer_${tool}_$T.log 2>&1
  echo "rc=$?" >> gpurun_out/sanitizer_${tool}_$T.log
done
