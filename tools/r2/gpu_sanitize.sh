# compute-sanitizer over tools/sanitize_run.py (tile kernels included)
mkdir -p gpurun_out
for tool in memcheck racecheck synccheck; do
  timeout 1500 compute-sanitizer --tool $tool --error-exitcode 99 --print-limit 20 python tools/sanitize_run.py > gpurun_out/sanitize_$tool.log 2>&1
  echo ${tool}_rc=$?; tail -2 gpurun_out/sanitize_$tool.log
done
