set -x
mkdir -p gpurun_out
for tool in memcheck racecheck synccheck initcheck; do
  timeout 1500 compute-sanitizer --tool $tool --print-limit 50 python tools/sanitize_target.py > gpurun_out/sanitize_${tool}_r02.log 2>&1
  echo "$tool rc=$?"; tail -4 gpurun_out/sanitize_${tool}_r02.log
done
