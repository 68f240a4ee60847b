set -x
timeout 1500 python -m pytest tests -m gpu -q -x 2>&1 | tail -5
timeout 300 python tools/quick_time.py C2 2>&1 | tail -5
timeout 300 python tools/quick_time.py C3 2>&1 | grep -E "DERIV|ALL"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:deriv3 -c 1 -f -o gpurun_out/prof_r02e python tools/ncu_target.py C2 1 > gpurun_out/ncu_r02e.log 2>&1
python tools/ncu_summary.py gpurun_out/r02e_ncu gpurun_out/prof_r02e.ncu-rep > /dev/null 2>&1; cat gpurun_out/r02e_ncu.md
rm -f gpurun_out/prof_r02e.ncu-rep
for tool in memcheck racecheck synccheck initcheck; do
  timeout 1500 compute-sanitizer --tool $tool --print-limit 50 python tools/sanitize_target.py > gpurun_out/sanitize_${tool}_r02.log 2>&1
  echo "$tool rc=$?"; tail -3 gpurun_out/sanitize_${tool}_r02.log
done
