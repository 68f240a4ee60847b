set -x
timeout 900 python -m pytest tests/test_gpu_ssim_cert.py -q -s 2>&1 | grep -E "exact|worst|passed|failed|Error|assert" | head -40
timeout 300 python tools/quick_time.py C2 2>&1 | tail -5
timeout 300 python tools/quick_time.py C3 2>&1 | tail -5
timeout 900 ncu --set full --clock-control none --import-source on -k regex:p3_kernel -c 1 -f -o gpurun_out/prof_r02c python tools/ncu_target.py C2 1 > gpurun_out/ncu_r02c.log 2>&1
python tools/ncu_summary.py gpurun_out/r02c_ncu gpurun_out/prof_r02c.ncu-rep > /dev/null 2>&1; cat gpurun_out/r02c_ncu.md
ncu -i gpurun_out/prof_r02c.ncu-rep --page source --csv > gpurun_out/r02c_p3_source.csv 2>/dev/null
ncu -i gpurun_out/prof_r02c.ncu-rep --page raw --csv > gpurun_out/r02c_p3_raw.csv 2>/dev/null
rm -f gpurun_out/prof_r02c.ncu-rep
