CZC_LIB=$PWD/abtest/tma.so timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_ssim_cert.py -q -x --deselect tests/test_gpu_parity.py::test_full_size_2048_cubed_smooth_pair 2>&1 | tail -2
python tools/ab_time.py C2 abtest/base.so abtest/tma.so
python tools/ab_time.py C3 abtest/base.so abtest/tma.so
timeout 600 ncu --set full --clock-control none -k regex:p1_tma -c 1 -f -o gpurun_out/prof_p1tma python tools/ncu_target.py C3 1 > /dev/null 2>&1; python tools/ncu_summary.py gpurun_out/p1tma_ncu gpurun_out/prof_p1tma.ncu-rep > /dev/null 2>&1; cat gpurun_out/p1tma_ncu.md; rm -f gpurun_out/prof_p1tma.ncu-rep
