python tools/ab_time.py C2 abtest/base.so abtest/f4.so
python tools/ab_time.py C3 abtest/base.so abtest/f4.so
CZC_LIB=$PWD/abtest/f4.so timeout 900 python -m pytest tests/test_gpu_ssim_cert.py tests/test_gpu_deriv_points.py -q -x 2>&1 | tail -2
