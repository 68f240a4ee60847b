python tools/ab_time.py C3 abtest/base.so abtest/pair.so abtest/u2.so
python tools/ab_time.py C2 abtest/base.so abtest/pair.so abtest/u2.so
CZC_LIB=$PWD/abtest/pair.so timeout 900 python -m pytest tests/test_gpu_ssim_cert.py -q -x 2>&1 | tail -2
