python tools/ab_time.py C3 abtest/base.so abtest/w12.so abtest/w16.so
python tools/ab_time.py C2 abtest/base.so abtest/w12.so abtest/w16.so
for w in 12 16; do CZC_LIB=$PWD/abtest/w$w.so timeout 900 python -m pytest tests/test_gpu_ssim_cert.py -q -x 2>&1 | tail -1; done
