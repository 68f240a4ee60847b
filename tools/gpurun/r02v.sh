python tools/ab_time.py C3 abtest/base.so abtest/cert2.so
python tools/ab_time.py C2 abtest/base.so abtest/cert2.so
CZC_LIB=$PWD/abtest/cert2.so timeout 900 python -m pytest tests/test_gpu_ssim_cert.py -q -x -s 2>&1 | grep -E "exact|passed|failed|Error" | tail -30
