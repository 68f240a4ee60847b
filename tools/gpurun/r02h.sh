python tools/ab_time.py C2 abtest/base.so abtest/tree.so abtest/tree_rs2.so
python tools/ab_time.py C3 abtest/base.so abtest/tree.so abtest/tree_rs2.so
CZC_LIB=$PWD/abtest/tree_rs2.so timeout 900 python -m pytest tests/test_gpu_ssim_cert.py -q -s 2>&1 | grep -E "exact|passed|failed" | head -30
