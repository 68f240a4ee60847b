python tools/ab_time.py C2 abtest/g2.so abtest/g2n.so abtest/g3n.so
python tools/ab_time.py C3 abtest/g2.so abtest/g2n.so abtest/g3n.so
CZC_LIB=$PWD/abtest/g3n.so python tools/dbg_g3.py 2>&1 | tail -2
CZC_LIB=$PWD/abtest/g3n.so timeout 900 python -m pytest tests/test_gpu_ssim_cert.py -q -x 2>&1 | tail -1
