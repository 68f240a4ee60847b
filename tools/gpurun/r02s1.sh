# strip SSIM kernel: parity (SSIM tests) with the default build (H=3) and H=4, then A/B timing
python -m paper_conf_cluster_yudgtc21_b200.build > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_ssim_cert.py -q -x 2>&1 | tail -3
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "ssim or window or extents or parity_configs" 2>&1 | tail -3
CZC_LIB=$PWD/abtest/s4.so timeout 900 python -m pytest tests/test_gpu_ssim_cert.py -q -x 2>&1 | tail -2
python tools/ab_time.py C2 abtest/base.so abtest/s3.so abtest/s4.so
python tools/ab_time.py C3 abtest/base.so abtest/s3.so abtest/s4.so
