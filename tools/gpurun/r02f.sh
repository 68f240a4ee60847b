set -x
timeout 900 python -m pytest tests/test_gpu_ssim_cert.py tests/test_gpu_parity.py -q -x 2>&1 | tail -3
timeout 300 python tools/quick_time.py C2 2>&1 | grep -E "SSIM|DERIV"
timeout 300 python tools/quick_time.py C3 2>&1 | grep -E "SSIM|DERIV"
