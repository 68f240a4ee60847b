for v in old ra0 ra1; do echo "== $v"; CZC_LIB=$PWD/abtest/$v.so timeout 900 python -m pytest tests/test_gpu_ssim_cert.py -q -x -s -k tall 2>&1 | grep -E "tall|passed|failed"; done
