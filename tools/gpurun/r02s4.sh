# long SSIM z-chunks (+ resync every 3 w): A/B on C2 / C3, C5 bench lines, SSIM parity with lc
python tools/ab_time.py C2 abtest/base.so abtest/lc.so abtest/lc_rs3.so
python tools/ab_time.py C3 abtest/base.so abtest/lc.so abtest/lc_rs3.so
for v in base lc lc_rs3; do
  CZC_LIB=$PWD/abtest/$v.so timeout 600 python bench.py --steps 3 --warmup 2 --no-e2e --no-extra --no-f64 --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$v', d['value'], d['ms_per_step'], d['per_pattern_ms'])"
done
CZC_LIB=$PWD/abtest/lc_rs3.so timeout 900 python -m pytest tests/test_gpu_ssim_cert.py -q -x 2>&1 | tail -1
CZC_LIB=$PWD/abtest/lc.so timeout 900 python -m pytest tests/test_gpu_ssim_cert.py tests/test_gpu_parity.py -q -x 2>&1 | tail -1
