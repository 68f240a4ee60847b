python tools/ab_time.py C3 abtest/rs3.so abtest/rs4.so abtest/rs6.so abtest/mc2k.so
for v in rs3 rs4 rs6 mc2k; do
  CZC_LIB=$PWD/abtest/$v.so timeout 600 python bench.py --steps 3 --warmup 2 --no-e2e --no-extra --no-f64 --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$v', d['value'], d['ms_per_step'], d['per_pattern_ms'], d['ssim_exact_windows'])"
done
for v in rs4 rs6; do CZC_LIB=$PWD/abtest/$v.so timeout 900 python -m pytest tests/test_gpu_ssim_cert.py -q -x -s 2>&1 | grep -E "exact recomputes|passed|failed"; done
