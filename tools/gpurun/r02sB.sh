python tools/ab_time.py C2 abtest/g2.so abtest/g3.so
python tools/ab_time.py C3 abtest/g2.so abtest/g3.so
for v in g2 g3; do
  CZC_LIB=$PWD/abtest/$v.so timeout 600 python bench.py --steps 3 --warmup 2 --no-e2e --no-extra --no-f64 --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$v', d['value'], d['ms_per_step'], d['per_pattern_ms'], d['ssim_exact_windows'])"
done
CZC_LIB=$PWD/abtest/g3.so timeout 900 python -m pytest tests/test_gpu_ssim_cert.py -q -x -s 2>&1 | grep -E "exact recomputes|passed|failed" | tail -12
