python tools/ab_time.py C2 abtest/notm.so abtest/tm2.so abtest/tm3.so
python tools/ab_time.py C3 abtest/notm.so abtest/tm2.so abtest/tm3.so
for v in notm tm2 tm3; do
  CZC_LIB=$PWD/abtest/$v.so timeout 600 python bench.py --steps 3 --warmup 2 --no-e2e --no-extra --no-f64 --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$v', d['value'], d['ms_per_step'], d['per_pattern_ms'], d['ssim_exact_windows'])"
done
CZC_LIB=$PWD/abtest/tm3.so timeout 900 python -m pytest tests/test_gpu_ssim_cert.py -q -x 2>&1 | tail -1
