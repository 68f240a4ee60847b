CZC_LIB=$PWD/abtest/tm.so timeout 120 python tools/dbg_g3.py 2>&1 | tail -3 || exit 1
CZC_LIB=$PWD/abtest/notm.so timeout 120 python tools/dbg_g3.py 2>&1 | tail -2
CZC_LIB=$PWD/abtest/tm.so timeout 600 python -m pytest tests/test_gpu_ssim_cert.py -q -x 2>&1 | tail -2
python tools/ab_time.py C2 abtest/notm.so abtest/tm.so
python tools/ab_time.py C3 abtest/notm.so abtest/tm.so
for v in notm tm; do
  CZC_LIB=$PWD/abtest/$v.so timeout 600 python bench.py --steps 3 --warmup 2 --no-e2e --no-extra --no-f64 --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$v', d['value'], d['ms_per_step'], d['per_pattern_ms'], d['ssim_exact_windows'])"
done
