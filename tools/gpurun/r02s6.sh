python tools/ab_time.py C2 abtest/base2.so abtest/acrows.so
python tools/ab_time.py C3 abtest/base2.so abtest/acrows.so
for v in base2 acrows; do
  CZC_LIB=$PWD/abtest/$v.so timeout 600 python bench.py --steps 3 --warmup 2 --no-e2e --no-extra --no-f64 --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$v', d['value'], d['ms_per_step'], d['per_pattern_ms'])"
done
CZC_LIB=$PWD/abtest/acrows.so timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "ac or autocorr or lag or parity_configs or full_size_c" 2>&1 | tail -1
