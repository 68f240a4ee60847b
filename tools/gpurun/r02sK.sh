python -m paper_conf_cluster_yudgtc21_b200.build > /dev/null 2>&1
timeout 1200 python -m pytest tests -m gpu -q -x 2>&1 | tail -1
python tools/ab_time.py C3 abtest/sB.so abtest/sA.so
for v in sB sA; do
  CZC_LIB=$PWD/abtest/$v.so timeout 600 python bench.py --steps 3 --warmup 2 --no-e2e --no-extra --no-f64 --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$v', d['value'], d['ms_per_step'], d['per_pattern_ms'])"
done
