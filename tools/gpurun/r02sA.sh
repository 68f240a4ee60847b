python -m paper_conf_cluster_yudgtc21_b200.build > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_ssim_cert.py tests/test_gpu_parity.py -q -x -s -k "tall or loopback" 2>&1 | grep -E "tall|passed|failed|Error" | tail -8
timeout 600 python bench.py --steps 5 --warmup 3 --no-e2e --no-f64 --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['ms_per_step'], d['per_pattern_ms'], d['ssim_exact_windows'], {k: (v['value'], v['ssim_exact_windows']) for k, v in d['other_configs'].items()})"
