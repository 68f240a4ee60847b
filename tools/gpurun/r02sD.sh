mkdir -p gpurun_out
python -m paper_conf_cluster_yudgtc21_b200.build > /dev/null 2>&1
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/r02sD_pytest.log 2>&1; tail -2 gpurun_out/r02sD_pytest.log
timeout 300 python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -1
timeout 1200 python bench.py > gpurun_out/bench_r02sD.json 2> gpurun_out/bench_r02sD.err; python -c "
import json; d=json.load(open('gpurun_out/bench_r02sD.json')); print(d['value'], d['ms_per_step'], d['per_pattern_ms'], d['ssim_exact_windows'], d['e2e']['value'], d['float64_inputs']['value'], {k: (v.get('value'), v.get('ssim_exact_windows'), v.get('error')) for k, v in d['other_configs'].items()}, d['clocks'])"
