set -x
timeout 900 python -m pytest tests/test_gpu_ssim_cert.py -q -s 2>&1 | grep -E "exact|worst|passed|failed|Error|assert" | head -60
timeout 1500 python -m pytest tests -m gpu -q -x 2>&1 | tail -15
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/bench_r02b.json 2> gpurun_out/bench_r02b.err; tail -c 5000 gpurun_out/bench_r02b.json; tail -5 gpurun_out/bench_r02b.err
