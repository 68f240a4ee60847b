set -x
nproc; free -g | head -2; lscpu | grep -E "Model name|Socket|Core|Thread|NUMA node\(s\)"; nvidia-smi --query-gpu=name,memory.total,clocks.max.sm --format=csv
timeout 900 python -m pytest tests/test_gpu_ssim_cert.py -q -s 2>&1 | tail -40
timeout 1500 python -m pytest tests -m gpu -q -x 2>&1 | tail -15
timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-f64 --no-cpu-baseline > gpurun_out/bench_r02a.json 2> gpurun_out/bench_r02a.err; tail -c 3000 gpurun_out/bench_r02a.json
