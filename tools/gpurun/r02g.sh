set -x
mkdir -p gpurun_out
timeout 1800 python -m pytest tests/test_gpu_parity.py -q -s -k "2048_cubed_smooth" 2>&1 | tail -6
timeout 900 python bench.py > gpurun_out/bench_r02g.json 2> gpurun_out/bench_r02g.err; tail -c 600 gpurun_out/bench_r02g.json; tail -3 gpurun_out/bench_r02g.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_ref_r02g.json 2> gpurun_out/bench_ref_r02g.err; cat gpurun_out/bench_ref_r02g.json
timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_r02g.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-f64 --no-extra > gpurun_out/ncu_bench_r02g.log 2>&1
tail -2 gpurun_out/ncu_bench_r02g.log
timeout 1500 ncu --set full --clock-control none --import-source on -f -o gpurun_out/prof_r02g python tools/ncu_target.py C3 1 > gpurun_out/ncu_full_r02g.log 2>&1
python tools/ncu_summary.py gpurun_out/r02g_ncu gpurun_out/prof_r02g.ncu-rep --launches gpurun_out/launches_r02g.csv > /dev/null 2>&1; cat gpurun_out/r02g_ncu.md
ncu -i gpurun_out/prof_r02g.ncu-rep --page source --csv --kernel-name regex:p3_kernel > gpurun_out/r02g_p3_source.csv 2>/dev/null
rm -f gpurun_out/prof_r02g.ncu-rep
