TAG=r01e
mkdir -p gpurun_out
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
    --log-file gpurun_out/launches_${TAG}.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-f64 > gpurun_out/ncu_bench_${TAG}.log 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -f -o gpurun_out/prof_${TAG} \
    python tools/ncu_target.py C2 1 > gpurun_out/ncu_full_${TAG}.log 2>&1
python tools/ncu_summary.py gpurun_out/${TAG}_ncu gpurun_out/prof_${TAG}.ncu-rep \
    --launches gpurun_out/launches_${TAG}.csv --dominant P3_ssim p3_kernel > gpurun_out/sum.log 2>&1
ncu -i gpurun_out/prof_${TAG}.ncu-rep --page source --csv --kernel-name regex:p3_kernel > gpurun_out/${TAG}_p3_source.csv 2>/dev/null
ls -la gpurun_out/prof_${TAG}.ncu-rep
[ "$(stat -c %s gpurun_out/prof_${TAG}.ncu-rep)" -gt 40000000 ] && rm -f gpurun_out/prof_${TAG}.ncu-rep
du -sh gpurun_out; tail -12 gpurun_out/sum.log
