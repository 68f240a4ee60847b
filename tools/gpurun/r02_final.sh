# One GPU call that refreshes every measurement the round reports (TAG = $1).
set -u
TAG=${1:-r02z}
mkdir -p gpurun_out
python -m paper_conf_cluster_yudgtc21_b200.build > gpurun_out/build_${TAG}.log 2>&1 || { tail gpurun_out/build_${TAG}.log; exit 1; }
timeout 2400 python -m pytest tests -m gpu -q -s -x > gpurun_out/pytest_gpu_${TAG}.log 2>&1; tail -3 gpurun_out/pytest_gpu_${TAG}.log
grep -E "C5 2048|oracle over|exact recomputes|worst window" gpurun_out/pytest_gpu_${TAG}.log | head -30
timeout 600 python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke_${TAG}.log 2>&1; tail -1 gpurun_out/smoke_${TAG}.log
timeout 1200 python bench.py > gpurun_out/bench_${TAG}.json 2> gpurun_out/bench_${TAG}.err; tail -c 400 gpurun_out/bench_${TAG}.json
timeout 900 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_ref_${TAG}.json 2> gpurun_out/bench_ref_${TAG}.err
timeout 1500 ncu --metrics gpu__time_duration.sum --clock-control none --kernel-name-base demangled -k regex:czc:: -c 200 --csv \
    --log-file gpurun_out/launches_${TAG}.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-f64 --no-extra > gpurun_out/ncu_bench_${TAG}.log 2>&1
timeout 1500 ncu --set full --clock-control none --import-source on -f -o gpurun_out/prof_${TAG} python tools/ncu_target.py C3 1 > gpurun_out/ncu_full_${TAG}.log 2>&1
python tools/ncu_summary.py gpurun_out/${TAG}_ncu gpurun_out/prof_${TAG}.ncu-rep --launches gpurun_out/launches_${TAG}.csv > /dev/null 2>&1; cat gpurun_out/${TAG}_ncu.md
ncu -i gpurun_out/prof_${TAG}.ncu-rep --page source --csv --kernel-name regex:p3_kernel > gpurun_out/${TAG}_p3_source.csv 2>/dev/null
rm -f gpurun_out/prof_${TAG}.ncu-rep
for tool in; do   # compute-sanitizer is closed on the GPU pool (round 2); logs of r02w stay
  timeout 1500 compute-sanitizer --tool $tool --print-limit 50 python tools/sanitize_target.py > gpurun_out/sanitize_${tool}_${TAG}.log 2>&1
  echo "$tool: $(tail -1 gpurun_out/sanitize_${tool}_${TAG}.log)"
done
