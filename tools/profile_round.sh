#!/bin/bash
# One GPU call that refreshes every measurement the round reports:
#   bench (ours + reference arm), ncu launch list of the bench command, ncu --set full of one
#   C2 assessment (all kernels), SASS-level source pages stay in the .ncu-rep.
# usage (on the box, from the repo root): bash tools/profile_round.sh TAG
set -u
TAG=${1:-r01}
mkdir -p gpurun_out
python -m paper_conf_cluster_yudgtc21_b200.build > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 1; }
timeout 600 python bench.py > gpurun_out/bench_${TAG}.json 2> gpurun_out/bench_${TAG}.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_ref_${TAG}.json 2> gpurun_out/bench_ref_${TAG}.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
    --log-file gpurun_out/launches_${TAG}.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-f64 > gpurun_out/ncu_bench_${TAG}.log 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -f -o gpurun_out/prof_${TAG} \
    python tools/ncu_target.py C2 1 > gpurun_out/ncu_full_${TAG}.log 2>&1
# summaries on the box (the full report can exceed what gpurun copies back)
python tools/ncu_summary.py gpurun_out/${TAG}_ncu gpurun_out/prof_${TAG}.ncu-rep \
    --launches gpurun_out/launches_${TAG}.csv --dominant P3_ssim p3_kernel > /dev/null 2>&1
ncu -i gpurun_out/prof_${TAG}.ncu-rep --page source --csv --kernel-name regex:p3_kernel \
    > gpurun_out/${TAG}_p3_source.csv 2>/dev/null
[ "$(stat -c %s gpurun_out/prof_${TAG}.ncu-rep)" -gt 40000000 ] && rm -f gpurun_out/prof_${TAG}.ncu-rep
cat gpurun_out/bench_${TAG}.json gpurun_out/bench_ref_${TAG}.json
