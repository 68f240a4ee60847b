#!/bin/bash
# SASS source pages (executed instructions + stall samples per instruction) of the pattern
# kernels of one C2 assessment, exported as CSV into gpurun_out/ (the .ncu-rep stays on the box).
# usage (on the box): bash tools/ncu_sources.sh TAG
TAG=${1:-src}
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -f -o /tmp/src_${TAG} \
    python tools/ncu_target.py C2 1 > gpurun_out/ncu_src_${TAG}.log 2>&1
for k in p1_kernel deriv3_kernel ac_zwalk_tma ac_plane p3_kernel; do
  ncu -i /tmp/src_${TAG}.ncu-rep --page source --csv --kernel-name regex:$k > gpurun_out/${TAG}_${k}_source.csv 2>/dev/null
done
ls -la gpurun_out/${TAG}_*
