mkdir -p gpurun_out
python -m paper_conf_cluster_yudgtc21_b200.build > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -f -k regex:"deriv3|ac_plane|p1_kernel" -o gpurun_out/prof_r02y python tools/ncu_target.py C3 1 > gpurun_out/ncu_r02y.log 2>&1
for k in deriv3_kernel ac_plane p1_kernel; do
  ncu -i gpurun_out/prof_r02y.ncu-rep --page source --csv --kernel-name regex:$k > gpurun_out/r02y_${k}_source.csv 2>/dev/null
done
rm -f gpurun_out/prof_r02y.ncu-rep
ls -la gpurun_out/ | grep r02y
