# HEAD verification (pytest -m gpu, smoke) + ncu source pages of the derivative and AC kernels
mkdir -p gpurun_out
python -m paper_conf_cluster_yudgtc21_b200.build > gpurun_out/build_s3.log 2>&1 || { tail gpurun_out/build_s3.log; exit 1; }
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/r02s3_pytest_gpu.log 2>&1; tail -3 gpurun_out/r02s3_pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02s3_smoke.log 2>&1; tail -2 gpurun_out/r02s3_smoke.log
timeout 600 ncu --set full --clock-control none --import-source on -f -k regex:"deriv3|ac_plane|ac_zwalk|p1_kernel" -c 4 -o gpurun_out/p2 python tools/ncu_target.py C2 1 > gpurun_out/ncu_p2.log 2>&1
for k in deriv3_kernel ac_plane ac_zwalk p1_kernel; do
  ncu -i gpurun_out/p2.ncu-rep --page source --csv --print-source sass --kernel-name regex:$k > gpurun_out/p2_${k}_sass.csv 2>/dev/null
done
ncu -i gpurun_out/p2.ncu-rep --page raw --csv > gpurun_out/p2_raw.csv 2>/dev/null
rm -f gpurun_out/*.ncu-rep
ls -la gpurun_out | grep -v p3_
