mkdir -p gpurun_out
for v in base s3; do
CZC_LIB=$PWD/abtest/$v.so timeout 600 ncu --set full --clock-control none --import-source on -f -k regex:"p3" -c 1 -o gpurun_out/p3_$v python tools/ncu_target.py C2 1 > gpurun_out/ncu_p3_$v.log 2>&1
ncu -i gpurun_out/p3_$v.ncu-rep --page raw --csv > gpurun_out/p3_${v}_raw.csv 2>/dev/null
ncu -i gpurun_out/p3_$v.ncu-rep --page source --csv --print-source sass > gpurun_out/p3_${v}_sass.csv 2>/dev/null
done
rm -f gpurun_out/*.ncu-rep; ls -la gpurun_out
