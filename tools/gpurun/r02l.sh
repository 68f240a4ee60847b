python tools/ab_time.py C2 abtest/pts2.so abtest/pts3.so abtest/pts4.so
python tools/ab_time.py C3 abtest/pts2.so abtest/pts3.so abtest/pts4.so
for P in 3 4; do CZC_LIB=$PWD/abtest/pts$P.so timeout 900 python -m pytest tests/test_gpu_deriv_points.py tests/test_gpu_parity.py -q -x -k "points or parity_configs or loopback" 2>&1 | tail -1; done
