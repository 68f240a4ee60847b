python tools/ab_time.py C2 abtest/base.so abtest/lines.so
python tools/ab_time.py C3 abtest/base.so abtest/lines.so
CZC_LIB=$PWD/abtest/lines.so timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "lags or plane_tile or parity_configs or loopback or misaligned_3d or full_size_nyx" 2>&1 | tail -2
