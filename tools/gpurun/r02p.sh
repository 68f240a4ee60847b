python tools/ab_time.py C3 abtest/base.so abtest/unit.so
python tools/ab_time.py C2 abtest/base.so abtest/unit.so
CZC_LIB=$PWD/abtest/unit.so timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "parity_configs or misaligned or sign_flip or full_size_nyx or f64_parity or pdf" 2>&1 | tail -2
