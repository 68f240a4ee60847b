timeout 1200 python -m pytest tests/test_gpu_deriv_points.py -q -x 2>&1 | tail -15
timeout 2400 python -m pytest tests -m gpu -q -x --deselect tests/test_gpu_parity.py::test_full_size_2048_cubed_smooth_pair 2>&1 | tail -3
timeout 300 python tools/quick_time.py C2 2>&1 | grep -E "ALL"
