timeout 1500 python -m pytest tests -m gpu -q -x --deselect tests/test_gpu_parity.py::test_full_size_2048_cubed_smooth_pair 2>&1 | tail -2
timeout 600 python -m pytest tests/test_gpu_parity.py -q -k "nccl" 2>&1 | tail -2
