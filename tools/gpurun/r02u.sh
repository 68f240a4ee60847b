timeout 600 python -m pytest tests/test_gpu_parity.py -q -k "nccl or loopback" 2>&1 | tail -3
