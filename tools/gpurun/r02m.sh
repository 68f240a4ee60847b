python tools/ab_time.py C2 abtest/base.so abtest/stub.so
python tools/ab_time.py C3 abtest/base.so abtest/stub.so
