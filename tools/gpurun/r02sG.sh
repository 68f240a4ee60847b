python tools/ab_time.py C2 abtest/du0.so abtest/du1.so abtest/du2.so abtest/du3.so
python tools/ab_time.py C3 abtest/du0.so abtest/du1.so abtest/du2.so abtest/du3.so
