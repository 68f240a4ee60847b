python tools/ab_concurrent.py C2 C3
