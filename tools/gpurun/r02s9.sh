for c in C3 C2 C2q; do for v in old ra1 ra1rs2; do CZC_LIB=$PWD/abtest/$v.so python tools/c3_flags.py $c 2>&1 | tail -1; done; done
