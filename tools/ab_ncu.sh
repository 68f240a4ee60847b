#!/bin/bash
# Per-kernel device times (ncu gpu__time_duration, cold-cache serialised) for several library
# builds on one config.  usage (on the box): bash tools/ab_ncu.sh CONFIG LIB...
cfg=$1; shift
for lib in "$@"; do
  echo "== $lib"
  CZC_LIB=$(realpath $lib) ncu --metrics gpu__time_duration.sum --clock-control none -s 12 -c 12 --csv \
    python tools/ncu_target.py $cfg 3 2>/dev/null | python -c "
import csv,sys,collections
rows=[r for r in csv.reader(sys.stdin) if len(r)>10]
h=rows[0]; ki=h.index('Kernel Name'); vi=h.index('Metric Value')
d=collections.defaultdict(list)
for r in rows[1:]:
    d[r[ki][:40]].append(float(r[vi]))
for k,v in d.items(): print(f'{k:40s} n={len(v)} min={min(v)/1e3:.1f}us')
"
done
